"""Pins for the oracle's structural steps (O2 levels, O3 sparsify, O4 indicator, O5 Alg. 2).

Every expected value here comes from the paper (golden fixture, cited), a closed
form, an invariant, or brute force — never from the oracle itself.
"""
import itertools
import math
import os

import numpy as np
import pytest

import gen
import oracle

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _read_golden(name):
    d = {}
    with open(os.path.join(GOLD, name)) as f:
        for line in f:
            if line.startswith("#") or not line.strip():
                continue
            k, *v = line.split()
            d[k] = v
    return d


# --------------------------------------------------------------------- P1
def test_fig1_worked_example_levels():
    """PAPER.md L211-283, Fig. 1: 3 wavefronts, 2 after dropping f."""
    g = _read_golden("fig1_wavefronts.txt")
    rp = np.array(g["rowptr"], np.int64)
    col = np.array(g["col"], np.int32)
    L = gen.CSR(4, rp, col, np.arange(1, 8, dtype=np.float64))
    w, lev = oracle.levels_lower(L)
    assert w == int(g["wavefronts"][0])
    assert lev.tolist() == [int(x) for x in g["levels"]]
    # drop f (entry named 'f' in Fig. 1b order)
    k = g["names"].index(g["drop"][0])
    keep = np.ones(7, bool)
    keep[k] = False
    rp2 = np.array([0] + [int(np.sum(keep[: rp[i + 1]])) for i in range(4)], np.int64)
    L2 = gen.CSR(4, rp2, col[keep], np.arange(1, 8, dtype=np.float64)[keep])
    w2, lev2 = oracle.levels_lower(L2)
    assert w2 == int(g["wavefronts_after"][0])
    assert lev2.tolist() == [int(x) for x in g["levels_after"]]


def test_fig1_symmetric_drop_selects_f():
    """The magnitude rule removes the smallest |a_ij|: with f the
    smallest off-diagonal of the symmetrised Fig. 1 matrix and one drop, the
    wavefronts go 3 -> 2 exactly as Fig. 1d."""
    d = np.zeros((4, 4))
    # a..g of Fig. 1a: a,b,d,g diagonal; c=(2,0) e=(3,0) f=(3,2)
    d[0, 0], d[1, 1], d[2, 2], d[3, 3] = 10.0, 10.0, 10.0, 10.0
    d[2, 0] = d[0, 2] = -2.0   # c
    d[3, 0] = d[0, 3] = -3.0   # e
    d[3, 2] = d[2, 3] = -0.5   # f (smallest)
    A = gen.from_dense(d)
    assert oracle.levels_lower(A)[0] == 3
    # N_L = 7 (lower triangle incl. diagonal, reading A1); floor(15*7/100) = 1
    Ah, S, m = oracle.sparsify(A, 15.0)
    assert m == 1
    assert oracle.levels_lower(Ah)[0] == 2
    assert S.to_dense()[3, 2] == -0.5 and S.to_dense()[2, 3] == -0.5


# --------------------------------------------------------------------- P2 / P4
def _brute_longest(n, deps):
    """longest path (in edges) ending at each vertex, by memoised DFS."""
    memo = {}

    def f(i):
        if i not in memo:
            memo[i] = 0 if not deps[i] else 1 + max(f(j) for j in deps[i])
        return memo[i]

    return [f(i) for i in range(n)]


def _deps_lower(M):
    return [[int(j) for j in M.col[M.row_ptr[i]:M.row_ptr[i + 1]] if j < i] for i in range(M.n)]


@pytest.mark.parametrize("nx,ny", [(7, 5), (16, 9), (32, 32), (1, 13)])
def test_levels_poisson2d_closed_form(nx, ny):
    A = gen.make("poisson2d", nx, ny)
    w, lev = oracle.levels_lower(A)
    assert w == nx + ny - 1
    # natural-order grid DAG: level of (x, y) = x + y
    x, y = np.arange(A.n) % nx, np.arange(A.n) // nx
    assert np.array_equal(lev, x + y)


@pytest.mark.parametrize("dims", [(6, 5, 4), (8, 8, 8)])
def test_levels_poisson3d_closed_form(dims):
    A = gen.make("poisson3d", *dims)
    assert oracle.levels_lower(A)[0] == sum(dims) - 2


@pytest.mark.parametrize("dims", [(5, 4, 3), (6, 6, 6)])
def test_levels_27pt_closed_form(dims):
    nx, ny, nz = dims
    A = gen.make("fem_q1", nx, ny, nz, 3)
    w, lev = oracle.levels_lower(A)
    assert w == nx + 2 * ny + 4 * nz - 6
    assert lev.tolist() == _brute_longest(A.n, _deps_lower(A))


def test_levels_random_dags_bruteforce():
    rng = np.random.default_rng(0)
    for trial in range(40):
        n = int(rng.integers(1, 50))
        d = np.zeros((n, n))
        mask = rng.random((n, n)) < rng.uniform(0.02, 0.3)
        d[mask] = 1.0
        d = np.tril(d, -1)
        d = d + d.T + np.eye(n)
        M = gen.from_dense(d)
        w, lev = oracle.levels_lower(M)
        bl = _brute_longest(n, _deps_lower(M))
        assert lev.tolist() == bl
        assert w == (max(bl) + 1 if n else 0)
        # upper: reverse the numbering
        wu, levu = oracle.levels_upper(M)
        deps_u = [[int(j) for j in M.col[M.row_ptr[i]:M.row_ptr[i + 1]] if j > i] for i in range(n)]
        memo = {}

        def fu(i):
            if i not in memo:
                memo[i] = 0 if not deps_u[i] else 1 + max(fu(j) for j in deps_u[i])
            return memo[i]

        assert levu.tolist() == [fu(i) for i in range(n)]


def test_level_sets_partition_and_order():
    A = gen.make("aniso_layered", 24, 17, 4)
    w, lev = oracle.levels_lower(A)
    ptr, rows = oracle.level_sets(lev, w)
    assert ptr[0] == 0 and ptr[-1] == A.n
    assert sorted(rows.tolist()) == list(range(A.n))
    for l in range(w):
        seg = rows[ptr[l]:ptr[l + 1]]
        assert np.all(lev[seg] == l)
        assert np.all(np.diff(seg) > 0)        # ascending inside a level (A17)


def test_levels_symmetric_pattern_upper_equals_lower():
    A = gen.make("fem_q1", 5, 6, 4, 7)
    wl, _ = oracle.levels_lower(A)
    wu, _ = oracle.levels_upper(A)
    assert wl == wu


# --------------------------------------------------------------------- P5
@pytest.mark.parametrize("fam,params", [("poisson2d", (16, 12)), ("aniso_layered", (40, 33, 4)),
                                        ("fem_q1", (5, 5, 5, 3))])
@pytest.mark.parametrize("t", [1.0, 5.0, 10.0, 37.5])
def test_sparsify_invariants(fam, params, t):
    A = gen.make(fam, *params)
    Ah, S, m = oracle.sparsify(A, t)
    Ad, Ahd, Sd = A.to_dense(), Ah.to_dense(), S.to_dense()
    # A = Ahat + S, bitwise, with disjoint patterns
    assert np.array_equal(Ahd + Sd, Ad)
    assert Ah.nnz + S.nnz == A.nnz
    assert np.array_equal(Sd, Sd.T) and np.array_equal(Ahd, Ahd.T)
    assert np.all(np.diag(Sd) == 0)
    # count rule (A1, A2): m = floor(t * nnz(tril A) / 100)
    NL = int(np.count_nonzero(np.tril(Ad != 0)))
    assert m == min(math.floor(t * NL / 100.0), int(np.count_nonzero(np.tril(Ad != 0, -1))))
    assert S.nnz == 2 * m
    # every dropped |a| <= every kept strictly-lower |a|; ties resolved row-major (A4)
    lowA = [(abs(A.val[q]), q) for i in range(A.n) for q in range(A.row_ptr[i], A.row_ptr[i + 1]) if A.col[q] < i]
    order = sorted(lowA)
    dropped = set(q for _, q in order[:m])
    for i in range(A.n):
        for q in range(A.row_ptr[i], A.row_ptr[i + 1]):
            j = A.col[q]
            if j < i:
                assert (Sd[i, j] != 0) == (q in dropped)


# --------------------------------------------------------------------- P6
@pytest.mark.parametrize("nx,ny,t", [(32, 32, 10.0), (32, 32, 5.0), (20, 30, 1.0), (64, 8, 10.0)])
def test_indicator_poisson2d_closed_form(nx, ny, t):
    A = gen.make("poisson2d", nx, ny)
    Ah, S, m = oracle.sparsify(A, t)
    ind, parts = oracle.indicator(Ah, S, 0)
    n = nx * ny
    nnz_off = A.nnz - n
    expect = 2.0 * math.sqrt(2 * m) / math.sqrt(16 * n + nnz_off - 2 * m)
    assert ind == pytest.approx(expect, rel=1e-14)
    assert parts["kappa"] == 2.0


def test_indicator_C1_value():
    """C1 at t = 10 gives 0.3486."""
    A = gen.config_matrix("C1")
    Ah, S, m = oracle.sparsify(A, 10.0)
    assert m == 300
    assert oracle.indicator(Ah, S)[0] == pytest.approx(0.3486, abs=5e-5)


def test_indicator_inf_reading_ties_tau_on_poisson():
    """Reading A6 alternative: with inf-norms the Poisson indicator at t=10 is exactly 1 = tau."""
    A = gen.make("poisson2d", 32, 32)
    Ah, S, m = oracle.sparsify(A, 10.0)
    ind, parts = oracle.indicator(Ah, S, 1)
    # all |a_ij| = 1 tie, so the 300 drops are the first strictly-lower entries in
    # row-major order; interior row 40 loses both lower neighbours and (as mirrors
    # of rows 41 and 72) both upper ones: ||S||_inf = 4, kappa = 8/4, ||Ahat||_inf = 8
    assert parts["kappa"] == 2.0 and parts["s_norm"] == 4.0
    assert ind == 1.0


# --------------------------------------------------------------------- P7
def test_alg2_branch_accept_first_ratio():
    A = gen.make("poisson2d", 32, 32)
    Ah, idx, tr, wA = oracle.alg2(A, omega=5.0)
    assert idx == 0 and tr[0]["ind"] < 1.0 and tr[0]["red"] >= 5.0
    assert Ah.nnz == A.nnz - 2 * oracle.drop_count(A, 10.0)


def test_alg2_branch_reject_tau_then_accept():
    A = gen.make("aniso_layered", 128, 128, 4)
    Ah, idx, tr, wA = oracle.alg2(A)
    assert wA == 255
    assert tr[0]["ind"] > 1.0 and tr[0]["w"] == -1          # t = 10 fails the indicator
    assert idx == 1 and tr[1]["ind"] < 1.0 and tr[1]["red"] >= 10.0
    assert oracle.levels_lower(Ah)[0] == 128 + 14            # N + 14


def test_alg2_branch_all_fail_tau_returns_most_aggressive():
    A = gen.make("poisson2d", 32, 32)
    Ah, idx, tr, wA = oracle.alg2(A, tau=0.05)
    assert len(tr) == 3 and all(x["ind"] > 0.05 for x in tr)
    ref, _, _ = oracle.sparsify(A, 10.0)                     # Alg. 2 line 6: A - S_10
    assert np.array_equal(Ah.col, ref.col) and np.array_equal(Ah.row_ptr, ref.row_ptr)


def test_alg2_branch_never_omega_returns_last():
    A = gen.make("poisson2d", 32, 32)
    Ah, idx, tr, wA = oracle.alg2(A)
    assert idx == 2 and all(x["red"] < 10.0 for x in tr)
    assert [x["w"] for x in tr] == [58, 61, 63]
    ref, _, _ = oracle.sparsify(A, 1.0)
    assert np.array_equal(Ah.col, ref.col)


def test_alg2_denominator_reading():
    """A8: Eq. 7 divides by w_A, Alg. 2 line 10 by w_Ahat; both readings selectable."""
    A = gen.make("aniso_layered", 64, 64, 4)
    _, _, tr0, wA = oracle.alg2(A, denom_mode=0)
    _, _, tr1, _ = oracle.alg2(A, denom_mode=1)
    w = tr0[-1]["w"]
    assert tr0[-1]["red"] == pytest.approx(100.0 * (wA - w) / wA)
    assert tr1[-1]["red"] == pytest.approx(100.0 * (wA - w) / w)


# --------------------------------------------------------------------- O1
def test_validate_rejects_bad_inputs():
    A = gen.make("poisson2d", 4, 4)
    assert oracle.validate(A) == 0
    bad = gen.CSR(A.n, A.row_ptr.copy(), A.col.copy(), A.val.copy())
    bad.val[1] = -2.0                       # breaks symmetry
    assert oracle.validate(bad) == oracle.BAD_MATRIX
    bad = gen.CSR(A.n, A.row_ptr.copy(), A.col.copy(), A.val.copy())
    bad.col[0], bad.col[1] = bad.col[1], bad.col[0]   # unsorted
    assert oracle.validate(bad) == oracle.BAD_MATRIX
    bad = gen.CSR(A.n, A.row_ptr.copy(), A.col.copy(), A.val.copy())
    bad.val[0] = float("nan")
    assert oracle.validate(bad) == oracle.BAD_MATRIX
    d = A.to_dense()
    d[3, 3] = 0.0
    z = gen.from_dense(d)
    z.val[z.row_ptr[3]:z.row_ptr[4]][z.col[z.row_ptr[3]:z.row_ptr[4]] == 3] = 0.0
    assert oracle.validate(z) == oracle.BAD_MATRIX


def test_generators_exact_symmetry_and_sizes():
    for fam, params, nnz in [("poisson2d", (13, 7), 5 * 13 * 7 - 2 * 13 - 2 * 7),
                             ("poisson3d", (5, 4, 3), 7 * 60 - 2 * (4 * 3 + 5 * 3 + 5 * 4)),
                             ("fem_q1", (6, 5, 4, 3), (6 + 10) * (5 + 8) * (4 + 6)),
                             ("aniso_layered", (33, 17, 4), 5 * 33 * 17 - 2 * 33 - 2 * 17)]:
        A = gen.make(fam, *params)
        assert A.nnz == nnz
        assert oracle.validate(A) == 0
        d = A.to_dense()
        assert np.array_equal(d, d.T)
        assert np.linalg.eigvalsh(d).min() > 0
    # nnz(C3) = 382^3 (27-point on 128^3) without building it
    assert (128 + 2 * 127) ** 3 == 55_742_968
