"""Pins for the oracle's numeric steps (O6 ILU(K) symbolic, O7 numeric ILU,
O9 SpTRSV / SpMV, O10 PCG) against closed forms, library routines and
brute force — never against the oracle itself."""
import math
from collections import deque

import numpy as np
import pytest
import scipy.linalg as sla
import scipy.sparse.linalg as spla

import gen
import oracle


def _pattern_set(M):
    return {(i, int(j)) for i in range(M.n) for j in M.col[M.row_ptr[i]:M.row_ptr[i + 1]]}


def _random_spd(rng, n, density):
    d = np.zeros((n, n))
    mask = np.tril(rng.random((n, n)) < density, -1)
    d[mask] = -rng.uniform(0.1, 1.0, mask.sum())
    d = d + d.T
    d[np.diag_indices(n)] = np.abs(d).sum(1) + rng.uniform(0.5, 2.0, n)
    return d


# --------------------------------------------------------------------- P11
def test_iluk_5pt_textbook_fill_offsets():
    """Saad: 5-point 2D ILU(1) adds the offsets +-(nx-1) at level 1, ILU(2) adds +-(nx-2) at level 2."""
    nx, ny = 9, 7
    A = gen.make("poisson2d", nx, ny)
    base = {(i, j) for (i, j) in _pattern_set(A)}
    for K, new_offs in [(1, {nx - 1}), (2, {nx - 1, nx - 2})]:
        P, lev = oracle.iluk_symbolic(A, K)
        S = _pattern_set(P)
        assert base <= S
        offs = {abs(i - j) for (i, j) in S - base}
        assert offs == new_offs
        # level of each entry: 0 on A, 1 for +-(nx-1), 2 for +-(nx-2)
        for i in range(P.n):
            for q in range(P.row_ptr[i], P.row_ptr[i + 1]):
                j = int(P.col[q])
                want = 0 if (i, j) in base else (1 if abs(i - j) == nx - 1 else 2)
                assert lev[q] == want


def test_iluk_K0_is_pattern_and_monotone():
    A = gen.make("fem_q1", 5, 4, 4, 3)
    P0, l0 = oracle.iluk_symbolic(A, 0)
    assert _pattern_set(P0) == _pattern_set(A) and np.all(l0 == 0)
    prev = _pattern_set(P0)
    for K in (1, 2, 3):
        PK, _ = oracle.iluk_symbolic(A, K)
        cur = _pattern_set(PK)
        assert prev <= cur
        assert cur == {(j, i) for (i, j) in cur}            # symmetric pattern
        prev = cur


def test_iluk_27pt_interior_row_count_K2():
    """115 nonzeros per interior row of the 27-point ILU(2) factor."""
    A = gen.make("fem_q1", 12, 12, 12, 3)
    P, _ = oracle.iluk_symbolic(A, 2)
    c = (6 - 1) + 12 * ((6 - 1) + 12 * (6 - 1))       # node (6,6,6)
    assert P.row_ptr[c + 1] - P.row_ptr[c] == 115


def _fill_path_levels(d, K):
    """Independent definition (Rose-Tarjan / Hysom-Pothen fill-path theorem):
    (i,j) is in ILU(K) with level l iff the shortest path i->j in G(A) whose
    intermediate vertices are all < min(i,j) has l+1 edges, l <= K."""
    n = d.shape[0]
    adj = [[j for j in range(n) if j != i and d[i, j] != 0] for i in range(n)]
    out = {}
    for i in range(n):
        for j in range(n):
            if i == j:
                out[(i, j)] = 0
                continue
            bound = min(i, j)
            dist = {i: 0}
            dq = deque([i])
            found = None
            while dq:
                v = dq.popleft()
                for u in adj[v]:
                    if u == j:
                        found = dist[v] + 1
                        break
                    if u < bound and u not in dist:
                        dist[u] = dist[v] + 1
                        dq.append(u)
                if found is not None:
                    break
            if found is not None and found - 1 <= K:
                out[(i, j)] = found - 1
    return out


def test_iluk_matches_fill_path_theorem_random():
    rng = np.random.default_rng(1)
    for trial in range(25):
        n = int(rng.integers(3, 28))
        d = _random_spd(rng, n, rng.uniform(0.05, 0.35))
        A = gen.from_dense(d)
        for K in (0, 1, 2, 4):
            P, lev = oracle.iluk_symbolic(A, K)
            got = {(i, int(P.col[q])): int(lev[q]) for i in range(n) for q in range(P.row_ptr[i], P.row_ptr[i + 1])}
            assert got == _fill_path_levels(d, K)


# --------------------------------------------------------------------- P8 / P9 / P10
def test_ilu0_tridiagonal_is_exact_lu():
    n = 40
    rng = np.random.default_rng(2)
    off = -rng.uniform(0.5, 1.0, n - 1)
    dg = 2.5 + rng.uniform(0.0, 0.5, n)
    d = np.diag(dg) + np.diag(off, 1) + np.diag(off, -1)
    A = gen.from_dense(d)
    L, U = oracle.iluk(A, 0)
    # Thomas algorithm (closed form of the tridiagonal LU): u_0 = d_0, l_i = o_i/u_{i-1}, u_i = d_i - l_i o_i
    u = np.zeros(n)
    l = np.zeros(n)
    u[0] = dg[0]
    for i in range(1, n):
        l[i] = off[i - 1] / u[i - 1]
        u[i] = dg[i] - l[i] * off[i - 1]
    Ld, Ud = L.to_dense(), U.to_dense()
    assert np.allclose(np.diag(Ld, -1), l[1:], rtol=1e-15, atol=0)
    assert np.allclose(np.diag(Ud), u, rtol=1e-15, atol=0)
    b, xt = gen.rhs(A)
    r = oracle.pcg(A, L, U, b, 1e-12, 50)
    assert r["k"] == 1 and r["status"] == 0


def test_ilu_product_matches_A_on_pattern():
    """Saad: (L U)_ij = Ahat_ij for (i,j) in the factor pattern (K = 0: pattern(Ahat))."""
    for fam, params, K in [("poisson2d", (12, 9), 0), ("fem_q1", (5, 5, 4, 3), 0),
                           ("fem_q1", (5, 5, 4, 3), 2), ("aniso_layered", (20, 11, 4), 1)]:
        A = gen.make(fam, *params)
        P, _ = oracle.iluk_symbolic(A, K)
        st, L, U, _ = oracle.ilu_numeric(A, P)
        assert st == 0
        LU = (L.to_dense() + np.eye(A.n)) @ U.to_dense()
        Ad = A.to_dense()
        for (i, j) in _pattern_set(P):
            assert abs(LU[i, j] - Ad[i, j]) <= 1e-13 * max(1.0, abs(Ad[i, i]))


def test_iluk_full_level_is_exact_lu():
    """K >= n-1 gives the complete LU; for SPD A: L = C diag(C)^-1, U = diag(C) C^T (C = cholesky)."""
    rng = np.random.default_rng(3)
    for n in (6, 15, 30):
        d = _random_spd(rng, n, 0.2)
        A = gen.from_dense(d)
        L, U = oracle.iluk(A, n)
        C = np.linalg.cholesky(d)
        Lr = C / np.diag(C)[None, :]
        Ur = np.diag(np.diag(C)) @ C.T
        assert np.allclose(L.to_dense() + np.eye(n), Lr, rtol=0, atol=1e-13)
        assert np.allclose(U.to_dense(), Ur, rtol=0, atol=1e-12)


def test_ilu_zero_pivot_reported():
    d = np.array([[1.0, 2.0], [2.0, 4.0]])      # singular: u_11 = 4 - 2*2 = 0
    A = gen.from_dense(d)
    P, _ = oracle.iluk_symbolic(A, 0)
    st, _, _, bad = oracle.ilu_numeric(A, P)
    assert st == oracle.ZERO_PIVOT and bad == 1


# --------------------------------------------------------------------- P13
def test_sptrsv_matches_dense_substitution():
    rng = np.random.default_rng(4)
    A = gen.make("fem_q1", 5, 4, 4, 11)
    L, U = oracle.iluk(A, 1)
    r = rng.standard_normal(A.n)
    y = oracle.sptrsv_lower(L, r)
    z = oracle.sptrsv_upper(U, y)
    yr = sla.solve_triangular(L.to_dense() + np.eye(A.n), r, lower=True, unit_diagonal=True)
    zr = sla.solve_triangular(U.to_dense(), yr, lower=False)
    assert np.allclose(y, yr, rtol=1e-14, atol=1e-14)
    assert np.allclose(z, zr, rtol=1e-13, atol=1e-14)
    p = rng.standard_normal(A.n)
    assert np.allclose(oracle.spmv(A, p), A.to_dense() @ p, rtol=1e-14, atol=1e-14)


# --------------------------------------------------------------------- P14 / P15 / P16
def test_cg_finite_termination_identity_preconditioner():
    """M = I: CG reaches ||r|| < 1e-8 in <= n steps on tiny SPD systems (exact arithmetic: n)."""
    rng = np.random.default_rng(5)
    for n in (4, 8, 12):
        d = _random_spd(rng, n, 0.6)
        A = gen.from_dense(d)
        b, xt = gen.rhs(A)
        r = oracle.pcg(A, None, None, b, 1e-8, 1000)
        assert r["status"] == 0 and r["k"] <= n
        assert np.allclose(r["x"], np.linalg.solve(d, b), atol=1e-7)


def _scipy_pcg_iterates(A, L, U, b, eps, kmax):
    As = A.to_scipy()
    Ls = L.to_scipy()
    Us = U.to_scipy()
    import scipy.sparse as sp
    Lu = Ls + sp.eye(A.n, format="csr")

    def msolve(r):
        y = spla.spsolve_triangular(Lu, r, lower=True, unit_diagonal=True)
        return spla.spsolve_triangular(Us, y, lower=False)

    M = spla.LinearOperator((A.n, A.n), matvec=msolve)
    its = []
    x, info = spla.cg(As, b, rtol=0.0, atol=eps, maxiter=kmax, M=M, callback=lambda xk: its.append(xk.copy()))
    return x, its


@pytest.mark.parametrize("fam,params,K", [("poisson2d", (32, 32), 0), ("aniso_layered", (48, 40, 4), 0),
                                          ("fem_q1", (6, 6, 6, 3), 2)])
def test_pcg_matches_scipy_cg(fam, params, K):
    A = gen.make(fam, *params)
    L, U, _ = oracle.setup(A, mode="alg2", K=K)
    b, xt = gen.rhs(A)
    r = oracle.pcg(A, L, U, b, 1e-8, 1000)
    xs, its = _scipy_pcg_iterates(A, L, U, b, 1e-8, 1000)
    assert abs(len(its) - r["k"]) <= 1
    assert np.linalg.norm(xs - r["x"]) <= 1e-8 * np.linalg.norm(xs) + 1e-9
    # identical iterate at equal k (survey: bit-identical up to rounding)
    kk = min(r["k"], len(its))
    rk = oracle.pcg(A, L, U, b, 0.0, kk)
    assert np.linalg.norm(rk["x"] - its[kk - 1]) <= 1e-12 * np.linalg.norm(its[kk - 1])


def test_pcg_error_bound_poisson():
    """||x - x_true|| <= ||A^-1|| ||b - A x||, lambda_min of the 2D Dirichlet Laplacian in closed form."""
    nx, ny = 40, 30
    A = gen.make("poisson2d", nx, ny)
    L, U, _ = oracle.setup(A, mode="none", K=0)
    b, xt = gen.rhs(A)
    r = oracle.pcg(A, L, U, b, 1e-8, 1000)
    lam = 4 - 2 * math.cos(math.pi / (nx + 1)) - 2 * math.cos(math.pi / (ny + 1))
    true_res = np.linalg.norm(b - oracle.spmv(A, r["x"]))
    assert true_res <= 1.01e-8
    assert np.linalg.norm(r["x"] - xt) <= true_res / lam * (1 + 1e-6)


def test_pcg_forced_k_and_kmax():
    A = gen.make("poisson2d", 16, 16)
    L, U, _ = oracle.setup(A, mode="none", K=0)
    b, _ = gen.rhs(A)
    r = oracle.pcg(A, L, U, b, 0.0, 7)
    assert r["k"] == 7 and r["status"] == 0
    r = oracle.pcg(A, L, U, b, 1e-30, 5)
    assert r["k"] == 5 and r["status"] == oracle.NOT_CONVERGED
    # monotone residual history is not guaranteed for CG, but rhist[0] = ||b|| = 1
    assert r["rhist"][0] == pytest.approx(1.0, rel=1e-15)


def test_pcg_initial_guess_branch_pins():
    """O10's x0 branch (Alg. 1 line 2, r0 = b - A x0; A15), pinned without the oracle:
    (a) x0 = the exact solution of a system whose b is formed exactly (small integers)
        gives r0 = 0, so the test before the first SpMV fires: k = 0, x = x0 bitwise;
    (b) a dense 3x3 SPD matrix: ILU(0) of a full pattern is its exact LU, so from ANY x0
        one iteration lands on x = A^-1 b (closed form of the 3x3 inverse by Cramer's
        rule) — a sign or operand error in r0 = b - A x0 gives a different point;
    (c) M = I (plain CG) on a 2x2 SPD system reaches the closed-form solution in <= 2
        iterations from x0 != 0."""
    d = np.array([[4.0, -1.0, 0.0], [-1.0, 4.0, -1.0], [0.0, -1.0, 4.0]])
    A = gen.from_dense(d)
    xs = np.array([1.0, 2.0, -3.0])
    b = d @ xs                                    # exact in fp64 (small integers)
    L, U = oracle.iluk(A, 0)
    r = oracle.pcg(A, L, U, b, 1e-12, 50, x0=xs)
    assert r["k"] == 0 and r["status"] == 0 and np.array_equal(r["x"], xs)
    # (b) dense 3x3 SPD, exact preconditioner
    d3 = np.array([[5.0, 2.0, 1.0], [2.0, 6.0, 3.0], [1.0, 3.0, 7.0]])
    A3 = gen.from_dense(d3)
    L3, U3 = oracle.iluk(A3, 0)
    b3 = np.array([1.0, -2.0, 0.5])
    # Cramer's rule: x_i = det(A with column i replaced by b) / det(A)
    det = np.linalg.det(d3)
    xc = np.array([np.linalg.det(np.column_stack([b3 if c == i else d3[:, c] for c in range(3)])) / det
                   for i in range(3)])
    x0 = np.array([10.0, -7.0, 3.0])
    r3 = oracle.pcg(A3, L3, U3, b3, 1e-13, 5, x0=x0)
    assert r3["k"] == 1
    assert np.allclose(r3["x"], xc, rtol=1e-13, atol=1e-14)
    # (c) 2x2, M = I: CG terminates in n = 2 steps (closed-form inverse)
    d2 = np.array([[3.0, 1.0], [1.0, 2.0]])
    A2 = gen.from_dense(d2)
    b2 = np.array([1.0, 1.0])
    x2 = np.array([2.0 * 1.0 - 1.0 * 1.0, -1.0 * 1.0 + 3.0 * 1.0]) / (3.0 * 2.0 - 1.0)   # (1/5, 2/5)
    r2 = oracle.pcg(A2, None, None, b2, 1e-14, 10, x0=np.array([-4.0, 9.0]))
    assert r2["k"] <= 2 and r2["status"] == 0
    assert np.allclose(r2["x"], x2, rtol=1e-14, atol=1e-15)


def test_pcg_breakdown_branch_pin():
    """O10's breakdown branch ((p, A p) <= 0, A12/§8(b) SPCG_ERR_BREAKDOWN): the
    symmetric matrix [[1,2],[2,1]] has a positive diagonal but eigenvalues 3 and -1.
    With b = (1,-1)/sqrt(2) (the -1 eigenvector) and M = I, p0 = b and
    (p0, A p0) = -1 in closed form; with ILU(0) (= exact LU here, u_22 = -3 < 0 is
    allowed) p0 = A^-1 b = -b and (p0, A p0) = -1 as well.  Both stop at k = 0
    with status BREAKDOWN and x = x0 = 0."""
    d = np.array([[1.0, 2.0], [2.0, 1.0]])
    A = gen.from_dense(d)
    b = np.array([1.0, -1.0]) / math.sqrt(2.0)
    assert float(b @ d @ b) == pytest.approx(-1.0, rel=1e-15)
    r = oracle.pcg(A, None, None, b, 1e-10, 10)
    assert r["status"] == oracle.BREAKDOWN and r["k"] == 0 and not np.any(r["x"])
    L, U = oracle.iluk(A, 0)
    assert U.val[U.row_ptr[1]] == -3.0                      # negative pivot: allowed (A12)
    r = oracle.pcg(A, L, U, b, 1e-10, 10)
    assert r["status"] == oracle.BREAKDOWN and r["k"] == 0 and not np.any(r["x"])


def test_norm_spec_power_method_pins():
    """SPECTRAL reading of ||M||_2 (A6 option; Alg. 2 line 4 writes the 2-norm):
    the oracle's 100-step power method against numpy's exact 2-norm.  With a spectral
    gap it converges to it; without one it stays a lower bound (||M v|| <= ||M|| ||v||)."""
    import numpy as np
    # diagonal with a gap, one dominant NEGATIVE eigenvalue (symmetric indefinite, like S)
    for d in (np.array([1.0, 2.0, 3.0, 9.0, 100.0]), np.array([-50.0, 1.0, 2.0, 3.0])):
        M = gen.from_dense(np.diag(d))
        assert abs(oracle.norm_spec(M) - np.abs(d).max()) <= 1e-12 * np.abs(d).max()
    # SPD with a dominant direction: I + 10 u u^T (exact norm 1 + 10 |u|^2)
    rng = np.random.default_rng(3)
    u = rng.standard_normal(8)
    D = np.eye(8) + 10.0 * np.outer(u, u)
    ex = np.linalg.norm(D, 2)
    assert abs(oracle.norm_spec(gen.from_dense(D)) - ex) <= 1e-10 * ex
    # Poisson (small gap): a lower bound, already close
    A = gen.make("poisson2d", 12, 12)
    ex = np.linalg.norm(A.to_scipy().toarray(), 2)
    est = oracle.norm_spec(A)
    assert est <= ex * (1 + 1e-14) and est >= 0.9 * ex
