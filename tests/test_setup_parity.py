"""Host-side setup of the library vs the oracle: bit-exact sparsified matrix,
Algorithm 2 trace, ILU(K) patterns + levels of fill, factor values, and level
sets.  Runs without a GPU (device = -1: host analysis only)."""
import re
import os

import numpy as np
import pytest

import gen
import oracle
import paper_conf_sc_maacsh25_b200 as lib

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="session", autouse=True)
def _built():
    lib._build.build()
    lib.load()


def test_library_exports_every_declared_symbol():
    hdr = open(os.path.join(ROOT, "include", "spcg.h")).read()
    declared = set(re.findall(r"\b(spcg_[a-z_]+)\s*\(", hdr)) - {"spcg_handle_s"}
    L = lib.load()
    for name in declared:
        assert hasattr(L, name), name
    assert declared == set(lib.EXPORTED)
    assert L.spcg_abi_version() == 3


CASES = [
    ("poisson2d", (32, 32), "alg2", 0, 0.0),       # C1
    ("poisson2d", (32, 32), "none", 0, 0.0),
    ("poisson3d", (12, 10, 9), "alg2", 0, 0.0),
    ("fem_q1", (7, 6, 5, 3), "alg2", 2, 0.0),      # C3 family, ILU(2)
    ("fem_q1", (6, 6, 6, 5), "fixed", 1, 10.0),
    ("aniso_layered", (96, 80, 4), "alg2", 0, 0.0),  # C4 family (t = 5 branch)
    ("aniso_layered", (64, 64, 4), "fixed", 3, 5.0),
]


def _oracle_setup(A, mode, K, t):
    if mode == "none":
        Ah = A
        info = dict(chosen=0.0)
    elif mode == "fixed":
        Ah, S, m = oracle.sparsify(A, t)
        info = dict(chosen=t, m=m)
    else:
        Ah, idx, tr, wA = oracle.alg2(A)
        info = dict(chosen=[10.0, 5.0, 1.0][idx], trace=tr, wA=wA)
    P, flev = oracle.iluk_symbolic(Ah, K)
    st, L, U, bad = oracle.ilu_numeric(Ah, P)
    assert st == 0
    return Ah, P, flev, L, U, info


@pytest.mark.parametrize("fam,params,mode,K,t", CASES)
def test_setup_bit_exact(fam, params, mode, K, t):
    A = gen.make(fam, *params)
    h = lib.SPCG(A, mode=mode, K=K, fixed_pct=t, device=-1)
    Ah, P, flev, L, U, info = _oracle_setup(A, mode, K, t)
    # sparsified matrix: pattern AND values bit for bit
    assert np.array_equal(h.export("ahat_rowptr"), Ah.row_ptr)
    assert np.array_equal(h.export("ahat_col"), Ah.col)
    assert np.array_equal(h.export("ahat_val").view(np.uint64), Ah.val.view(np.uint64))
    assert h.info["chosen_pct"] == info["chosen"]
    if mode == "alg2":
        tr = info["trace"]
        assert h.info["n_tried"] == len(tr)
        assert h.info["w_A"] == info["wA"]
        for k, x in enumerate(tr):
            assert h.info["tried_pct"][k] == x["t"]
            assert h.info["indicator"][k] == x["ind"]              # same summation order: bitwise
            assert h.info["tried_w"][k] == x["w"]
    # ILU(K) patterns and levels of fill
    assert np.array_equal(h.export("l_rowptr"), L.row_ptr)
    assert np.array_equal(h.export("l_col"), L.col)
    assert np.array_equal(h.export("u_rowptr"), U.row_ptr)
    assert np.array_equal(h.export("u_col"), U.col)
    assert np.array_equal(h.export("fill_level"), flev)
    # numeric factors: same IKJ operation order, no FMA contraction -> bitwise
    assert np.array_equal(h.export("l_val").view(np.uint64), L.val.view(np.uint64))
    assert np.array_equal(h.export("u_val").view(np.uint64), U.val.view(np.uint64))
    # level sets of the factors (O8)
    wl, levl = oracle.levels_lower(L)
    wu, levu = oracle.levels_upper(U)
    assert h.info["levels_L"] == wl and h.info["levels_U"] == wu
    assert np.array_equal(h.export("level_l"), levl)
    assert np.array_equal(h.export("level_u"), levu)
    pl, rl = oracle.level_sets(levl, wl)
    assert np.array_equal(h.export("levelptr_l"), pl)
    assert np.array_equal(h.export("levelrows_l"), rl)
    pu, ru = oracle.level_sets(levu, wu)
    assert np.array_equal(h.export("levelptr_u"), pu)
    assert np.array_equal(h.export("levelrows_u"), ru)
    assert h.info["w_Ahat"] == oracle.levels_lower(Ah)[0]
    h.close()


def test_setup_random_patterns_bit_exact():
    rng = np.random.default_rng(11)
    for trial in range(30):
        n = int(rng.integers(2, 60))
        d = np.zeros((n, n))
        mask = np.tril(rng.random((n, n)) < rng.uniform(0.05, 0.4), -1)
        # many equal magnitudes so the tie-break (A4) matters
        d[mask] = -rng.choice([0.25, 0.5, 1.0], mask.sum())
        d = d + d.T
        d[np.diag_indices(n)] = np.abs(d).sum(1) + 1.0
        A = gen.from_dense(d)
        for K in (0, 1, 3):
            for mode, t in (("alg2", 0.0), ("fixed", 20.0)):
                h = lib.SPCG(A, mode=mode, K=K, fixed_pct=t, device=-1)
                Ah, P, flev, L, U, info = _oracle_setup(A, mode, K, t)
                assert np.array_equal(h.export("ahat_col"), Ah.col)
                assert np.array_equal(h.export("u_col"), U.col)
                assert np.array_equal(h.export("fill_level"), flev)
                assert np.array_equal(h.export("u_val").view(np.uint64), U.val.view(np.uint64))
                h.close()


def test_setup_rejects_bad_matrices():
    A = gen.make("poisson2d", 5, 4)
    bad = gen.CSR(A.n, A.row_ptr.copy(), A.col.copy(), A.val.copy())
    bad.val[1] = -0.5                                   # asymmetric
    with pytest.raises(lib.SpcgError) as e:
        lib.SPCG(bad, device=-1)
    assert e.value.status == lib.ERR_BAD_MATRIX
    bad = gen.CSR(A.n, A.row_ptr.copy(), A.col.copy(), A.val.copy())
    bad.val[A.row_ptr[2]:A.row_ptr[3]][A.col[A.row_ptr[2]:A.row_ptr[3]] == 2] = -4.0   # negative diagonal
    with pytest.raises(lib.SpcgError) as e:
        lib.SPCG(bad, device=-1)
    assert e.value.status == lib.ERR_BAD_MATRIX
    bad = gen.CSR(A.n, A.row_ptr.copy(), A.col.copy(), A.val.copy())
    bad.val[3] = np.inf
    with pytest.raises(lib.SpcgError):
        lib.SPCG(bad, device=-1)
    # zero pivot: singular 2x2
    S = gen.from_dense(np.array([[1.0, 2.0], [2.0, 4.0]]))
    with pytest.raises(lib.SpcgError) as e:
        lib.SPCG(S, mode="none", device=-1)
    assert e.value.status == lib.ERR_ZERO_PIVOT
    # empty system
    E = gen.CSR(0, np.zeros(1, np.int64), np.zeros(0, np.int32), np.zeros(0))
    with pytest.raises(lib.SpcgError) as e:
        lib.SPCG(E, device=-1)
    assert e.value.status == lib.ERR_INVALID_ARG


def test_host_only_handle_refuses_device_calls():
    A = gen.make("poisson2d", 8, 8)
    h = lib.SPCG(A, device=-1)
    with pytest.raises(lib.SpcgError) as e:
        h.solve_host(np.ones(A.n))
    assert e.value.status == lib.ERR_NO_DEVICE
    h.close()


def test_setup_info_bytes_formula():
    A = gen.make("poisson3d", 10, 10, 10)
    h = lib.SPCG(A, mode="none", device=-1)
    i = h.info
    n = A.n
    nUs = i["nnz_U"] - n
    expect = 12 * (A.nnz + i["nnz_L"] + nUs) + 8 * n + 12 * (n + 1) + 8 * n + 120 * n
    assert i["algo_bytes_per_iter"] == expect
    assert i["levels_L"] == 28 and i["levels_U"] == 28
    h.close()


def test_resident_executor_host_checks():
    """RESIDENT (one CTA, vectors in shared memory) is accepted up to
    RESIDENT_MAX_N rows, runs as one part, and is refused above (INVALID_ARG at
    setup, before any device work)."""
    A = gen.make("poisson2d", 64, 64)
    h = lib.SPCG(A, mode="none", sptrsv="resident", parts=9, device=-1)
    assert h.info["sptrsv_name"] == "resident" and h.info["parts"] == 1
    assert h.info["levels_L"] == 127                 # nx + ny - 1 (P2)
    h.close()
    with pytest.raises(lib.SpcgError):
        lib.SPCG(gen.make("poisson2d", 65, 64), sptrsv="resident", device=-1)


@pytest.mark.parametrize("fam,params", [("aniso_layered", (96, 80, 4)), ("poisson2d", (20, 20))])
def test_setup_spectral_reading_bit_exact(fam, params):
    """The SPECTRAL reading of the indicator norms (power method, 100 steps) gives the
    oracle's Algorithm 2 trace bit for bit (same operations, same order)."""
    A = gen.make(fam, *params)
    h = lib.SPCG(A, mode="alg2", K=0, device=-1, norm="spectral")
    Ah, idx, tr, wA = oracle.alg2(A, norm_reading=2)
    assert h.info["chosen_pct"] == [10.0, 5.0, 1.0][idx]
    assert h.info["n_tried"] == len(tr)
    for k, x in enumerate(tr):
        assert h.info["indicator"][k] == x["ind"]
        assert h.info["tried_w"][k] == x["w"]
    assert np.array_equal(h.export("ahat_col"), Ah.col)
    h.close()
