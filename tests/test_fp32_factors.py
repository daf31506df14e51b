"""NEXT-2: fp32 factors with fp64 vectors — the paper's
preconditioner precision inside the fp64 iteration.

The operator is M = fl32(L) fl32(U) (every stored factor value rounded to the nearest
fp32) applied in fp64; oracle.round_factors_f32 is that definition.  Pins (CPU):
the rounding error bound |fl32(v) - v| <= 2^-24 |v| and idempotence; on the
tridiagonal case, where ILU(0) is the exact LU (PCG converges in 1 iteration, P8),
the rounded factors no longer are (more than one iteration) yet CG still converges in
a handful; the library's exported factors equal the oracle's rounded ones bit for bit.
GPU: the solve with fp32 records against the oracle's PCG on the rounded factors
(k +- 1, forced-k element-wise).
"""
import numpy as np
import pytest

import gen
import oracle
import paper_conf_sc_maacsh25_b200 as lib
from parity_util import check_x_elementwise


def _tridiag(n=64):
    rp = np.zeros(n + 1, np.int64)
    col, val = [], []
    for i in range(n):
        for j, v in ((i - 1, -1.0), (i, 2.5 + 0.01 * (i % 7)), (i + 1, -1.0)):
            if 0 <= j < n:
                col.append(j)
                val.append(v)
        rp[i + 1] = len(col)
    return gen.CSR(n, rp, np.array(col, np.int32), np.array(val))


def test_rounding_bound_and_idempotence():
    A = gen.make("aniso_layered", 40, 33, 4)
    L, U, _ = oracle.setup(A, mode="alg2", K=0)
    Lr, Ur = oracle.round_factors_f32(L, U)
    for M, Mr in ((L, Lr), (U, Ur)):
        assert np.all(np.abs(Mr.val - M.val) <= 2.0 ** -24 * np.abs(M.val))
        assert np.array_equal(Mr.val.astype(np.float32).astype(np.float64), Mr.val)
        assert np.array_equal(Mr.col, M.col) and np.array_equal(Mr.row_ptr, M.row_ptr)
    assert np.any(Lr.val != L.val)           # the layered field's values are not fp32 numbers


def test_rounded_exact_lu_is_no_longer_exact():
    A = _tridiag()
    b, _ = gen.rhs(A)
    L, U, _ = oracle.setup(A, mode="none", K=0)
    r64 = oracle.pcg(A, L, U, b, 1e-12, 50)
    assert r64["k"] == 1                      # P8: ILU(0) of a tridiagonal matrix is exact
    Lr, Ur = oracle.round_factors_f32(L, U)
    r32 = oracle.pcg(A, Lr, Ur, b, 1e-12, 50)
    assert 1 < r32["k"] <= 6 and r32["status"] == 0
    assert np.linalg.norm(r32["x"] - r64["x"]) <= 1e-10 * np.linalg.norm(r64["x"])


@pytest.mark.parametrize("fam,params,K", [("aniso_layered", (150, 67, 4), 0), ("poisson3d", (13, 11, 9), 0),
                                          ("fem_q1", (6, 5, 4, 3), 2)])
def test_library_rounds_like_the_oracle(fam, params, K):
    A = gen.make(fam, *params)
    h = lib.SPCG(A, mode="alg2", K=K, device=-1, factors="f32")
    L, U, _ = oracle.setup(A, mode="alg2", K=K)
    Lr, Ur = oracle.round_factors_f32(L, U)
    assert np.array_equal(h.export("l_val").view(np.uint64), Lr.val.view(np.uint64))
    assert np.array_equal(h.export("u_val").view(np.uint64), Ur.val.view(np.uint64))
    assert h.info["factor_precision"] == 1
    h.close()


@pytest.mark.gpu
@pytest.mark.parametrize("fam,params,K,ex", [("aniso_layered", (150, 67, 4), 0, "wchain"),
                                             ("aniso_layered", (512, 384, 4), 0, "auto"),
                                             ("poisson2d", (37, 29), 0, "wchain"),
                                             ("poisson3d", (13, 11, 9), 0, "chunked"),
                                             ("fem_q1", (9, 8, 7, 3), 2, "auto")])
def test_gpu_fp32_factors_match_oracle(fam, params, K, ex):
    torch = pytest.importorskip("torch")
    A = gen.make(fam, *params)
    b, _ = gen.rhs(A)
    try:
        h = lib.SPCG(A, mode="alg2", K=K, sptrsv=ex, factors="f32")
    except lib.SpcgError as e:
        assert e.status == lib.ERR_INVALID_ARG
        pytest.skip("executor does not apply")
    if h.info["sptrsv_name"] == "wchain":
        assert h.info["record_value_bytes"] == 4
    L, U, _ = oracle.setup(A, mode="alg2", K=K)
    Lr, Ur = oracle.round_factors_f32(L, U)
    ro = oracle.pcg(A, Lr, Ur, b, 1e-8, 20000)
    bd = torch.from_numpy(b).cuda()
    x, si = h.solve(bd, eps=1e-8, kmax=20000)
    assert si["status"] == 0 and abs(si["iterations"] - ro["k"]) <= 1, (si, ro["k"])
    xf, sf = h.solve(bd, eps=0.0, kmax=ro["k"])
    check_x_elementwise(xf.cpu().numpy(), ro["x"])
    h.close()
