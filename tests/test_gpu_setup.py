"""NEXT-1: the setup of Fig. 2 on the GPU (ILU(0)) against the host
setup and the oracle.

Bit-exact: Ahat pattern and values, m_t, the chosen t, w_A, w_Ahat,
the tried w, L_s / U patterns and values (IKJ in the definition's order, explicit
round-to-nearest arithmetic, no contraction), fill levels, per-row levels and level
sets.  The Frobenius indicator sums run in a different (blocked) order on the GPU
(reading A6g): they agree with the oracle's row-major chain to within
the bound on reordering a sum of N non-negative terms, 2 (N - 1) 2^-53 relative per
sum, and no tested case sits that close to tau.  With the INF reading every indicator
term is an exact per-row sum or a max: bit-exact there too.
"""
import numpy as np
import pytest

import gen
import oracle
import paper_conf_sc_maacsh25_b200 as lib
from parity_util import check_setup_bit_exact

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

U53 = 2.0 ** -53

CASES = [("poisson2d", (32, 32), "alg2", 0.0),        # C1
         ("poisson2d", (32, 32), "none", 0.0),
         ("poisson2d", (37, 29), "fixed", 5.0),
         ("poisson3d", (13, 11, 9), "alg2", 0.0),
         ("aniso_layered", (150, 67, 4), "alg2", 0.0),
         ("aniso_layered", (256, 256, 4), "alg2", 0.0),
         ("fem_q1", (9, 8, 7, 3), "alg2", 0.0),      # 27-point, K = 0
         ("fem_q1", (9, 8, 7, 3), "fixed", 10.0)]

EXPORTS = ["ahat_rowptr", "ahat_col", "ahat_val", "l_rowptr", "l_col", "l_val", "u_rowptr", "u_col", "u_val",
           "fill_level", "level_l", "level_u", "levelptr_l", "levelrows_l", "levelptr_u", "levelrows_u"]
INFO_EXACT = ["chosen_pct", "m_t", "w_A", "w_Ahat", "n_tried", "tried_pct", "tried_w", "tried_reduction_pct",
              "nnz_A", "nnz_Ahat", "nnz_L", "nnz_U", "levels_L", "levels_U"]


def _ind_tol(A):
    # two orders of a sum of N non-negative terms differ by <= 2 (N - 1) u of the sum; the
    # indicator is a product / quotient of such sums and their square roots
    return 8.0 * A.nnz * U53


@pytest.mark.parametrize("fam,params,mode,pct", CASES)
def test_gpu_setup_matches_host_and_oracle(fam, params, mode, pct):
    A = gen.make(fam, *params)
    hg = lib.SPCG(A, mode=mode, fixed_pct=pct, K=0, setup="gpu")
    hh = lib.SPCG(A, mode=mode, fixed_pct=pct, K=0, setup="host", device=-1)
    assert hg.info["setup_device"] == 1 and hh.info["setup_device"] == 0
    for e in EXPORTS:
        a, b = hg.export(e), hh.export(e)
        assert a.dtype == b.dtype and np.array_equal(a.view(np.uint8), b.view(np.uint8)), e
    for k in INFO_EXACT:
        assert hg.info[k] == hh.info[k], k
    tol = _ind_tol(A)
    for r in range(hh.info["n_tried"]):
        ig, ih = hg.info["indicator"][r], hh.info["indicator"][r]
        assert abs(ig - ih) <= tol * abs(ih), (r, ig, ih)
        assert abs(ih - 1.0) > 1e3 * tol            # no case near tau: the branch is the same
    # and the oracle (independent code): the exact products bit for bit
    L, U, oinfo = oracle.setup(A, mode=mode, K=0, fixed_pct=pct)
    check_setup_bit_exact(hg, A, oinfo["Ahat"], L, U, oinfo["fill_level"], {"chosen_pct": oinfo["chosen_pct"]})
    for r, x in enumerate(oinfo.get("trace", [])):
        assert hg.info["tried_w"][r] == x["w"]
        assert abs(hg.info["indicator"][r] - x["ind"]) <= tol * abs(x["ind"])
    hg.close()
    hh.close()


def test_gpu_setup_inf_reading_bit_exact():
    """INF norms: every indicator term is an exact row sum or a max -> bit-exact."""
    A = gen.make("aniso_layered", 150, 67, 4)
    hg = lib.SPCG(A, mode="alg2", K=0, setup="gpu", norm="inf")
    hh = lib.SPCG(A, mode="alg2", K=0, setup="host", device=-1, norm="inf")
    for r in range(hh.info["n_tried"]):
        assert hg.info["indicator"][r] == hh.info["indicator"][r]
    assert hg.info["chosen_pct"] == hh.info["chosen_pct"]


def test_gpu_setup_solve_identical():
    """Same products -> same layout -> the solve is bitwise that of the host-set-up handle."""
    A = gen.make("aniso_layered", 256, 192, 4)
    b, _ = gen.rhs(A)
    bd = torch.from_numpy(b).cuda()
    xs = []
    for setup in ("gpu", "host"):
        h = lib.SPCG(A, mode="alg2", K=0, setup=setup)
        x, si = h.solve(bd, eps=1e-8, kmax=5000)
        assert si["status"] == 0
        xs.append((x.cpu().numpy(), si["iterations"]))
        h.close()
    assert xs[0][1] == xs[1][1]
    assert np.array_equal(xs[0][0].view(np.uint64), xs[1][0].view(np.uint64))


def test_gpu_setup_errors():
    # not symmetric (values)
    A = gen.make("poisson2d", 8, 8)
    val = A.val.copy()
    val[1] = -0.5                       # (0,1) != (1,0)
    B = gen.CSR(A.n, A.row_ptr, A.col, val)
    with pytest.raises(lib.SpcgError) as e:
        lib.SPCG(B, setup="gpu")
    assert e.value.status == lib.ERR_BAD_MATRIX
    # non-positive diagonal
    val = A.val.copy()
    val[0] = -4.0
    with pytest.raises(lib.SpcgError) as e:
        lib.SPCG(gen.CSR(A.n, A.row_ptr, A.col, val), setup="gpu")
    assert e.value.status == lib.ERR_BAD_MATRIX
    # a row pointer that runs past nnz then back (rp[n] == nnz still): no out-of-range read
    rp = A.row_ptr.copy()
    rp[3] = rp[-1] + 5
    for setup in ("gpu", "host"):
        with pytest.raises(lib.SpcgError) as e:
            lib.SPCG(gen.CSR(A.n, rp, A.col, A.val), setup=setup)
        assert e.value.status == lib.ERR_BAD_MATRIX
    # zero pivot: [[1, 1], [1, 1]] has u_11 = 1 - 1 = 0; the host reports the same row
    Z = gen.CSR(2, np.array([0, 2, 4], np.int64), np.array([0, 1, 0, 1], np.int32), np.ones(4))
    for setup in ("gpu", "host"):
        with pytest.raises(lib.SpcgError) as e:
            lib.SPCG(Z, mode="none", setup=setup)
        assert e.value.status == lib.ERR_ZERO_PIVOT


def test_gpu_setup_k_nonzero_runs_on_host():
    A = gen.make("fem_q1", 6, 5, 4, 3)
    h = lib.SPCG(A, mode="alg2", K=2, setup="gpu")
    assert h.info["setup_device"] == 0
    h.close()
