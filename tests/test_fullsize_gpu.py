"""Parity at BASELINE.json's full sizes (C1-C4), in the launch configuration
bench.py times (AUTO executor, default CTAs, Algorithm 2), through the C ABI.

For every config:
  * setup products bit for bit against the oracle (Ahat pattern + values, the
    Algorithm 2 trace, L_s / U patterns, levels of fill, factor values, per-row
    levels and level sets) — SURVEY §8(c.4);
  * Algorithm 1 to eps = 1e-8: |k_gpu - k_oracle| <= 1; then forced k = k_oracle:
    every x_i within 1e-8 ||x_oracle||_inf (one iteration more or less moves x by
    2e-7..1e-6, hence forced-k);
  * one forward and one backward triangular solve of the bench's kernel checked on
    EVERY row against the oracle's rows of L / U (the defining recurrence,
    P:L201-209), and the SpMV with the ORIGINAL A on every row.
The unsparsified PCG (mode none) is checked the same way on C1/C2 and by setup +
forced-k on C4.  Oracle results are computed once per config (module cache).
"""
import numpy as np
import pytest

import gen
import oracle
import paper_conf_sc_maacsh25_b200 as lib
from parity_util import (check_lower_all_rows, check_setup_bit_exact, check_upper_all_rows,
                         check_x_elementwise, csr_scipy)

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


def _dev(a):
    return torch.from_numpy(np.ascontiguousarray(a, np.float64)).cuda()


def _operators_all_rows(h, A, L, U, seed=11):
    rng = np.random.default_rng(seed)
    r = rng.standard_normal(A.n)
    y = torch.zeros(A.n, dtype=torch.float64, device="cuda")
    h.apply_lower(_dev(r), y)
    yh = y.cpu().numpy()
    check_lower_all_rows(L, r, yh)
    z = torch.zeros_like(y)
    h.apply_upper(y, z)
    check_upper_all_rows(U, yh, z.cpu().numpy())
    p = rng.standard_normal(A.n)
    w = torch.zeros_like(y)
    h.apply_spmv(_dev(p), w)
    As = csr_scipy(A)
    ref = As @ p
    scale = abs(As) @ np.abs(p)
    assert np.all(np.abs(w.cpu().numpy() - ref) <= 1e-13 * scale)


def _full_solve_parity(h, A, b, L, U, kmax=20000):
    ro = oracle.pcg(A, L, U, b, 1e-8, kmax)
    assert ro["status"] == 0
    x, si = h.solve(_dev(b), eps=1e-8, kmax=kmax)
    assert si["status"] == 0 and abs(si["iterations"] - ro["k"]) <= 1, (si, ro["k"])
    xf, sf = h.solve(_dev(b), eps=0.0, kmax=ro["k"])
    assert sf["iterations"] == ro["k"] and sf["status"] == 0
    check_x_elementwise(xf.cpu().numpy(), ro["x"])
    return ro["k"]


@pytest.mark.parametrize("name", ["C1", "C2", "C3", "C4"])
def test_full_size_alg2(name):
    A = gen.config_matrix(name)
    b, _ = gen.rhs(A)
    K = gen.CONFIGS[name]["K"]
    L, U, info = oracle.setup(A, mode="alg2", K=K)
    h = lib.SPCG(A, mode="alg2", K=K)
    check_setup_bit_exact(h, A, info["Ahat"], L, U, info["fill_level"], info)
    if K == 0:
        _gpu_setup_same_products(A, h, info)
    _operators_all_rows(h, A, L, U)
    _full_solve_parity(h, A, b, L, U)
    h.close()


def _gpu_setup_same_products(A, h, info):
    """NEXT-1 at full size: the GPU setup (gsetup.cu) yields the host setup's products bit
    for bit (the host handle h is itself checked against the oracle above); the Frobenius
    indicators agree with the oracle's up to summation order (reading A6g: 2 (N-1) 2^-53
    per sum, N = nnz(A) terms)."""
    hg = lib.SPCG(A, mode="alg2", K=0, setup="gpu")
    assert hg.info["setup_device"] == 1
    for e in ("ahat_rowptr", "ahat_col", "ahat_val", "l_rowptr", "l_col", "l_val", "u_rowptr", "u_col", "u_val",
              "level_l", "level_u", "levelrows_l", "levelrows_u"):
        assert np.array_equal(hg.export(e).view(np.uint8), h.export(e).view(np.uint8)), e
    for k in ("chosen_pct", "m_t", "w_A", "w_Ahat", "n_tried", "tried_w", "levels_L", "levels_U"):
        assert hg.info[k] == h.info[k], k
    tol = 8.0 * A.nnz * 2.0 ** -53
    for r, x in enumerate(info["trace"]):
        assert abs(hg.info["indicator"][r] - x["ind"]) <= tol * abs(x["ind"]), (r, hg.info["indicator"][r], x)
    hg.close()


@pytest.mark.parametrize("name", ["C1", "C2"])
def test_full_size_pcg_unsparsified(name):
    A = gen.config_matrix(name)
    b, _ = gen.rhs(A)
    L, U, info = oracle.setup(A, mode="none", K=0)
    h = lib.SPCG(A, mode="none", K=0)
    check_setup_bit_exact(h, A, A, L, U, info["fill_level"])
    _operators_all_rows(h, A, L, U)
    _full_solve_parity(h, A, b, L, U)
    h.close()


def test_full_size_c4_pcg_setup_and_forced_k():
    A = gen.config_matrix("C4")
    b, _ = gen.rhs(A)
    L, U, info = oracle.setup(A, mode="none", K=0)
    h = lib.SPCG(A, mode="none", K=0)
    check_setup_bit_exact(h, A, A, L, U, info["fill_level"])
    _operators_all_rows(h, A, L, U, seed=12)
    ro = oracle.pcg(A, L, U, b, 0.0, 5)
    xf, sf = h.solve(_dev(b), eps=0.0, kmax=5)
    assert sf["iterations"] == 5
    check_x_elementwise(xf.cpu().numpy(), ro["x"])
    h.close()


def test_c5_lane_scheduled_systems_match_oracle():
    """C5 lanes: members of the batch set up exactly as the bench does
    (4 lanes of 37 CTAs; 1 CTA for n <= 4096, 16 up to 16384), all in flight at once
    on their lane streams (spcg_solve_async), each compared with the oracle: k +- 1 to
    eps, then forced k = k_oracle element-wise."""
    from paper_conf_sc_maacsh25_b200 import batch
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    systems = [s for s in batch.batch_systems(64) if s.index in (6, 7, 13, 16, 20, 21, 23, 35)]
    hs = batch.setup_rank(systems, device=0, lanes=4, sms=sms)
    ref = {}
    for s, A, b, h, _ in hs:
        L, U, _ = oracle.setup(A, mode="alg2", K=s.K)
        ref[s.index] = (L, U, oracle.pcg(A, L, U, b, 1e-8, 20000))
    bufs = {}
    for s, A, b, h, _ in hs:
        with torch.cuda.stream(h.stream):
            bufs[s.index] = (_dev(b), torch.empty(A.n, dtype=torch.float64, device="cuda"))
    torch.cuda.synchronize()
    for eps_mode in ("eps", "forced"):
        for s, A, b, h, _ in hs:
            bd, xd = bufs[s.index]
            ro = ref[s.index][2]
            if eps_mode == "eps":
                h.solve_async(bd, xd, eps=1e-8, kmax=20000)
            else:
                h.solve_async(bd, xd, eps=0.0, kmax=ro["k"])
        for s, A, b, h, _ in hs:
            info = h.solve_wait()
            ro = ref[s.index][2]
            assert info["status"] == 0, (s.index, info)
            if eps_mode == "eps":
                assert abs(info["iterations"] - ro["k"]) <= 1, (s.index, info, ro["k"])
            else:
                assert info["iterations"] == ro["k"]
                check_x_elementwise(bufs[s.index][1].cpu().numpy(), ro["x"])
    for s, A, b, h, _ in hs:
        h.close()
