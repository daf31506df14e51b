"""Shared checks of the parity tests (library vs oracle).  Test infrastructure only.

Tolerances: a row of SpTRSV is a sum of <= 115 fp64 products, so a
different rounding order moves it by <= len * 2^-53 * (sum of |terms|) ~ 1.3e-14 of
the row's absolute term sum; 1e-12 of that sum bounds it with margin.
"""
import numpy as np
import scipy.sparse as sp

import oracle


def csr_scipy(M):
    return sp.csr_matrix((M.val, M.col, M.row_ptr), shape=(M.n, M.n))


def check_setup_bit_exact(h, A, Ahat, L, U, flev, info=None):
    """Setup products the oracle fixes exactly: Ahat pattern and values,
    the Algorithm 2 trace, L_s / U patterns, levels of fill, factor values (same IKJ
    order, no FMA contraction), per-row levels and level sets of both factors."""
    assert np.array_equal(h.export("ahat_rowptr"), Ahat.row_ptr)
    assert np.array_equal(h.export("ahat_col"), Ahat.col)
    assert np.array_equal(h.export("ahat_val").view(np.uint64), Ahat.val.view(np.uint64))
    if info is not None and "chosen_pct" in info:
        assert h.info["chosen_pct"] == info["chosen_pct"]
    if info is not None and "trace" in info:
        tr = info["trace"]
        assert h.info["n_tried"] == len(tr)
        assert h.info["w_A"] == info["w_A"]
        for k, x in enumerate(tr):
            assert h.info["tried_pct"][k] == x["t"]
            assert h.info["indicator"][k] == x["ind"]
            assert h.info["tried_w"][k] == x["w"]
    assert np.array_equal(h.export("l_rowptr"), L.row_ptr)
    assert np.array_equal(h.export("l_col"), L.col)
    assert np.array_equal(h.export("u_rowptr"), U.row_ptr)
    assert np.array_equal(h.export("u_col"), U.col)
    assert np.array_equal(h.export("fill_level"), flev)
    assert np.array_equal(h.export("l_val").view(np.uint64), L.val.view(np.uint64))
    assert np.array_equal(h.export("u_val").view(np.uint64), U.val.view(np.uint64))
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
    assert h.info["w_Ahat"] == oracle.levels_lower(Ahat)[0]


def check_lower_all_rows(L, r, y, rtol=1e-12):
    """y = L^-1 r with unit diagonal: every row i satisfies y_i = r_i - sum_j l_ij y_j
    (the oracle's rows of L applied to the GPU's own y)."""
    Ls = csr_scipy(L)
    res = y + Ls @ y - r
    scale = np.abs(r) + abs(Ls) @ np.abs(y)
    bad = np.nonzero(np.abs(res) > rtol * scale + 1e-300)[0]
    assert bad.size == 0, (bad[:5], res[bad[:5]], scale[bad[:5]])


def check_upper_all_rows(U, y, z, rtol=1e-12):
    """z = U^-1 y: every row i satisfies sum_j u_ij z_j = y_i (diagonal included)."""
    Us = csr_scipy(U)
    res = Us @ z - y
    scale = np.abs(y) + abs(Us) @ np.abs(z)
    bad = np.nonzero(np.abs(res) > rtol * scale + 1e-300)[0]
    assert bad.size == 0, (bad[:5], res[bad[:5]], scale[bad[:5]])


def check_x_elementwise(x_gpu, x_or, rtol=1e-8):
    """|x_gpu - x_oracle|_i <= rtol * ||x_oracle||_inf for every i (forced-k runs)."""
    err = np.abs(x_gpu - x_or).max()
    assert err <= rtol * np.abs(x_or).max(), (err, np.abs(x_or).max())
