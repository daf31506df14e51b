"""CUDA path (through the C ABI) vs the oracle, element by element, on seeded
inputs.  Tolerances: SpMV / SpTRSV <= 1e-12 relative to the
row's absolute sum of terms; PCG |k_gpu - k_oracle| <= 1 on convergence runs and
||x_gpu - x_oracle|| <= 1e-8 ||x_oracle|| in forced-k runs (eps = 0, kmax = k)."""
import numpy as np
import pytest

import gen
import oracle
import paper_conf_sc_maacsh25_b200 as lib
from parity_util import check_x_elementwise

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

EXECUTORS = ["level", "syncfree", "chunked", "resident", "wchain"]


def _fits(ex, A, K=0, parts=0):
    """The resident executor takes n <= RESIDENT_MAX_N (one CTA's shared memory); the
    warp-chain executor rows of <= 16 dependencies (not 27-point ILU(2))."""
    if ex == "resident" and A.n > lib.RESIDENT_MAX_N:
        pytest.skip("resident executor: n > RESIDENT_MAX_N")
    if ex == "wchain":
        try:
            lib.SPCG(A, K=K, sptrsv="wchain", parts=parts, device=-1).close()
        except lib.SpcgError as e:
            assert e.status == lib.ERR_INVALID_ARG
            pytest.skip("warp-chain executor does not apply")


def _dev(a):
    return torch.from_numpy(np.ascontiguousarray(a, np.float64)).cuda()


def _csr_abs(M):
    return gen.CSR(M.n, M.row_ptr, M.col, np.abs(M.val))


# sizes: several 32-row slices, a ragged tail, more rows than one CTA's block
SMALL = [("poisson2d", (37, 29), 0), ("poisson3d", (13, 11, 9), 0), ("fem_q1", (9, 8, 7, 3), 2),
         ("aniso_layered", (150, 67, 4), 0)]


@pytest.mark.parametrize("fam,params,K", SMALL)
@pytest.mark.parametrize("ex", EXECUTORS)
@pytest.mark.parametrize("parts", [1, 7, 0])
def test_operators_match_oracle(fam, params, K, ex, parts):
    A = gen.make(fam, *params)
    _fits(ex, A, K, parts)
    h = lib.SPCG(A, mode="alg2", K=K, sptrsv=ex, parts=parts)
    L, U, _ = oracle.setup(A, mode="alg2", K=K)
    rng = np.random.default_rng(5)
    p = rng.standard_normal(A.n)
    # SpMV w = A p and (p, w)
    w = torch.zeros(A.n, dtype=torch.float64, device="cuda")
    pw = h.apply_spmv(_dev(p), w)
    wr = oracle.spmv(A, p)
    scale = oracle.spmv(_csr_abs(A), np.abs(p)) + 1e-300
    assert np.all(np.abs(w.cpu().numpy() - wr) <= 1e-13 * scale)
    assert pw == pytest.approx(float(np.dot(p, wr)), rel=1e-12)
    # forward solve y = L^-1 r
    r = rng.standard_normal(A.n)
    y = torch.zeros_like(w)
    h.apply_lower(_dev(r), y)
    yr = oracle.sptrsv_lower(L, r)
    assert np.allclose(y.cpu().numpy(), yr, rtol=1e-12, atol=1e-12 * np.abs(yr).max())
    # backward solve z = U^-1 y with (r, z)
    z = torch.zeros_like(w)
    rz = h.apply_upper(_dev(yr), z, _dev(r))
    zr = oracle.sptrsv_upper(U, yr)
    assert np.allclose(z.cpu().numpy(), zr, rtol=1e-12, atol=1e-12 * np.abs(zr).max())
    assert rz == pytest.approx(float(np.dot(r, zr)), rel=1e-11)
    # whole preconditioner
    z2 = torch.zeros_like(w)
    h.apply_precond(_dev(r), z2)
    assert np.allclose(z2.cpu().numpy(), zr, rtol=1e-12, atol=1e-12 * np.abs(zr).max())
    h.close()


@pytest.mark.parametrize("fam,params,K", SMALL + [("poisson2d", (32, 32), 0)])
@pytest.mark.parametrize("mode", ["alg2", "none"])
@pytest.mark.parametrize("ex", EXECUTORS)
def test_pcg_matches_oracle(fam, params, K, mode, ex):
    A = gen.make(fam, *params)
    _fits(ex, A, K)
    b, xt = gen.rhs(A)
    h = lib.SPCG(A, mode=mode, K=K, sptrsv=ex)
    L, U, _ = oracle.setup(A, mode=mode, K=K)
    ro = oracle.pcg(A, L, U, b, 1e-8, 5000)
    x, info = h.solve(_dev(b), eps=1e-8, kmax=5000)
    assert info["status"] == 0 and info["converged"]
    assert abs(info["iterations"] - ro["k"]) <= 1
    # true residual of the GPU solution
    xg = x.cpu().numpy()
    assert np.linalg.norm(b - oracle.spmv(A, xg)) <= 1.01e-8 * 1.5
    # forced-k: same number of iterations, solution within 1e-8 (expect ~1e-13)
    k = ro["k"]
    xf, inf2 = h.solve(_dev(b), eps=0.0, kmax=k)
    assert inf2["iterations"] == k and inf2["status"] == 0
    check_x_elementwise(xf.cpu().numpy(), ro["x"])
    # residual history agrees with the oracle's
    rh = h.rhist()
    assert len(rh) == k + 1
    assert np.allclose(rh, ro["rhist"], rtol=1e-6, atol=1e-14)
    h.close()


def test_identity_preconditioner_is_cg():
    A = gen.make("poisson2d", 40, 23)
    b, _ = gen.rhs(A)
    h = lib.SPCG(A, mode="none", K=-1)
    ro = oracle.pcg(A, None, None, b, 1e-8, 5000)
    x, info = h.solve(_dev(b), eps=1e-8, kmax=5000)
    assert abs(info["iterations"] - ro["k"]) <= 1
    xf, _ = h.solve(_dev(b), eps=0.0, kmax=ro["k"])
    check_x_elementwise(xf.cpu().numpy(), ro["x"])


@pytest.mark.parametrize("ex", EXECUTORS)
def test_deterministic_bitwise(ex):
    A = gen.make("aniso_layered", 300, 211, 4) if ex != "resident" else gen.make("aniso_layered", 64, 60, 4)
    b, _ = gen.rhs(A)
    h = lib.SPCG(A, sptrsv=ex)
    x1, i1 = h.solve(_dev(b), eps=1e-8, kmax=5000)
    x2, i2 = h.solve(_dev(b), eps=1e-8, kmax=5000)
    assert i1["iterations"] == i2["iterations"]
    assert torch.equal(x1, x2)


def test_host_pointer_path_matches_device_path():
    A = gen.make("poisson3d", 20, 20, 20)
    b, _ = gen.rhs(A)
    h = lib.SPCG(A)
    xd, i1 = h.solve(_dev(b), eps=1e-8, kmax=5000)
    xh, i2 = h.solve_host(b, eps=1e-8, kmax=5000)
    assert i1["iterations"] == i2["iterations"]
    assert np.array_equal(xd.cpu().numpy(), xh)


def test_initial_guess_and_kmax():
    A = gen.make("poisson2d", 33, 31)
    b, xt = gen.rhs(A)
    h = lib.SPCG(A)
    L, U, _ = oracle.setup(A, mode="alg2", K=0)
    x0 = 0.5 * xt
    ro = oracle.pcg(A, L, U, b, 0.0, 6, x0=x0)
    xg = _dev(x0)
    h.solve(_dev(b), xg, eps=0.0, kmax=6, use_x0=True)
    check_x_elementwise(xg.cpu().numpy(), ro["x"], rtol=1e-10)
    x, info = h.solve(_dev(b), eps=1e-30, kmax=4)
    assert info["iterations"] == 4 and info["status"] == lib.NOT_CONVERGED


def test_tridiagonal_one_iteration():
    n = 1000
    d = np.zeros((n, n))
    A = gen.from_dense(np.diag(np.full(n, 2.5)) + np.diag(np.full(n - 1, -1.0), 1) + np.diag(np.full(n - 1, -1.0), -1))
    b, _ = gen.rhs(A)
    for ex in EXECUTORS:
        h = lib.SPCG(A, mode="none", sptrsv=ex, parts=4)
        x, info = h.solve(_dev(b), eps=1e-12, kmax=50)
        assert info["iterations"] == 1, ex       # ILU(0) of a tridiagonal matrix is exact (P8)
        h.close()


def test_calibrate_handoffs_are_ordered():
    """Chain-floor calibration: every handoff measured, positive and
    in the order the hardware fixes (intra-CTA < cross-CTA flag < grid barrier)."""
    c = lib.calibrate(0)
    assert c["sms"] >= 100
    for k in ("grid_sync_ns", "graph_kernel_ns", "flag_same_die_ns", "flag_cross_die_ns", "syncthreads_ns",
              "cluster_sync_ns"):
        assert 0.0 < c[k] < 1e5, (k, c)
    assert c["syncthreads_ns"] < c["flag_same_die_ns"] <= c["flag_cross_die_ns"]
    assert c["flag_same_die_ns"] < c["grid_sync_ns"]


def test_ll_flags_never_tear():
    """Robustness of the 16-byte LL ready flags {lo32, epoch, hi32, epoch} (DESIGN.md
    §5.3): under concurrent rewrites from half the SMs and random polling from the
    other half, no load ever sees both epochs current with a value from another epoch.
    Small slot counts put producer and consumers on the same lines constantly."""
    for nslots, rounds in ((64, 20000), (4096, 2000), (1 << 20, 20)):
        r = lib.ll_stress(0, nslots, rounds)
        assert r["torn"] == 0, (nslots, rounds, r)
        assert r["ok"] > 0, r


def test_async_concurrent_solves_match_sync():
    """spcg_solve_async / spcg_solve_wait: independent systems in flight on separate
    streams (C5 lanes) give bitwise the results of spcg_solve."""
    mats = [gen.make("poisson2d", 40, 33), gen.make("aniso_layered", 96, 64, 4), gen.make("poisson3d", 12, 11, 10)]
    streams = [torch.cuda.Stream() for _ in mats]
    hs, bs, xs = [], [], []
    for A, st in zip(mats, streams):
        b, _ = gen.rhs(A)
        hs.append(lib.SPCG(A, mode="alg2", K=0, parts=4, stream=st))
        bs.append(_dev(b))
        xs.append(torch.empty_like(bs[-1]))
    for h, b, x in zip(hs, bs, xs):
        h.solve_async(b, x, eps=1e-8, kmax=5000)
    infos = [h.solve_wait() for h in hs]
    for h, b, x, inf in zip(hs, bs, xs, infos):
        xr, ir = h.solve(b, eps=1e-8, kmax=5000)
        assert inf["status"] == 0 and inf["iterations"] == ir["iterations"]
        assert torch.equal(x, xr)
    with pytest.raises(lib.SpcgError):
        hs[0].solve_wait()                       # nothing in flight


@pytest.mark.parametrize("ex", EXECUTORS)
def test_degenerate_cases(ex):
    """Edge cases of Algorithm 1 on every executor: b = 0 stops at k = 0
    with x = 0 (test before the first SpMV, A13); kmax = 0 returns x0 = 0 with
    NOT_CONVERGED (A14); n = 1 and a diagonal matrix (no off-diagonals: empty L,
    one wavefront) converge in one iteration with the exact solution."""
    A = gen.make("poisson2d", 37, 29)
    h = lib.SPCG(A, sptrsv=ex, parts=5)
    x, info = h.solve(torch.zeros(A.n, dtype=torch.float64, device="cuda"), eps=1e-8, kmax=100)
    assert info["iterations"] == 0 and info["status"] == 0 and not torch.any(x != 0)
    b, _ = gen.rhs(A)
    x, info = h.solve(_dev(b), eps=1e-8, kmax=0)
    assert info["iterations"] == 0 and info["status"] == lib.NOT_CONVERGED and not torch.any(x != 0)
    h.close()
    for d in (np.array([[3.0]]), np.diag(np.linspace(1.0, 7.0, 5000 if ex != "resident" else 4096))):
        Ad = gen.from_dense(d) if d.shape[0] == 1 else gen.CSR(d.shape[0], np.arange(d.shape[0] + 1, dtype=np.int64),
                                                               np.arange(d.shape[0], dtype=np.int32), np.diag(d).copy())
        bd = np.linspace(-1.0, 1.0, Ad.n) if Ad.n > 1 else np.array([1.5])
        hd = lib.SPCG(Ad, mode="alg2", sptrsv=ex)
        assert hd.info["levels_L"] == 1
        xd, info = hd.solve(_dev(bd), eps=1e-12, kmax=10)
        assert info["iterations"] == 1 and info["status"] == 0
        assert np.allclose(xd.cpu().numpy(), bd / np.diag(d), rtol=1e-15, atol=0)
        hd.close()


def test_resident_limits_and_initial_guess():
    """RESIDENT executor: the largest system it takes (n = RESIDENT_MAX_N, 64x64
    Poisson) matches the oracle in forced-k mode from a user x0 (x copied in and out
    of shared memory); one row more is rejected with INVALID_ARG at setup."""
    A = gen.make("poisson2d", 64, 64)
    assert A.n == lib.RESIDENT_MAX_N
    b, xt = gen.rhs(A)
    h = lib.SPCG(A, sptrsv="resident")
    assert h.info["sptrsv_name"] == "resident" and h.info["parts"] == 1
    L, U, _ = oracle.setup(A, mode="alg2", K=0)
    x0 = 0.25 * xt
    ro = oracle.pcg(A, L, U, b, 0.0, 9, x0=x0)
    xg = _dev(x0)
    h.solve(_dev(b), xg, eps=0.0, kmax=9, use_x0=True)
    assert np.linalg.norm(xg.cpu().numpy() - ro["x"]) <= 1e-10 * np.linalg.norm(ro["x"])
    h.close()
    with pytest.raises(lib.SpcgError):
        lib.SPCG(gen.make("poisson2d", 65, 64), sptrsv="resident")


@pytest.mark.parametrize("ex", EXECUTORS)
def test_breakdown_status(ex):
    """SPCG_ERR_BREAKDOWN (§8(b)): the indefinite [[1,2],[2,1]] with b on its -1
    eigenvector gives (p0, A p0) = -1 at k = 0 (pinned in test_oracle_numeric); the
    device loop must stop with status BREAKDOWN on every executor, as the oracle does."""
    A = gen.from_dense(np.array([[1.0, 2.0], [2.0, 1.0]]))
    b = np.array([1.0, -1.0]) / np.sqrt(2.0)
    L, U, _ = oracle.setup(A, mode="none", K=0)
    assert oracle.pcg(A, L, U, b, 1e-10, 10)["status"] == oracle.BREAKDOWN
    h = lib.SPCG(A, mode="none", K=0, sptrsv=ex)
    with pytest.raises(lib.SpcgError) as e:
        h.solve(_dev(b), eps=1e-10, kmax=10)
    assert e.value.status == lib.ERR_BREAKDOWN
    h.close()
