"""Python face of the plain fp64 CPU ORACLE (oracle/spcg_oracle.c).

TEST INFRASTRUCTURE ONLY: imported by tests/, __graft_entry__.smoke() and the
cpu_baseline / ``--impl reference`` legs of bench.py — never by the product
package ``paper_conf_sc_maacsh25_b200``.  The oracle shares no code with the
CUDA library; its only common dependency is the seeded input module ``gen``.

Each function cites the PAPER.md passage it follows (see the C source header);
readings of silent passages follow SURVEY.md §8(c) and DESIGN.md §2.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import time

import numpy as np

from gen import CSR

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "spcg_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

OK, NOT_CONVERGED, BAD_MATRIX, ZERO_PIVOT, BREAKDOWN = 0, 1, -2, -3, -4


class _Csr(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("nnz", ctypes.c_int64),
                ("rowptr", ctypes.POINTER(ctypes.c_int64)),
                ("col", ctypes.POINTER(ctypes.c_int32)),
                ("val", ctypes.POINTER(ctypes.c_double))]


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math", "-fPIC",
                               "-shared", "-o", _LIB + ".tmp", _SRC, "-lm"])
        os.replace(_LIB + ".tmp", _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        P = ctypes.c_void_p
        CP = ctypes.POINTER(_Csr)
        lib.or_validate.argtypes = [CP]
        lib.or_levels_lower.argtypes = [CP, P]
        lib.or_levels_lower.restype = ctypes.c_int64
        lib.or_levels_upper.argtypes = [CP, P]
        lib.or_levels_upper.restype = ctypes.c_int64
        lib.or_level_sets.argtypes = [ctypes.c_int64, P, ctypes.c_int64, P, P]
        lib.or_drop_count.argtypes = [CP, ctypes.c_double]
        lib.or_drop_count.restype = ctypes.c_int64
        lib.or_sparsify.argtypes = [CP, ctypes.c_double, CP, CP]
        lib.or_sparsify.restype = ctypes.c_int64
        lib.or_indicator.argtypes = [CP, CP, ctypes.c_int, P]
        lib.or_indicator.restype = ctypes.c_double
        lib.or_norm_fro.argtypes = [CP]
        lib.or_norm_fro.restype = ctypes.c_double
        lib.or_norm_inf.argtypes = [CP]
        lib.or_norm_inf.restype = ctypes.c_double
        lib.or_norm_spec.argtypes = [CP]
        lib.or_norm_spec.restype = ctypes.c_double
        lib.or_alg2.argtypes = [CP, P, ctypes.c_int, ctypes.c_double, ctypes.c_double, ctypes.c_int,
                                ctypes.c_int, CP, P, P, P]
        lib.or_iluk_symbolic.argtypes = [CP, ctypes.c_int, CP, ctypes.POINTER(ctypes.POINTER(ctypes.c_int32))]
        lib.or_ilu_numeric.argtypes = [CP, CP, CP, CP, P]
        lib.or_spmv.argtypes = [CP, P, P]
        lib.or_sptrsv_lower.argtypes = [CP, P, P]
        lib.or_sptrsv_upper.argtypes = [CP, P, P]
        lib.or_pcg.argtypes = [CP, CP, CP, P, P, ctypes.c_double, ctypes.c_int64, P, P, P, P]
        lib.or_csr_free.argtypes = [CP]
        lib.or_free.argtypes = [P]
        _lib = lib
    return _lib


def _p(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def _in(M: CSR) -> _Csr:
    # keep references alive on the struct
    rp = np.ascontiguousarray(M.row_ptr, np.int64)
    col = np.ascontiguousarray(M.col, np.int32)
    val = np.ascontiguousarray(M.val, np.float64)
    s = _Csr(M.n, int(rp[-1]) if len(rp) else 0,
             rp.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)),
             col.ctypes.data_as(ctypes.POINTER(ctypes.c_int32)),
             val.ctypes.data_as(ctypes.POINTER(ctypes.c_double)))
    s._keep = (rp, col, val)
    return s


def _out(s: _Csr, name: str = "") -> CSR:
    n, nnz = s.n, s.nnz
    rp = np.ctypeslib.as_array(s.rowptr, shape=(n + 1,)).copy()
    col = np.ctypeslib.as_array(s.col, shape=(max(nnz, 1),))[:nnz].copy()
    val = np.ctypeslib.as_array(s.val, shape=(max(nnz, 1),))[:nnz].copy()
    _load().or_csr_free(ctypes.byref(s))
    return CSR(n, rp, col, val, name)


# ---------------------------------------------------------------- O1
def validate(A: CSR) -> int:
    return _load().or_validate(ctypes.byref(_in(A)))


# ---------------------------------------------------------------- O2
def levels_lower(M: CSR):
    lev = np.zeros(max(M.n, 1), np.int32)
    w = _load().or_levels_lower(ctypes.byref(_in(M)), _p(lev))
    return int(w), lev[: M.n]


def levels_upper(M: CSR):
    lev = np.zeros(max(M.n, 1), np.int32)
    w = _load().or_levels_upper(ctypes.byref(_in(M)), _p(lev))
    return int(w), lev[: M.n]


def level_sets(lev: np.ndarray, w: int):
    n = len(lev)
    ptr = np.zeros(w + 1, np.int64)
    rows = np.zeros(max(n, 1), np.int32)
    _load().or_level_sets(n, _p(np.ascontiguousarray(lev, np.int32)), w, _p(ptr), _p(rows))
    return ptr, rows[:n]


# ---------------------------------------------------------------- O3 / O4
def drop_count(A: CSR, t_pct: float) -> int:
    return int(_load().or_drop_count(ctypes.byref(_in(A)), t_pct))


def sparsify(A: CSR, t_pct: float):
    """Returns (Ahat, S, m_t)."""
    Ah, S = _Csr(), _Csr()
    m = _load().or_sparsify(ctypes.byref(_in(A)), t_pct, ctypes.byref(Ah), ctypes.byref(S))
    return _out(Ah, "Ahat"), _out(S, "S"), int(m)


def indicator(Ahat: CSR, S: CSR, norm_reading: int = 0):
    out = np.zeros(3)
    v = _load().or_indicator(ctypes.byref(_in(Ahat)), ctypes.byref(_in(S)), norm_reading, _p(out))
    return float(v), dict(kappa=out[0], inv_norm=out[1], s_norm=out[2])


def norm_spec(M: CSR) -> float:
    """SPECTRAL reading of ||M||_2: the power method, 100 steps from the all-ones vector."""
    return float(_load().or_norm_spec(ctypes.byref(_in(M))))


def alg2(A: CSR, ratios=(10.0, 5.0, 1.0), tau=1.0, omega=10.0, norm_reading=0, denom_mode=0):
    """Algorithm 2.  Returns (Ahat, chosen_index, trace(list of dicts), w_A)."""
    nr = len(ratios)
    r = np.array(ratios, np.float64)
    trace = np.zeros(5 * nr)
    wA = np.zeros(1, np.int64)
    ntried = np.zeros(1, np.int32)
    Ah = _Csr()
    idx = _load().or_alg2(ctypes.byref(_in(A)), _p(r), nr, tau, omega, norm_reading, denom_mode,
                          ctypes.byref(Ah), _p(trace), _p(wA), _p(ntried))
    tr = [dict(t=trace[5 * k], m=int(trace[5 * k + 1]), ind=trace[5 * k + 2], w=int(trace[5 * k + 3]),
               red=trace[5 * k + 4]) for k in range(int(ntried[0]))]
    return _out(Ah, "Ahat"), int(idx), tr, int(wA[0])


# ---------------------------------------------------------------- O6 / O7
def iluk_symbolic(Ahat: CSR, K: int):
    """Returns (pattern CSR (val 0), level-of-fill per entry)."""
    P = _Csr()
    levp = ctypes.POINTER(ctypes.c_int32)()
    _load().or_iluk_symbolic(ctypes.byref(_in(Ahat)), K, ctypes.byref(P), ctypes.byref(levp))
    nnz = P.nnz
    lev = np.ctypeslib.as_array(levp, shape=(max(nnz, 1),))[:nnz].copy()
    _load().or_free(ctypes.cast(levp, ctypes.c_void_p))
    return _out(P, "pattern"), lev


def ilu_numeric(Ahat: CSR, P: CSR):
    """Returns (status, L_s, U, bad_row)."""
    L, U = _Csr(), _Csr()
    bad = np.zeros(1, np.int64)
    st = _load().or_ilu_numeric(ctypes.byref(_in(Ahat)), ctypes.byref(_in(P)), ctypes.byref(L),
                                ctypes.byref(U), _p(bad))
    if st != 0:
        return st, None, None, int(bad[0])
    return st, _out(L, "L_s"), _out(U, "U"), -1


def iluk(Ahat: CSR, K: int, with_levels: bool = False):
    P, lev = iluk_symbolic(Ahat, K)
    st, L, U, bad = ilu_numeric(Ahat, P)
    if st != 0:
        raise ZeroDivisionError(f"zero pivot at row {bad}")
    return (L, U, lev) if with_levels else (L, U)


# ---------------------------------------------------------------- O9 / O10
def spmv(A: CSR, x: np.ndarray) -> np.ndarray:
    y = np.zeros(A.n)
    _load().or_spmv(ctypes.byref(_in(A)), _p(np.ascontiguousarray(x, np.float64)), _p(y))
    return y


def sptrsv_lower(L: CSR, r: np.ndarray) -> np.ndarray:
    y = np.zeros(L.n)
    _load().or_sptrsv_lower(ctypes.byref(_in(L)), _p(np.ascontiguousarray(r, np.float64)), _p(y))
    return y


def sptrsv_upper(U: CSR, y: np.ndarray) -> np.ndarray:
    z = np.zeros(U.n)
    _load().or_sptrsv_upper(ctypes.byref(_in(U)), _p(np.ascontiguousarray(y, np.float64)), _p(z))
    return z


def pcg(A: CSR, L: CSR | None, U: CSR | None, b: np.ndarray, eps: float, kmax: int, x0=None):
    """Algorithm 1.  L = None means M = I.  Returns dict(x, k, rnorm, status, rhist, seconds)."""
    x = np.zeros(A.n)
    k = np.zeros(1, np.int64)
    rn = np.zeros(1)
    rh = np.zeros(kmax + 2)
    Ls = ctypes.byref(_in(L)) if L is not None else None
    Us = ctypes.byref(_in(U)) if U is not None else None
    t0 = time.perf_counter()
    st = _load().or_pcg(ctypes.byref(_in(A)), Ls, Us, _p(np.ascontiguousarray(b, np.float64)),
                        _p(None if x0 is None else np.ascontiguousarray(x0, np.float64)),
                        eps, kmax, _p(x), _p(k), _p(rn), _p(rh))
    dt = time.perf_counter() - t0
    kk = int(k[0])
    return dict(x=x, k=kk, rnorm=float(rn[0]), status=int(st), rhist=rh[: kk + 1], seconds=dt)


def setup(A: CSR, mode: str = "alg2", K: int = 0, fixed_pct: float = 0.0, **alg2_kw):
    """Whole oracle setup (Fig. 2): Ahat by mode, then ILU(K) of Ahat.
    mode: 'none' (PCG, Ahat = A), 'fixed' (A - S_t), 'alg2' (Algorithm 2)."""
    info = {}
    if mode == "none":
        Ahat = A
        info["chosen_pct"] = 0.0
    elif mode == "fixed":
        Ahat, S, m = sparsify(A, fixed_pct)
        info["chosen_pct"] = fixed_pct
        info["m_t"] = m
    else:
        Ahat, idx, tr, wA = alg2(A, **alg2_kw)
        ratios = alg2_kw.get("ratios", (10.0, 5.0, 1.0))
        info.update(chosen_pct=ratios[idx], trace=tr, w_A=wA)
    L, U, flev = iluk(Ahat, K, with_levels=True)
    info["Ahat"] = Ahat
    info["fill_level"] = flev          # level of fill per entry of pattern(L + U), row-major (O6)
    return L, U, info


def round_factors_f32(L: CSR, U: CSR):
    """NEXT-2: the paper's fp32 preconditioner applied in fp64 — every stored
    factor value rounded to the nearest fp32 (IEEE round to nearest even, as a C
    (float) cast), the operator M = fl32(L) fl32(U).  Returns new CSRs."""
    def r(M):
        return CSR(M.n, M.row_ptr, M.col, M.val.astype(np.float32).astype(np.float64), M.name)
    return r(L), r(U)


# ---------------------------------------------------------------- multicore baseline
_OMP_SRC = os.path.join(_HERE, "spcg_oracle_omp.c")
_OMP_LIB = os.path.join(_HERE, "liboracle_omp.so")
_omp = None


def build_omp(force: bool = False) -> str:
    if force or not os.path.exists(_OMP_LIB) or os.path.getmtime(_OMP_LIB) < os.path.getmtime(_OMP_SRC):
        subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math", "-fopenmp", "-fPIC",
                               "-shared", "-o", _OMP_LIB + ".tmp", _OMP_SRC, "-lm"])
        os.replace(_OMP_LIB + ".tmp", _OMP_LIB)
    return _OMP_LIB


def _load_omp():
    global _omp
    if _omp is None:
        lib = ctypes.CDLL(build_omp())
        P = ctypes.c_void_p
        CP = ctypes.POINTER(_Csr)
        lib.or_pcg_omp.argtypes = [CP, CP, CP, P, P, ctypes.c_int64, P, P, ctypes.c_int64, P, ctypes.c_double,
                                   ctypes.c_int64, ctypes.c_int, P, P, P, P]
        lib.or_pcg_omp.restype = ctypes.c_int
        lib.or_omp_threads.restype = ctypes.c_int
        _omp = lib
    return _omp


def omp_threads() -> int:
    return int(_load_omp().or_omp_threads())


def pcg_omp(A: CSR, L: CSR, U: CSR, b: np.ndarray, eps: float, kmax: int, threads: int = 0):
    """Algorithm 1 on all host cores (OpenMP, level-scheduled SpTRSV over the oracle's
    own level sets).  The multicore CPU baseline (not a parity reference: reductions
    sum in a thread-dependent order).  Returns dict(x, k, rnorm, status, seconds, threads)."""
    wl, levl = levels_lower(L)
    wu, levu = levels_upper(U)
    pl, rl = level_sets(levl, wl)
    pu, ru = level_sets(levu, wu)
    x = np.zeros(A.n)
    k = np.zeros(1, np.int64)
    rn = np.zeros(1)
    sec = np.zeros(1)
    st = _load_omp().or_pcg_omp(ctypes.byref(_in(A)), ctypes.byref(_in(L)), ctypes.byref(_in(U)), _p(pl), _p(rl), wl,
                                _p(pu), _p(ru), wu, _p(np.ascontiguousarray(b, np.float64)), eps, kmax, threads,
                                _p(x), _p(k), _p(rn), _p(sec))
    return dict(x=x, k=int(k[0]), rnorm=float(rn[0]), status=int(st), seconds=float(sec[0]),
                threads=threads if threads > 0 else omp_threads())
