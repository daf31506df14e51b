"""B200-native SPCG: thin Python binding of the C ABI in include/spcg.h.

Argument marshalling only — every step of the iterative phase runs in the
sm_100a kernels of libspcg.so, and the preconditioner construction runs in the
library's host C++.  There is NO Python or CPU fallback: if the extension is
missing, importing the binding raises.  PyTorch is used only for device memory
and streams (``torch.Tensor.data_ptr()`` / ``torch.cuda.current_stream()``).

Names follow the paper: ``spcg_setup(A, drop_params, K)`` builds Â (Algorithm 2)
and M = {L, U} = ILU(K)(Â); ``spcg_solve(b, x, eps, kmax)`` runs Algorithm 1.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

from . import _build

_LIB_PATH = os.environ.get("SPCG_LIB", _build.LIB)   # SPCG_LIB: an experiment variant of the same library
_lib = None

OK, NOT_CONVERGED = 0, 1
ERR_INVALID_ARG, ERR_BAD_MATRIX, ERR_ZERO_PIVOT, ERR_BREAKDOWN = -1, -2, -3, -4
ERR_OOM, ERR_CUDA, ERR_INTERNAL, ERR_NO_DEVICE = -5, -6, -7, -8

DROP_NONE, DROP_FIXED, DROP_WAVEFRONT_AWARE = 0, 1, 2
SPTRSV = {"auto": 0, "level": 1, "syncfree": 2, "chunked": 3, "resident": 4, "wchain": 5}
EXEC = {"auto": 0, "persistent": 1, "graph_while": 2}
PARTITION_NAME = {0: "contiguous", 1: "strided", 2: "affinity", 3: "components", 4: "tiles",
                  5: "chain-components", 6: "chain-grid3d", 7: "chain-grid2d"}
RESIDENT_MAX_N = 4096          # include/spcg.h SPCG_RESIDENT_MAX_N
SPTRSV_NAME = {v: k for k, v in SPTRSV.items()}
USE_X0, HOST_PTRS = 0x1, 0x2

EXPORT = dict(ahat_rowptr=1, ahat_col=2, ahat_val=3, l_rowptr=4, l_col=5, l_val=6, u_rowptr=7, u_col=8,
              u_val=9, fill_level=10, level_l=11, level_u=12, levelptr_l=13, levelrows_l=14,
              levelptr_u=15, levelrows_u=16, rhist=17, dbg_stream=100, dbg_part_chunk=101, dbg_part_uchunk=102,
              dbg_part_begin=103, dbg_chain_recl=104, dbg_chain_recu=105, dbg_chain_perm=106,
              dbg_chain_step=107, dbg_chain_flags=108, dbg_chain_a_eoff=109, dbg_chain_a_col=110,
              dbg_chain_a_val=111)
_EXPORT_DT = dict(ahat_rowptr=np.int64, ahat_col=np.int32, ahat_val=np.float64, l_rowptr=np.int64,
                  l_col=np.int32, l_val=np.float64, u_rowptr=np.int64, u_col=np.int32, u_val=np.float64,
                  fill_level=np.int32, level_l=np.int32, level_u=np.int32, levelptr_l=np.int64,
                  levelrows_l=np.int32, levelptr_u=np.int64, levelrows_u=np.int32, rhist=np.float64,
                  dbg_stream=np.uint8, dbg_part_chunk=np.int32, dbg_part_uchunk=np.int32, dbg_part_begin=np.int64,
                  dbg_chain_recl=np.uint8, dbg_chain_recu=np.uint8, dbg_chain_perm=np.int32, dbg_chain_step=np.int64,
                  dbg_chain_flags=np.uint32, dbg_chain_a_eoff=np.int64, dbg_chain_a_col=np.int32,
                  dbg_chain_a_val=np.float64)


class SpcgError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"spcg status {status}: {msg}")
        self.status = status


class _CsrT(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("nnz", ctypes.c_int64), ("row_ptr", ctypes.c_void_p),
                ("col_idx", ctypes.c_void_p), ("val", ctypes.c_void_p)]


class DropParams(ctypes.Structure):
    _fields_ = [("mode", ctypes.c_int32), ("fixed_pct", ctypes.c_double), ("n_ratios", ctypes.c_int32),
                ("ratios_pct", ctypes.c_double * 8), ("tau", ctypes.c_double), ("omega_pct", ctypes.c_double),
                ("norm_reading", ctypes.c_int32), ("reduction_denominator", ctypes.c_int32)]


_ALLOC_FN = ctypes.CFUNCTYPE(ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_void_p)
_FREE_FN = ctypes.CFUNCTYPE(None, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_void_p)


class Options(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int32), ("stream", ctypes.c_void_p), ("sptrsv", ctypes.c_int32),
                ("parts", ctypes.c_int32), ("host_threads", ctypes.c_int32), ("exec", ctypes.c_int32),
                ("dev_alloc", _ALLOC_FN), ("dev_free", _FREE_FN), ("alloc_ctx", ctypes.c_void_p),
                ("wide_min", ctypes.c_double), ("chunk_partition", ctypes.c_int32),
                ("setup_device", ctypes.c_int32), ("factor_precision", ctypes.c_int32),
                ("reserved", ctypes.c_int32 * 5)]


class SetupInfo(ctypes.Structure):
    _fields_ = [("chosen_pct", ctypes.c_double), ("m_t", ctypes.c_int64), ("w_A", ctypes.c_int64),
                ("w_Ahat", ctypes.c_int64), ("n_tried", ctypes.c_int32), ("tried_pct", ctypes.c_double * 8),
                ("indicator", ctypes.c_double * 8), ("tried_w", ctypes.c_int64 * 8),
                ("tried_reduction_pct", ctypes.c_double * 8), ("n", ctypes.c_int64), ("nnz_A", ctypes.c_int64),
                ("nnz_Ahat", ctypes.c_int64), ("nnz_L", ctypes.c_int64), ("nnz_U", ctypes.c_int64),
                ("levels_L", ctypes.c_int64), ("levels_U", ctypes.c_int64), ("zero_pivot_row", ctypes.c_int64),
                ("setup_ms_validate", ctypes.c_double), ("setup_ms_sparsify", ctypes.c_double),
                ("setup_ms_symbolic", ctypes.c_double), ("setup_ms_numeric", ctypes.c_double),
                ("setup_ms_layout", ctypes.c_double), ("setup_ms_upload", ctypes.c_double),
                ("sptrsv", ctypes.c_int32), ("parts", ctypes.c_int32), ("device_bytes", ctypes.c_int64),
                ("algo_bytes_per_iter", ctypes.c_double), ("algo_flops_per_iter", ctypes.c_double),
                ("partition", ctypes.c_int32), ("chains", ctypes.c_int32), ("positions", ctypes.c_int64),
                ("chain_entries", ctypes.c_int64 * 4), ("setup_device", ctypes.c_int32),
                ("setup_ms_total", ctypes.c_double), ("factor_precision", ctypes.c_int32),
                ("record_value_bytes", ctypes.c_int32)]


class SolveInfo(ctypes.Structure):
    _fields_ = [("iterations", ctypes.c_int64), ("rnorm", ctypes.c_double), ("converged", ctypes.c_int32),
                ("status", ctypes.c_int32), ("iter_phase_ms", ctypes.c_double), ("total_ms", ctypes.c_double)]


EXPORTED = ["spcg_abi_version", "spcg_status_string", "spcg_last_error", "spcg_drop_params_default",
            "spcg_options_default", "spcg_setup", "spcg_get_setup_info", "spcg_solve", "spcg_apply_spmv",
            "spcg_apply_lower", "spcg_apply_upper", "spcg_apply_precond", "spcg_export", "spcg_destroy",
            "spcg_calibrate", "spcg_solve_async", "spcg_solve_wait", "spcg_set_stream", "spcg_ll_stress",
            "spcg_solve_multi"]


def load(path: str | None = None):
    """Load libspcg.so (raises if it is missing: there is no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    path = path or _LIB_PATH
    if not os.path.exists(path):
        raise ImportError(f"libspcg.so not built ({path}); run __graft_entry__.build()")
    lib = ctypes.CDLL(path)
    V, P, I32, I64, D = ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_double
    lib.spcg_abi_version.restype = I32
    lib.spcg_status_string.restype = ctypes.c_char_p
    lib.spcg_status_string.argtypes = [I32]
    lib.spcg_last_error.restype = ctypes.c_char_p
    lib.spcg_drop_params_default.argtypes = [ctypes.POINTER(DropParams)]
    lib.spcg_options_default.argtypes = [ctypes.POINTER(Options)]
    lib.spcg_setup.argtypes = [ctypes.POINTER(_CsrT), ctypes.POINTER(DropParams), I32, ctypes.POINTER(Options),
                               ctypes.POINTER(V)]
    lib.spcg_setup.restype = I32
    lib.spcg_get_setup_info.argtypes = [V, ctypes.POINTER(SetupInfo)]
    lib.spcg_get_setup_info.restype = I32
    lib.spcg_solve.argtypes = [V, P, P, D, I64, ctypes.c_uint32, ctypes.POINTER(SolveInfo)]
    lib.spcg_solve.restype = I32
    lib.spcg_apply_spmv.argtypes = [V, P, P, ctypes.POINTER(D)]
    lib.spcg_apply_spmv.restype = I32
    lib.spcg_apply_lower.argtypes = [V, P, P]
    lib.spcg_apply_lower.restype = I32
    lib.spcg_apply_upper.argtypes = [V, P, P, P, ctypes.POINTER(D)]
    lib.spcg_apply_upper.restype = I32
    lib.spcg_apply_precond.argtypes = [V, P, P, ctypes.POINTER(D)]
    lib.spcg_apply_precond.restype = I32
    lib.spcg_export.argtypes = [V, I32, P, ctypes.POINTER(ctypes.c_size_t)]
    lib.spcg_export.restype = I32
    lib.spcg_destroy.argtypes = [V]
    lib.spcg_destroy.restype = None
    lib.spcg_solve_async.argtypes = [V, P, P, D, I64, ctypes.c_uint32]
    lib.spcg_solve_async.restype = I32
    lib.spcg_solve_wait.argtypes = [V, ctypes.POINTER(SolveInfo)]
    lib.spcg_solve_wait.restype = I32
    lib.spcg_set_stream.argtypes = [V, V]
    lib.spcg_set_stream.restype = I32
    lib.spcg_calibrate.argtypes = [I32, ctypes.POINTER(Calib)]
    lib.spcg_calibrate.restype = I32
    lib.spcg_solve_multi.argtypes = [V, P, P, I32, D, I64, ctypes.c_uint32, ctypes.POINTER(SolveInfo)]
    lib.spcg_solve_multi.restype = I32
    lib.spcg_ll_stress.argtypes = [I32, I32, I32, ctypes.POINTER(ctypes.c_uint64)]
    lib.spcg_ll_stress.restype = I32
    if lib.spcg_abi_version() != 3:
        raise ImportError("libspcg ABI version mismatch")
    _lib = lib
    return lib


class Calib(ctypes.Structure):
    _fields_ = [("grid_sync_ns", ctypes.c_double), ("graph_kernel_ns", ctypes.c_double),
                ("flag_same_die_ns", ctypes.c_double), ("flag_cross_die_ns", ctypes.c_double),
                ("syncthreads_ns", ctypes.c_double), ("cluster_sync_ns", ctypes.c_double),
                ("sm_clock_mhz", ctypes.c_double), ("sms", ctypes.c_int32), ("flag_pairs_near", ctypes.c_int32),
                ("flag_relaxed_same_die_ns", ctypes.c_double), ("flag_relaxed_cross_die_ns", ctypes.c_double)]


def calibrate(device: int = 0) -> dict:
    """spcg_calibrate: handoff costs for the chain floor."""
    c = Calib()
    _check(load().spcg_calibrate(device, ctypes.byref(c)), "spcg_calibrate")
    return {f: getattr(c, f) for f, _ in Calib._fields_}


def ll_stress(device: int = 0, nslots: int = 4096, rounds: int = 2000) -> dict:
    """spcg_ll_stress: torn / mixed / good reads of the 16-byte LL ready flags."""
    out = (ctypes.c_uint64 * 3)()
    _check(load().spcg_ll_stress(device, nslots, rounds, out), "spcg_ll_stress")
    return {"torn": int(out[0]), "mixed": int(out[1]), "ok": int(out[2])}


def _check(st, what=""):
    if st < 0:
        lib = load()
        raise SpcgError(st, f"{what}: {lib.spcg_status_string(st).decode()} — {lib.spcg_last_error().decode()}")
    return st


def drop_params(mode="alg2", fixed_pct=0.0, ratios=(10.0, 5.0, 1.0), tau=1.0, omega=10.0, norm="fro",
                denominator="w_A") -> DropParams:
    p = DropParams()
    load().spcg_drop_params_default(ctypes.byref(p))
    p.mode = {"none": DROP_NONE, "fixed": DROP_FIXED, "alg2": DROP_WAVEFRONT_AWARE}[mode]
    p.fixed_pct = fixed_pct
    p.n_ratios = len(ratios)
    for i, r in enumerate(ratios):
        p.ratios_pct[i] = r
    p.tau = tau
    p.omega_pct = omega
    p.norm_reading = {"fro": 0, "inf": 1, "spectral": 2}[norm]
    p.reduction_denominator = {"w_A": 0, "w_Ahat": 1}[denominator]
    return p


def _torch():
    import torch
    return torch


class _TorchAllocator:
    """spcg_options_t.dev_alloc / dev_free backed by PyTorch's caching allocator, so the
    library's device buffers are owned by torch (north_star: PyTorch provides device
    memory and streams).  The ctypes callbacks are kept alive by the handle."""

    def __init__(self, device: int):
        torch = _torch()
        self.device = device
        self.live = {}

        def _alloc(nbytes, stream, ctx):
            try:
                ptr = torch.cuda.caching_allocator_alloc(int(nbytes), self.device, int(stream or 0))
            except Exception:          # OOM: the library reports SPCG_ERR_OOM
                return None
            self.live[ptr] = nbytes
            return ptr

        def _free(ptr, nbytes, stream, ctx):
            if ptr in self.live:
                del self.live[ptr]
                try:
                    torch.cuda.caching_allocator_delete(ptr)
                except Exception:      # interpreter shutdown: the process frees the device memory
                    pass

        self.alloc_fn = _ALLOC_FN(_alloc)
        self.free_fn = _FREE_FN(_free)


class SPCG:
    """A set-up SPCG preconditioner + solver bound to one device (or host-only, device=-1).

    allocator: "torch" (default: device buffers from PyTorch's caching allocator through
    the spcg_options_t hooks) or "cuda" (the library's own cudaMalloc).
    setup: "host" (default) or "gpu" (NEXT-1: validation, Algorithm 2, ILU(0) and the
    level sets on the device; K = 0 only, other K run on the host).
    factors: "f64" (default) or "f32" (NEXT-2: factor values rounded to fp32, the paper's
    preconditioner precision; vectors stay fp64)."""

    def __init__(self, A, mode="alg2", K=0, fixed_pct=0.0, sptrsv="auto", parts=0, device=0, stream=None,
                 host_threads=0, allocator="torch", exec="auto", wide_min=0.0, chunk_partition=-1, setup="host",
                 factors="f64", **drop_kw):
        lib = load()
        rp = np.ascontiguousarray(A.row_ptr, np.int64)
        col = np.ascontiguousarray(A.col, np.int32)
        val = np.ascontiguousarray(A.val, np.float64)
        self.n = int(A.n)
        c = _CsrT(self.n, int(rp[-1]), rp.ctypes.data, col.ctypes.data, val.ctypes.data)
        dp = drop_params(mode, fixed_pct, **drop_kw)
        opt = Options()
        lib.spcg_options_default(ctypes.byref(opt))
        opt.device = device
        opt.sptrsv = SPTRSV[sptrsv] if isinstance(sptrsv, str) else int(sptrsv)
        opt.parts = parts
        opt.host_threads = host_threads
        opt.exec = EXEC[exec]
        opt.wide_min = wide_min
        opt.chunk_partition = chunk_partition
        opt.setup_device = {"host": 0, "gpu": 1}[setup]
        opt.factor_precision = {"f64": 0, "f32": 1}[factors]
        self.device = device
        self._alloc = None
        if device >= 0:
            torch = _torch()
            if stream is None:
                stream = torch.cuda.current_stream(device)
            self.stream = stream
            opt.stream = stream.cuda_stream
            if allocator == "torch":
                self._alloc = _TorchAllocator(device)
                opt.dev_alloc = self._alloc.alloc_fn
                opt.dev_free = self._alloc.free_fn
        h = ctypes.c_void_p()
        _check(lib.spcg_setup(ctypes.byref(c), ctypes.byref(dp), K, ctypes.byref(opt), ctypes.byref(h)), "spcg_setup")
        self._h = h
        si = SetupInfo()
        _check(lib.spcg_get_setup_info(h, ctypes.byref(si)))
        self.info = {f[0]: (list(getattr(si, f[0])) if isinstance(getattr(si, f[0]), ctypes.Array)
                            else getattr(si, f[0])) for f in SetupInfo._fields_}
        self.info["sptrsv_name"] = SPTRSV_NAME.get(self.info["sptrsv"], "?")
        self.info["partition_name"] = PARTITION_NAME.get(self.info["partition"], "-")

    def close(self):
        h = getattr(self, "_h", None)
        self._h = None
        if h and _lib is not None:
            try:
                _lib.spcg_destroy(h)
            except Exception:      # interpreter shutdown
                pass

    __del__ = close

    # ------------------------------------------------------------ export
    def export(self, what: str) -> np.ndarray:
        lib = load()
        nb = ctypes.c_size_t(0)
        _check(lib.spcg_export(self._h, EXPORT[what], None, ctypes.byref(nb)))
        dt = _EXPORT_DT[what]
        out = np.zeros(nb.value // np.dtype(dt).itemsize, dt)
        _check(lib.spcg_export(self._h, EXPORT[what], out.ctypes.data, ctypes.byref(nb)))
        return out

    def factors(self):
        L = (self.export("l_rowptr"), self.export("l_col"), self.export("l_val"))
        U = (self.export("u_rowptr"), self.export("u_col"), self.export("u_val"))
        return L, U

    # ------------------------------------------------------------ solve
    def _order_after_current(self, *tensors):
        """The handle's stream waits (on the device) for the caller's current stream, where
        b / x were produced; tensors used asynchronously are recorded on the handle's stream
        so the caching allocator does not recycle them early."""
        torch = _torch()
        cur = torch.cuda.current_stream(self.device)
        if cur.cuda_stream != self.stream.cuda_stream:
            ev = torch.cuda.Event()
            ev.record(cur)
            self.stream.wait_event(ev)
            for t in tensors:
                t.record_stream(self.stream)

    def solve(self, b, x=None, eps=1e-8, kmax=10000, use_x0=False):
        """b, x: float64 CUDA tensors of length n on this handle's device (x allocated if None)."""
        torch = _torch()
        assert b.dtype == torch.float64 and b.is_cuda and b.is_contiguous() and b.numel() == self.n
        if x is None:
            x = torch.empty_like(b)
        self._order_after_current(b, x)
        info = SolveInfo()
        flags = USE_X0 if use_x0 else 0
        st = load().spcg_solve(self._h, b.data_ptr(), x.data_ptr(), float(eps), int(kmax), flags, ctypes.byref(info))
        _check(st, "spcg_solve")
        return x, self._solve_info(info)

    def solve_multi(self, B, X=None, eps=1e-8, kmax=10000):
        """spcg_solve_multi (NEXT-4): B is an (nrhs, n) float64 CUDA tensor, one right-hand
        side per row (= the column-major n x nrhs block of the C ABI); returns (X, [info])."""
        torch = _torch()
        assert B.dtype == torch.float64 and B.is_cuda and B.is_contiguous() and B.dim() == 2 and B.shape[1] == self.n
        nrhs = int(B.shape[0])
        if X is None:
            X = torch.empty_like(B)
        self._order_after_current(B, X)
        infos = (SolveInfo * nrhs)()
        st = load().spcg_solve_multi(self._h, B.data_ptr(), X.data_ptr(), nrhs, float(eps), int(kmax), 0, infos)
        if st < 0 and st != ERR_BREAKDOWN:
            _check(st, "spcg_solve_multi")
        return X, [self._solve_info(infos[j]) for j in range(nrhs)]

    def solve_async(self, b, x, eps=1e-8, kmax=10000):
        """spcg_solve_async: enqueue on the handle's stream (b, x device tensors kept alive by the caller)."""
        self._order_after_current(b, x)
        _check(load().spcg_solve_async(self._h, b.data_ptr(), x.data_ptr(), float(eps), int(kmax), 0),
               "spcg_solve_async")

    def set_stream(self, stream):
        """spcg_set_stream: later solves of this handle run on `stream` (a torch.cuda.Stream)."""
        _check(load().spcg_set_stream(self._h, stream.cuda_stream), "spcg_set_stream")
        self.stream = stream

    def solve_wait(self):
        """spcg_solve_wait: finish the in-flight solve, returns its info dict."""
        info = SolveInfo()
        st = load().spcg_solve_wait(self._h, ctypes.byref(info))
        _check(st, "spcg_solve_wait")
        return self._solve_info(info)

    def solve_host(self, b, eps=1e-8, kmax=10000, x0=None, out=None):
        """Host buffers: the library copies b (and x0) in and x out inside the call (e2e path).
        b: numpy array or (pinned) CPU torch tensor; out: optional host buffer of the same kind
        for x (returned)."""
        if isinstance(b, np.ndarray):
            b = np.ascontiguousarray(b, np.float64)
            bp = b.ctypes.data
            x = out if out is not None else np.zeros(self.n)
            if x0 is not None:
                x[:] = x0
            xp = x.ctypes.data
        else:                                    # CPU torch tensor (e.g. pin_memory=True)
            assert not b.is_cuda and b.is_contiguous() and b.numel() == self.n
            bp = b.data_ptr()
            x = out if out is not None else _torch().zeros_like(b)
            if x0 is not None:
                x.copy_(_torch().as_tensor(x0))
            xp = x.data_ptr()
        info = SolveInfo()
        flags = HOST_PTRS | (USE_X0 if x0 is not None else 0)
        st = load().spcg_solve(self._h, bp, xp, float(eps), int(kmax), flags, ctypes.byref(info))
        _check(st, "spcg_solve")
        return x, self._solve_info(info)

    @staticmethod
    def _solve_info(info):
        return dict(iterations=info.iterations, rnorm=info.rnorm, converged=bool(info.converged),
                    status=info.status, iter_phase_ms=info.iter_phase_ms, total_ms=info.total_ms)

    def rhist(self) -> np.ndarray:
        return self.export("rhist")

    # ------------------------------------------------------------ single operators
    def apply_spmv(self, p, w):
        d = ctypes.c_double(0.0)
        _check(load().spcg_apply_spmv(self._h, p.data_ptr(), w.data_ptr(), ctypes.byref(d)), "spmv")
        return d.value

    def apply_lower(self, r, y):
        _check(load().spcg_apply_lower(self._h, r.data_ptr(), y.data_ptr()), "lower")

    def apply_upper(self, y, z, r=None):
        d = ctypes.c_double(0.0)
        _check(load().spcg_apply_upper(self._h, y.data_ptr(), z.data_ptr(), None if r is None else r.data_ptr(),
                                       ctypes.byref(d)), "upper")
        return d.value

    def apply_precond(self, r, z):
        d = ctypes.c_double(0.0)
        _check(load().spcg_apply_precond(self._h, r.data_ptr(), z.data_ptr(), ctypes.byref(d)), "precond")
        return d.value


def spcg_setup(A, drop_params=None, K=0, **kw) -> SPCG:
    """Paper-named entry point: sparsify (Alg. 2), ILU(K), level sets, upload."""
    kw = dict(kw)
    if drop_params is not None:
        kw.update(drop_params)
    return SPCG(A, K=K, **kw)


def spcg_solve(h: SPCG, b, x=None, eps=1e-8, kmax=10000):
    """Paper-named entry point: Algorithm 1 on the device."""
    return h.solve(b, x, eps, kmax)
