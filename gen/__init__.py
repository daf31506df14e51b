"""Seeded synthetic SPD workload generators (the shared INPUT module).

Holds none of the SPCG method's arithmetic: it only writes A (full symmetric
CSR, int64 row_ptr / int32 col / f64 val), b and x_true.  Both the oracle
(``oracle/``) and the CUDA library consume these inputs.  Recipe: SURVEY.md
§8(d) "Workloads", restated in DESIGN.md §3.  The C source is
``gen/spcg_gen.c``; it is compiled in-tree with gcc on first use.
"""
from __future__ import annotations

import ctypes
import math
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "spcg_gen.c")
_LIB = os.path.join(_HERE, "libspcg_gen.so")
_lib = None

FAMILIES = {"poisson2d": 0, "poisson3d": 1, "fem_q1": 2, "aniso_layered": 3}


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fPIC", "-shared",
                               "-o", _LIB + ".tmp", _SRC, "-lm"])
        os.replace(_LIB + ".tmp", _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        P = ctypes.c_void_p
        lib.gen_count.argtypes = [ctypes.c_int, P, P, P]
        lib.gen_fill.argtypes = [ctypes.c_int, P, P, P, P]
        lib.gen_rhs.argtypes = [ctypes.c_int64, P, P, P, ctypes.c_uint64, P, P]
        lib.gen_u.argtypes = [ctypes.c_uint64, ctypes.c_uint64]
        lib.gen_u.restype = ctypes.c_double
        _lib = lib
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


@dataclass
class CSR:
    """Full symmetric CSR, 0-based: row_ptr int64[n+1], col int32[nnz], val f64[nnz]."""
    n: int
    row_ptr: np.ndarray
    col: np.ndarray
    val: np.ndarray
    name: str = ""

    @property
    def nnz(self) -> int:
        return int(self.row_ptr[-1])

    def to_scipy(self):
        import scipy.sparse as sp
        return sp.csr_matrix((self.val, self.col, self.row_ptr), shape=(self.n, self.n))

    def to_dense(self) -> np.ndarray:
        d = np.zeros((self.n, self.n))
        for i in range(self.n):
            for q in range(self.row_ptr[i], self.row_ptr[i + 1]):
                d[i, self.col[q]] += self.val[q]
        return d


def u(seed: int, i: int) -> float:
    """The survey's counter RNG u(seed, i) in [0, 1)."""
    return float(_load().gen_u(seed, i))


def make(family: str, *params: int) -> CSR:
    fam = FAMILIES[family]
    lib = _load()
    p = np.zeros(8, dtype=np.int64)
    p[: len(params)] = params
    n = np.zeros(1, np.int64)
    nnz = np.zeros(1, np.int64)
    if lib.gen_count(fam, _ptr(p), _ptr(n), _ptr(nnz)) != 0:
        raise ValueError(family)
    rp = np.zeros(int(n[0]) + 1, np.int64)
    col = np.zeros(int(nnz[0]), np.int32)
    val = np.zeros(int(nnz[0]), np.float64)
    lib.gen_fill(fam, _ptr(p), _ptr(rp), _ptr(col), _ptr(val))
    return CSR(int(n[0]), rp, col, val, name=f"{family}{tuple(params)}")


def rhs(A: CSR, seed: int = 99):
    """b = A x_true with x_true_i = 2u(seed,i)-1, both scaled so ||b||_2 = 1."""
    b = np.zeros(A.n)
    xt = np.zeros(A.n)
    _load().gen_rhs(A.n, _ptr(A.row_ptr), _ptr(A.col), _ptr(A.val), seed, _ptr(b), _ptr(xt))
    return b, xt


def from_dense(d: np.ndarray, name: str = "dense") -> CSR:
    """Tiny hand-built matrices for pins (structural entries = non-zero entries)."""
    n = d.shape[0]
    rp = [0]
    cols, vals = [], []
    for i in range(n):
        for j in range(n):
            if d[i, j] != 0.0 or i == j:
                cols.append(j)
                vals.append(d[i, j])
        rp.append(len(cols))
    return CSR(n, np.array(rp, np.int64), np.array(cols, np.int32), np.array(vals, np.float64), name)


# ---------------------------------------------------------------- configs
# BASELINE.json configs, SURVEY.md §8 table.  ``small`` variants keep the same
# family/structure at sizes the oracle finishes in seconds.
CONFIGS = {
    "C1": dict(family="poisson2d", params=(32, 32), K=0),
    "C2": dict(family="poisson3d", params=(64, 64, 64), K=0),
    "C3": dict(family="fem_q1", params=(128, 128, 128, 3), K=2),
    "C4": dict(family="aniso_layered", params=(4096, 4096, 4), K=0),
}


def config_matrix(name: str) -> CSR:
    c = CONFIGS[name]
    A = make(c["family"], *c["params"])
    A.name = name
    return A


def batch_spec(i: int):
    """C5 system i: family i mod 4, size exponent s = 12 + floor(9 u(7,i)),
    n ~ 2^s with side = round(sqrt or cbrt), seed 1000+i, K = 2 for fem_q1 else 0."""
    fams = ["poisson2d", "poisson3d", "fem_q1", "aniso_layered"]
    fam = fams[i % 4]
    s = 12 + int(math.floor(9.0 * u(7, i)))
    seed = 1000 + i
    if fam in ("poisson2d", "aniso_layered"):
        side = int(round(math.sqrt(2.0 ** s)))
        params = (side, side) if fam == "poisson2d" else (side, side, seed)
    else:
        side = int(round((2.0 ** s) ** (1.0 / 3.0)))
        params = (side, side, side) if fam == "poisson3d" else (side, side, side, seed)
    return dict(family=fam, params=params, K=2 if fam == "fem_q1" else 0, seed=seed)
