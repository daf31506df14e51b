"""Diagnostics of the chunked executor (not part of the product): per-CTA
timeline of one iteration (SPCG_TRACE) and solver-warp counters (spcg_dbg_counts).

  python tools/diag.py aniso_layered 2048 2048 4 [--K 0] [--k 10]
"""
import argparse
import ctypes
import json
import os
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
tr_path = os.path.join(tempfile.mkdtemp(), "trace.txt")
os.environ["SPCG_TRACE"] = tr_path

import numpy as np  # noqa: E402
import torch  # noqa: E402

import gen  # noqa: E402
from paper_conf_sc_maacsh25_b200 import _build  # noqa: E402

DBG_LIB = _build.LIB.replace("libspcg.so", "libspcg_dbg.so")
if True:   # always rebuild: the knob is compile-time
    _build.build(defines=["-DSPCG_DEBUG_COUNTS=1"], out=DBG_LIB)
os.environ["SPCG_LIB"] = DBG_LIB
import paper_conf_sc_maacsh25_b200 as spcg  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("family")
ap.add_argument("params", type=int, nargs="+")
ap.add_argument("--K", type=int, default=0)
ap.add_argument("--k", type=int, default=10)
ap.add_argument("--mode", default="alg2")
ap.add_argument("--sptrsv", default="chunked")
a = ap.parse_args()

lib = spcg.load(DBG_LIB)
lib.spcg_dbg_counts.argtypes = [ctypes.c_void_p]
A = gen.make(a.family, *a.params)
b, _ = gen.rhs(A)
bd = torch.from_numpy(b).cuda()
h = spcg.SPCG(A, mode=a.mode, K=a.K, sptrsv=a.sptrsv, device=0)
h.solve(bd, eps=0.0, kmax=a.k)                       # warm-up
open(tr_path, "w").close()
cnt = np.zeros(16, np.uint64)
lib.spcg_dbg_counts(cnt.ctypes.data)                 # enable + zero
_, si = h.solve(bd, eps=0.0, kmax=a.k)
lib.spcg_dbg_counts(cnt.ctypes.data)
line = open(tr_path).read().strip().splitlines()[-1].split()
parts = int(line[1].split("=")[1])
t = np.array([int(v) for v in line[2:]], dtype=np.int64)
cta = t[8:8 + 4 * parts].reshape(parts, 4).astype(np.float64)
t0 = cta[cta > 0].min() if (cta > 0).any() else 0
rel = (cta - t0) / 1e3                               # us
iters = a.k
out = {"n": A.n, "levels": [h.info["levels_L"], h.info["levels_U"]], "parts": parts,
       "ms_per_iter": si["iter_phase_ms"] / iters,
       "partition": h.info.get("partition_name"), "counts": {"fast": int(cnt[0]), "ext_fast": int(cnt[1]), "ext_slow": int(cnt[2]), "other_slow": int(cnt[6]),
                  "records": int(cnt[5])},
       "solver_wait_frac": float(cnt[3]) / max(float(cnt[4]), 1.0),
       "records_per_chunk": float(cnt[5]) / max(float(cnt[7]), 1.0),
       "cycles_per_record": {"total": float(cnt[4]) / max(float(cnt[5]), 1.0),
                             "vfull_wait": float(cnt[3]) / max(float(cnt[5]), 1.0),
                             "prep": float(cnt[8]) / max(float(cnt[5]), 1.0),
                             "solve": float(cnt[9]) / max(float(cnt[5]), 1.0)},
       "solver_cycles_per_record": float(cnt[4]) / max(float(cnt[5]), 1.0) / parts * parts,
       "timeline_us": {
           "L_first_record": [float(rel[:, 0].min()), float(np.median(rel[:, 0])), float(rel[:, 0].max())],
           "L_done": [float(rel[:, 1].min()), float(np.median(rel[:, 1])), float(rel[:, 1].max())],
           "U_done": [float(rel[:, 2].min()), float(np.median(rel[:, 2])), float(rel[:, 2].max())],
           "phase_end": [float(rel[:, 3].min()), float(np.median(rel[:, 3])), float(rel[:, 3].max())],
           "cta0": rel[0].tolist(), "cta_last": rel[-1].tolist(), "cta_mid": rel[parts // 2].tolist()}}
print(json.dumps(out))
