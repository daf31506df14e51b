"""Experiment helper: ms per iteration of the persistent solve for one library
variant (SPCG_LIB=...), forced-k, on a chosen matrix.  Not part of the product.

  SPCG_LIB=.../libspcg_vg1.so python tools/exp_iter.py aniso_layered 2048 2048 4 --k 30
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_maacsh25_b200 as spcg  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("family")
ap.add_argument("params", type=int, nargs="+")
ap.add_argument("--k", type=int, default=30)
ap.add_argument("--K", type=int, default=0)
ap.add_argument("--modes", default="alg2,none")
ap.add_argument("--sptrsv", default="auto")
ap.add_argument("--reps", type=int, default=5)
ap.add_argument("--parts", type=int, default=0)
ap.add_argument("--tag", default=os.path.basename(os.environ.get("SPCG_LIB", "libspcg.so")))
a = ap.parse_args()

A = gen.make(a.family, *a.params)
b, _ = gen.rhs(A)
bd = torch.from_numpy(b).cuda()
out = {"tag": a.tag, "family": a.family, "params": a.params, "n": A.n, "parts_req": a.parts}
for mode in a.modes.split(","):
    h = spcg.SPCG(A, mode=mode, K=a.K, sptrsv=a.sptrsv, parts=a.parts, device=0)
    x, si = h.solve(bd, eps=1e-8, kmax=10000)
    k_conv = si["iterations"]
    ms = []
    for _ in range(a.reps):
        _, sf = h.solve(bd, eps=0.0, kmax=a.k)
        assert sf["status"] == 0, sf
        ms.append(sf["iter_phase_ms"])
    out[mode] = {"k_conv": k_conv, "conv_ms": si["iter_phase_ms"], "ms_per_iter_forced": float(np.median(ms)) / a.k,
                 "levels": [h.info["levels_L"], h.info["levels_U"]], "sptrsv": h.info["sptrsv_name"],
                 "partition": h.info.get("partition_name", "")}
    h.close()
print(json.dumps(out))
