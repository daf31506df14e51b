#!/usr/bin/env python
"""Warp-chain executor diagnostics (not part of the product): per-iteration time and,
with a -DSPCG_CHAIN_PROF=1 build (SPCG_LIB=...), per-pass cycle counters: cycles per
step, cycles blocked on the stage mbarrier, cycles in the flag prefetch.

  SPCG_LIB=paper_conf_sc_maacsh25_b200/libspcg_prof.so python tools/chain_prof.py fam p1 p2 [p3] [mode]
"""
import ctypes
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_maacsh25_b200 as lib  # noqa: E402


def main():
    args = sys.argv[1:]
    mode = args[-1] if args[-1] in ("alg2", "none") else "alg2"
    nums = [int(a) for a in args[1:] if a.lstrip("-").isdigit()]
    fam = args[0]
    A = gen.make(fam, *nums)
    b, _ = gen.rhs(A)
    L = lib.load()
    prof = hasattr(L, "spcg_dbg_chain_prof")
    buf = (ctypes.c_ulonglong * 24)()
    if prof:
        L.spcg_dbg_chain_prof(buf)
    t = time.time()
    h = lib.SPCG(A, mode=mode, K=0, sptrsv=os.environ.get("SPTRSV", "auto"))
    setup_s = time.time() - t
    bd = torch.from_numpy(b).cuda()
    k = int(os.environ.get("K", "10"))
    h.solve(bd, eps=0.0, kmax=k)
    if prof:
        L.spcg_dbg_chain_prof(buf)
    _, info = h.solve(bd, eps=0.0, kmax=k)
    out = dict(case=f"{fam}{tuple(nums)}", mode=mode, n=A.n, sptrsv=h.info["sptrsv_name"],
               partition=h.info["partition_name"], chains=h.info["chains"], ctas=h.info["parts"],
               levels=h.info["levels_L"], setup_s=round(setup_s, 2), ms_per_iter=info["iter_phase_ms"] / (k + 1),
               entries=list(h.info["chain_entries"]))
    if prof and L.spcg_dbg_chain_prof(buf) == 1:
        v = list(buf)
        for nm, o in (("L", 0), ("U", 8)):
            passes = max(v[o + 6], 1)
            steps = max(v[o + 3], 1)
            out[nm] = dict(passes=v[o + 6], cyc_per_step=v[o + 0] / steps, wait_per_step=v[o + 1] / steps,
                           ext_per_step=v[o + 2] / steps, steps_per_pass=steps / passes, chunks=v[o + 4],
                           gen_passes=v[o + 5])
        it = max(k, 1) * int(out["ctas"])
        out["phase_cyc_per_iter_per_cta"] = dict(spmv=v[16] / it, spmv_bar=v[17] / it, tri=v[18] / it,
                                                 tri_bar=v[19] / it, pupd=v[20] / it, pupd_bar=v[21] / it,
                                                 spmv_warp_wait=v[22] / it / 8, spmv_warp_total=v[23] / it / 8)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
