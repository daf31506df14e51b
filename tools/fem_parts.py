"""Small FEM ILU(2) systems (C5's fem_q1 members, wide rows -> sync-free executor):
per-iteration time against the CTA count."""
import json
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import gen
import paper_conf_sc_maacsh25_b200 as lib

for N in (12, 20, 32, 40):
    A = gen.make("fem_q1", N, N, N, 1000 + N)
    b, _ = gen.rhs(A)
    bd = torch.from_numpy(b).cuda()
    for parts in (1, 4, 16, 37, 148):
        h = lib.SPCG(A, mode="alg2", K=2, parts=parts)
        x, si = h.solve(bd, eps=0.0, kmax=3)
        x, si = h.solve(bd, eps=0.0, kmax=10)
        print(json.dumps({"N": N, "n": A.n, "parts": h.info["parts"], "sptrsv": h.info["sptrsv_name"],
                          "us_per_it": 1000 * si["iter_phase_ms"] / 10, "levels_L": h.info["levels_L"]}), flush=True)
        h.close()
