"""C5's makespan-bounding member (Poisson-2D 1024^2, Alg. 2 -> t = 1 %): per-iteration
time against the CTA count it gets (C5 lanes give it 37 of 148)."""
import json
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import gen
import paper_conf_sc_maacsh25_b200 as lib

A = gen.make("poisson2d", 1024, 1024)
b, _ = gen.rhs(A)
bd = torch.from_numpy(b).cuda()
for parts in (148, 74, 37, 16):
    h = lib.SPCG(A, mode="alg2", K=0, parts=parts)
    x, si = h.solve(bd, eps=0.0, kmax=20)
    x, si = h.solve(bd, eps=0.0, kmax=60)
    print(json.dumps({"parts": parts, "partition": h.info.get("partition_name"), "us_per_it": 1000 * si["iter_phase_ms"] / 60,
                      "levels_L": h.info["levels_L"]}), flush=True)
    h.close()
