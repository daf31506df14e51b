"""Small-system executor comparison: per-iteration time of every executor on
systems of n <= RESIDENT_MAX_N (the C1 / smoke / small C5 members)."""
import json
import sys
import os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import gen
import paper_conf_sc_maacsh25_b200 as lib

cases = [("poisson2d", (32, 32)), ("aniso_layered", (64, 48, 4)), ("poisson2d", (64, 64)),
         ("poisson3d", (16, 16, 16)), ("fem_q1", (12, 12, 12, 3))]
for fam, prm in cases:
    A = gen.make(fam, *prm)
    b, _ = gen.rhs(A)
    bd = torch.from_numpy(b).cuda()
    K = 2 if fam == "fem_q1" else 0
    row = {"case": f"{fam}{prm}", "n": A.n}
    for ex in ["chunked", "level", "syncfree", "resident"]:
        h = lib.SPCG(A, mode="alg2", K=K, sptrsv=ex)
        for _ in range(3):
            x, si = h.solve(bd, eps=1e-8, kmax=5000)
        ts = []
        for _ in range(10):
            x, si = h.solve(bd, eps=1e-8, kmax=5000)
            ts.append(si["iter_phase_ms"])
        ts.sort()
        row[ex] = {"ms": ts[5], "k": si["iterations"], "us_per_it": 1000 * ts[5] / max(si["iterations"], 1)}
        h.close()
    print(json.dumps(row), flush=True)
