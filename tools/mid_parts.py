"""Mid-size narrow systems (4096 < n <= 16384, C5's aniso/Poisson members): chunked
executor per-iteration time against the CTA count (default: 1 CTA)."""
import json
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import gen
import paper_conf_sc_maacsh25_b200 as lib

for fam, prm in [("aniso_layered", (128, 128, 1007)), ("poisson2d", (128, 128)), ("poisson3d", (25, 25, 25)),
                 ("aniso_layered", (90, 91, 1005))]:
    A = gen.make(fam, *prm)
    b, _ = gen.rhs(A)
    bd = torch.from_numpy(b).cuda()
    for parts in (1, 2, 4, 8, 16, 37):
        h = lib.SPCG(A, mode="alg2", K=0, parts=parts)
        x, si = h.solve(bd, eps=0.0, kmax=3)
        x, si = h.solve(bd, eps=0.0, kmax=20)
        print(json.dumps({"case": f"{fam}{prm}", "n": A.n, "parts": h.info["parts"], "sptrsv": h.info["sptrsv_name"],
                          "partition": h.info.get("partition_name"), "us_per_it": 1000 * si["iter_phase_ms"] / 20,
                          "levels_L": h.info["levels_L"]}), flush=True)
        h.close()
