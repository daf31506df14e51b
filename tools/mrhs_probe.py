"""NEXT-4 probe (not part of the product): one spcg_solve_multi launch on a layered
field, forced k, for ncu captures and timing.
  python tools/mrhs_probe.py N NRHS K"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_maacsh25_b200 as lib  # noqa: E402

N, m, k = (int(a) for a in sys.argv[1:4])
A = gen.make("aniso_layered", N, N, 4)
h = lib.SPCG(A, setup="gpu")
B = torch.from_numpy(np.stack([gen.rhs(A, seed=99 + j)[0] for j in range(m)])).cuda()
b1 = B[0].clone()
_, si = h.solve(b1, eps=0.0, kmax=k)
_, inf = h.solve_multi(B, eps=0.0, kmax=k)
_, inf = h.solve_multi(B, eps=0.0, kmax=k)
print({"n": A.n, "nrhs": m, "k": k, "single_ms": si["iter_phase_ms"], "multi_ms": inf[0]["iter_phase_ms"],
       "per_rhs_ms": inf[0]["iter_phase_ms"] / m})
