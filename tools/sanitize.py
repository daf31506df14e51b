#!/usr/bin/env python
"""compute-sanitizer driver (not part of the product): small solves and single
operators on every executor, for

  compute-sanitizer --tool memcheck|synccheck|racecheck python tools/sanitize.py

Each case: one solve to eps = 1e-8 (kmax 300), one forced-k solve, apply_lower /
apply_upper / apply_spmv; results checked against each other loosely (the parity
tests do the real checking) so a sanitizer-induced abort shows up as a failed case.
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_maacsh25_b200 as lib  # noqa: E402

CASES = [("poisson2d", (37, 29), 0), ("poisson3d", (13, 11, 9), 0), ("fem_q1", (9, 8, 7, 3), 2),
         ("aniso_layered", (150, 67, 4), 0)]
EXECS = sys.argv[1].split(",") if len(sys.argv) > 1 else ["level", "syncfree", "chunked", "resident", "wchain"]


def main():
    fails = 0
    for fam, params, K in CASES:
        A = gen.make(fam, *params)
        b, _ = gen.rhs(A)
        bd = torch.from_numpy(b).cuda()
        for ex in EXECS:
            try:
                h = lib.SPCG(A, mode="alg2", K=K, sptrsv=ex, parts=0)
            except lib.SpcgError as e:
                print(f"{fam}{params} {ex}: not applicable ({e})", flush=True)
                continue
            x, si = h.solve(bd, eps=1e-8, kmax=300)
            _, sf = h.solve(bd, eps=0.0, kmax=5)
            r = torch.from_numpy(np.random.default_rng(1).standard_normal(A.n)).cuda()
            y = torch.zeros_like(r)
            z = torch.zeros_like(r)
            w = torch.zeros_like(r)
            h.apply_lower(r, y)
            h.apply_upper(y, z)
            h.apply_spmv(r, w)
            torch.cuda.synchronize()
            ok = si["status"] == 0 and sf["status"] == 0 and bool(torch.isfinite(x).all())
            fails += not ok
            print(f"{fam}{params} {ex} ({h.info['sptrsv_name']}): k={si['iterations']} status={si['status']} "
                  f"forced={sf['status']} {'ok' if ok else 'FAIL'}", flush=True)
            h.close()
    print("FAILED CASES:", fails)
    sys.exit(1 if fails else 0)


if __name__ == "__main__":
    main()
