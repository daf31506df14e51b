#!/usr/bin/env python
"""Writes oracle/kref.json: the ORACLE's own iteration counts to eps = 1e-8 for the
BASELINE configs C1-C4 (SPCG = Algorithm 2, PCG = no sparsification), from one full
single-thread oracle solve each.  Calls only gen/ (inputs) and oracle/.

bench.py's reference arm (and the cpu_baseline leg) time a bounded forced-k sample
of the oracle per step and project the iterative phase to THIS k (never a guess).
"""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import gen  # noqa: E402
import oracle  # noqa: E402


def main():
    out = {}
    for name in ("C1", "C2", "C3", "C4"):
        A = gen.config_matrix(name)
        b, _ = gen.rhs(A)
        K = gen.CONFIGS[name]["K"]
        out[name] = {}
        for mode in ("alg2", "none"):
            L, U, info = oracle.setup(A, mode=mode, K=K)
            t = time.perf_counter()
            r = oracle.pcg(A, L, U, b, 1e-8, 20000)
            out[name][mode] = dict(k=r["k"], status=r["status"], rnorm=r["rnorm"], chosen_pct=info["chosen_pct"],
                                   seconds=time.perf_counter() - t)
            print(name, mode, out[name][mode], flush=True)
    json.dump(out, open(os.path.join(ROOT, "oracle", "kref.json"), "w"), indent=1)


if __name__ == "__main__":
    main()
