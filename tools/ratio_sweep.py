"""NEXT-3: ratio sweep and "paper-Oracle" evaluation of Algorithm 2
on the synthetic families, through the C ABI on the GPU.

For every matrix: PCG (t = 0), fixed t in {1, 5, 10} and Algorithm 2's choice are
solved to eps = 1e-8; the paper's "Oracle" is the fastest of the fixed ratios
(Table 1: "Oracle" = the best ratio found by exhaustive search), the
match rate of Algorithm 2 against it is Fig. 7's statistic, and the
wavefront reduction is correlated with the per-iteration speedup (Spearman, the
statistic of §5.2 / Fig. 10).

  python tools/ratio_sweep.py [--out profiles/r02/ratio_sweep.jsonl] [--small]

The pure functions (spearman, paper_oracle, summarize) are tested on the CPU in
tests/test_ratio_study.py; run_sweep is tested on small matrices on the GPU
(iteration counts against the oracle's PCG).
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

MATS = [("poisson2d", (1024, 1024), 0), ("poisson3d", (64, 64, 64), 0), ("fem_q1", (48, 48, 48, 3), 2),
        ("fem_q1", (64, 64, 64, 3), 0), ("aniso_layered", (1024, 1024, 4), 0), ("aniso_layered", (2048, 2048, 4), 0),
        ("aniso_layered", (2048, 2048, 7), 0)]
SMALL = [("poisson2d", (48, 40), 0), ("aniso_layered", (128, 96, 4), 0), ("fem_q1", (10, 9, 8, 3), 2)]
RUNS = [("pcg", dict(mode="none")), ("t1", dict(mode="fixed", fixed_pct=1.0)),
        ("t5", dict(mode="fixed", fixed_pct=5.0)), ("t10", dict(mode="fixed", fixed_pct=10.0)),
        ("alg2", dict(mode="alg2"))]
FIXED = ("t1", "t5", "t10")


def spearman(a, b):
    """Spearman rank correlation (no tie correction: ties are ranked by position)."""
    ra = np.argsort(np.argsort(np.asarray(a, float), kind="stable"), kind="stable").astype(float)
    rb = np.argsort(np.argsort(np.asarray(b, float), kind="stable"), kind="stable").astype(float)
    ra -= ra.mean()
    rb -= rb.mean()
    den = np.sqrt((ra * ra).sum() * (rb * rb).sum())
    return float((ra * rb).sum() / den) if den > 0 else None


def paper_oracle(res):
    """The paper's "Oracle" ratio: the fixed t with the smallest iterative-phase time among
    the runs that converged (status 0); ties go to the smaller t.  None if none did."""
    ok = [t for t in FIXED if t in res and res[t]["status"] == 0]
    if not ok:
        return None
    return min(ok, key=lambda t: (res[t]["ms"], float(t[1:])))


def row_of(name, K, n, res):
    p = res["pcg"]
    o = paper_oracle(res)
    return {"matrix": name, "K": K, "n": n, "runs": res,
            "alg2_pct": res["alg2"]["chosen_pct"],
            "alg2_speedup": p["ms"] / res["alg2"]["ms"],
            "alg2_per_iter_speedup": p["ms_per_iter"] / res["alg2"]["ms_per_iter"],
            "oracle_pct": float(o[1:]) if o else None,
            "oracle_speedup": p["ms"] / res[o]["ms"] if o else None}


def summarize(rows):
    """Fig. 7 / Fig. 10 statistics over the sweep rows."""
    pts = []
    for r in rows:
        res = r["runs"]
        p = res["pcg"]
        for t in FIXED:
            if t in res and res[t]["status"] == 0 and p["levels"] > 0:
                red = (p["levels"] - res[t]["levels"]) / p["levels"]
                pts.append((red, p["ms_per_iter"] / res[t]["ms_per_iter"]))
    sp = [r["alg2_speedup"] for r in rows]
    return {"summary": True,
            "spearman_wavefront_reduction_vs_per_iter_speedup":
                spearman([x for x, _ in pts], [y for _, y in pts]) if len(pts) > 2 else None,
            "points": len(pts),
            "alg2_matches_oracle": sum(1 for r in rows if r["oracle_pct"] is not None and
                                       r["alg2_pct"] == r["oracle_pct"]),
            "matrices": len(rows),
            "alg2_speedup_geomean": float(np.exp(np.mean(np.log(sp)))) if sp else None,
            "paper_context": "P:L56-58 / Table 1: 1.23x (ILU(0)) and 1.65x (ILU(K)) per iteration on A100 fp32; "
                             "Spearman 0.61 between wavefront reduction and speedup (P:L1185-1208)"}


def run_sweep(mats, reps=3, kmax=20000, device=0):
    """Every run of every matrix through the C ABI; returns the rows (plus each run's k,
    for the parity test against the oracle)."""
    import torch

    import gen
    import paper_conf_sc_maacsh25_b200 as spcg
    rows = []
    for fam, params, K in mats:
        A = gen.make(fam, *params)
        b, _ = gen.rhs(A)
        bd = torch.from_numpy(b).cuda(device)
        res = {}
        for tag, kw in RUNS:
            h = spcg.SPCG(A, K=K, device=device, **kw)
            h.solve(bd, eps=1e-8, kmax=kmax)
            ms, k, inf = [], 0, None
            for _ in range(reps):
                _, inf = h.solve(bd, eps=1e-8, kmax=kmax)
                ms.append(inf["iter_phase_ms"])
                k = inf["iterations"]
            res[tag] = {"ms": float(np.median(ms)), "k": k, "ms_per_iter": float(np.median(ms)) / max(k, 1),
                        "levels": h.info["levels_L"], "chosen_pct": h.info["chosen_pct"], "status": inf["status"],
                        "sptrsv": h.info["sptrsv_name"], "partition": h.info["partition_name"]}
            h.close()
        rows.append(row_of(f"{fam}{params}", K, A.n, res))
    return rows


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "ratio_sweep.jsonl"))
    ap.add_argument("--small", action="store_true")
    a = ap.parse_args()
    rows = run_sweep(SMALL if a.small else MATS)
    for r in rows:
        print(json.dumps({k: v for k, v in r.items() if k != "runs"}), flush=True)
    summ = summarize(rows)
    print(json.dumps(summ))
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    with open(a.out, "w") as f:
        for r in rows:
            f.write(json.dumps(r) + "\n")
        f.write(json.dumps(summ) + "\n")


if __name__ == "__main__":
    main()
