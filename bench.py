#!/usr/bin/env python
"""bench.py — SPCG iterative phase on B200 (BASELINE.json metric).

Metric: "SPCG iter-phase ms to eps=1e-8 + HBM GB/s per iter vs unsparsified PCG".
A *step* is one full pass of the hot path: one solve of Algorithm 1 (prologue +
iterations to ||r|| < 1e-8) on the workload, inputs resident in HBM.  The
default workload at N = 1 is the largest single-GPU config of BASELINE.json,
C4 (2-D layered anisotropic diffusion 4096^2, n = 16.8 M, ILU(0); SPCG =
Algorithm 2 vs PCG = no sparsification, plus the fixed-t sweep t in {1,5,10}),
where the working set (4.2 GB per iteration) is far beyond L2 and the HBM
roofline applies.  C1-C3 stay selectable (--workload).  At N > 1 the default is
the C5 batch (64 independent systems, LPT over the ranks: strong scaling).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--workload C4] [--sptrsv auto]
  python bench.py --impl reference ...      # the oracle (plain fp64 C, host cores)

N > 1 with C1-C4 (torchrun): every rank solves its own replica (a single system
does not shard: DESIGN.md §7), no collective on the data path; times are max
over ranks.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import gen  # noqa: E402  (seeded inputs; no method arithmetic)

EPS = 1e-8
KMAX = 10000
PAPER_CONTEXT = {"paper_iter_speedup_ilu0_a100_fp32": 1.23, "paper_iter_speedup_iluk_a100_fp32": 1.65,
                 "paper_e2e_speedup_ilu0_a100_fp32": 1.68, "paper_e2e_speedup_iluk_a100_fp32": 3.73}
WORKLOADS = {
    "C1": "C1: 2D 5-point Poisson 32x32 (n=1024), ILU(0)",
    "C2": "C2: 3D 7-point Poisson 64^3 (n=262144), ILU(0)",
    "C3": "C3: 3D 27-point Q1 FEM 128^3 (n=2097152), ILU(2)",
    "C4": "C4: 2D layered anisotropic diffusion 4096^2 (n=16777216), ILU(0)",
    "C5": "C5: batch of 64 independent mixed SPD systems (Poisson 2D/3D, FEM ILU(2), layered), LPT over GPUs",
}


def _dist():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


def _peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, burst copy)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def _ncu_traffic(workload: str, impl: str, iterations: int):
    """DRAM bytes (read + write) of the persistent kernel per launch of THIS bench's solve:
    the committed ncu capture's bytes per iteration (launch bytes / (k_capture + 1 for the
    prologue)) x (iterations + 1)."""
    p = os.path.join(ROOT, "profiles", "ncu_summary.json")
    if not os.path.exists(p):
        return None
    try:
        d = json.load(open(p))
        e = d.get(workload, {}).get(impl)
        if e is None:
            return None
        per = float(e.get("dram_bytes_per_iter", e["dram_bytes_per_launch"]))
        return per * (iterations + 1) if "dram_bytes_per_iter" in e else per
    except Exception:
        return None


class Clocks:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md clocks line)."""

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.path = f"/tmp/spcg_clocks_{os.getpid()}.csv"

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), "--query-gpu=clocks.sm,clocks.max.sm,power.draw,"
                 "clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
                 "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
                 "clocks_event_reasons.sw_power_cap", "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=open(self.path, "w"), stderr=subprocess.DEVNULL)
            time.sleep(0.3)
        except Exception:
            self.proc = None
        return self

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            self.proc.wait()

    def summary(self):
        try:
            rows = [l.split(", ") for l in open(self.path).read().strip().splitlines() if l.strip()]
        except Exception:
            return None
        if not rows:
            return None
        sm = [float(r[0]) for r in rows if r[0].replace(".", "").isdigit()]
        mx = max(float(r[1]) for r in rows)
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[k] for r in rows for k in range(4) if len(r) > 4 + k and r[4 + k].strip() == "Active"})
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": mx, "reasons": reasons,
                "samples": len(rows)}


def _cpu_info():
    model = ""
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                model = line.split(":", 1)[1].strip()
                break
    except Exception:
        pass
    return model


def _kref():
    """The oracle's own iteration counts to eps (oracle/kref.json, written by
    tools/oracle_kref.py from one full single-thread oracle solve per config/mode)."""
    p = os.path.join(ROOT, "oracle", "kref.json")
    return json.load(open(p)) if os.path.exists(p) else {}


def _smt():
    try:
        return open("/sys/devices/system/cpu/smt/active").read().strip() == "1"
    except Exception:
        return None


def run_oracle(name: str, A, b, steps: int, warmup: int, budget_s: float = 20.0, multicore: bool = False,
               modes=("alg2", "none")):
    """The oracle's iterative phase (Alg. 1 from the prologue to loop exit, A19), as it
    stands, timed on the host: single thread (spcg_oracle.c) or, multicore=True, the
    OpenMP build of the same solve phase on all cores (spcg_oracle_omp.c).

    Each of warmup + steps steps is a full solve to eps when that fits the per-step
    share of budget_s; otherwise a bounded forced-k sample (eps = 0, k_s iterations,
    same code) whose time is projected to the oracle's OWN k to eps (oracle/kref.json,
    one full oracle solve per config and mode) as t_s / (k_s + 1) x (k + 1)."""
    import oracle
    c = gen.CONFIGS[name]
    kref = _kref().get(name, {})
    res = {}
    per_step = budget_s / len(modes) / max(steps + warmup, 1)
    for mode in modes:
        L, U, info = oracle.setup(A, mode=mode, K=c["K"])
        if multicore:
            run = lambda e, km: oracle.pcg_omp(A, L, U, b, e, km)   # noqa: E731
        else:
            run = lambda e, km: oracle.pcg(A, L, U, b, e, km)       # noqa: E731
        probe = run(0.0, 2)
        per_it = probe["seconds"] / 3.0
        threads = probe.get("threads", 1)
        k = kref.get(mode, {}).get("k")
        full = k is None or per_it * (k + 1) <= per_step
        times, ks, k_s = [], [], 0
        for sidx in range(steps + warmup):
            if full:
                r = run(EPS, KMAX)
                t, kk = r["seconds"] * 1e3, r["k"]
            else:
                k_s = max(2, int(per_step / per_it) - 1)
                r = run(0.0, k_s)
                t, kk = r["seconds"] * 1e3 / (k_s + 1) * (k + 1), k
            if sidx >= warmup:
                times.append(t)
                ks.append(kk)
        sample = (f"{len(times)} full solve(s) to eps" if full else
                  f"{len(times)} forced-k sample(s) of {k_s} iterations (+ prologue) each, projected to the "
                  f"oracle's own k = {k} (oracle/kref.json)")
        res[mode] = dict(ms=float(np.mean(times)), k=int(ks[-1]), samples=len(times), projected=not full,
                         chosen_pct=info["chosen_pct"], sample=sample, threads=threads)
    return res


def _cpu_line(name: str, o: dict, cores: int, kind_note: str) -> dict:
    return {"value": o["alg2"]["ms"], "unit": "ms", "cores": cores, "kind": "oracle",
            "sample": f"{name} iterative phase: {o['alg2']['sample']}, {kind_note}, {_cpu_info()}, "
                      f"nproc {os.cpu_count()}, SMT {'on' if _smt() else 'off' if _smt() is False else '?'}; "
                      f"PCG {o['none']['ms']:.1f} ms ({o['none']['sample']})",
            "pcg_value": o["none"]["ms"], "iterations": o["alg2"]["k"], "pcg_iterations": o["none"]["k"],
            "per_iter_speedup_spcg_vs_pcg": (o["none"]["ms"] / max(o["none"]["k"] + 1, 1)) /
                                            (o["alg2"]["ms"] / max(o["alg2"]["k"] + 1, 1))}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--workload", default=None, choices=sorted(WORKLOADS),
                    help="default: C4 at N = 1, C5 at N > 1")
    ap.add_argument("--impl", default="spcg", choices=["spcg", "reference"])
    ap.add_argument("--sptrsv", default="auto")
    ap.add_argument("--parts", type=int, default=0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-host-setup", action="store_true", help="skip timing the host setup beside the GPU one")
    ap.add_argument("--no-f32", action="store_true", help="skip the fp32-factor (NEXT-2) leg of C4")
    ap.add_argument("--no-multi-rhs", action="store_true", help="skip the multi-RHS (NEXT-4) leg of C4")
    ap.add_argument("--batch-count", type=int, default=64)
    ap.add_argument("--lanes", type=int, default=4,
                    help="C5: concurrent streams per GPU (each with SMs/lanes persistent CTAs)")
    ap.add_argument("--sched", default="static", choices=["static", "dynamic"],
                    help="C5 lanes: static LPT lanes, all enqueued up front (default), or host list scheduling")
    ap.add_argument("--sweep", default=None,
                    help="comma list of fixed drop ratios t%% timed beside Alg. 2 and PCG (default: 1,5,10 for C4)")
    args = ap.parse_args()
    ws, rank, local = _dist()
    name = args.workload or ("C4" if ws == 1 else "C5")
    args.workload = name
    if name == "C5":
        return run_batch(args, ws, rank, local)
    A = gen.config_matrix(name)
    b, _ = gen.rhs(A)
    K = gen.CONFIGS[name]["K"]

    if args.impl == "reference":
        if rank != 0:
            return
        o = run_oracle(name, A, b, args.steps, args.warmup, budget_s=150.0)
        v = o["alg2"]["ms"]
        cpu = _cpu_line(name, o, 1, "single thread (the oracle as it stands)")
        line = {"metric": "SPCG iter-phase ms to eps=1e-8 + HBM GB/s per iter vs unsparsified PCG",
                "impl": "reference", "value": v, "unit": "ms", "n_gpus": args.gpus, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": v, "higher_is_better": False, "scaling": "weak",
                "vs_baseline": None, "dtype": "f64", "data": "synthetic",
                "config": {"workload": WORKLOADS[name], "n": A.n, "nnz": A.nnz, "K": K, "eps": EPS},
                "iterations": o["alg2"]["k"], "pcg": {"value": o["none"]["ms"], "iterations": o["none"]["k"]},
                "cpu_baseline": cpu,
                "e2e": {"value": v, "unit": "ms", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
        print(json.dumps(line))
        return

    import torch
    import paper_conf_sc_maacsh25_b200 as spcg

    if ws > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl" if torch.cuda.is_available() else "gloo")
    dev = local if torch.cuda.is_available() else 0
    torch.cuda.set_device(dev)
    stream = torch.cuda.current_stream(dev)

    # bring the GPU out of its idle clocks before anything is timed (the setup timings are
    # reported too): ~0.5 s of streaming work
    warm = torch.empty(64 * 1024 * 1024, dtype=torch.float32, device=f"cuda:{dev}")
    t_w = time.perf_counter()
    while time.perf_counter() - t_w < 0.5:
        warm.mul_(1.0)
        torch.cuda.synchronize(dev)
    del warm
    # NEXT-1: ILU(0) systems are set up on the GPU (validation, Algorithm 2, ILU(0), level
    # sets: gsetup.cu); the host setup of the same products is timed once for comparison
    setup_kind = "gpu" if K == 0 and A.n >= 65536 else "host"     # tiny systems: the host is quicker
    handles = {}
    for mode in ("alg2", "none"):
        handles[mode] = spcg.SPCG(A, mode=mode, K=K, sptrsv=args.sptrsv, parts=args.parts, device=dev, stream=stream,
                                  setup=setup_kind)
    host_setup_ms = None
    if K == 0 and not args.no_host_setup:
        hh = spcg.SPCG(A, mode="alg2", K=K, sptrsv=args.sptrsv, parts=args.parts, device=dev, stream=stream,
                       setup="host")
        host_setup_ms = hh.info["setup_ms_total"]
        hh.close()
    bd = torch.from_numpy(b).to(f"cuda:{dev}")
    xd = torch.empty_like(bd)
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device=f"cuda:{dev}")

    def barrier():
        torch.cuda.synchronize(dev)
        if ws > 1:
            torch.distributed.barrier()
            torch.cuda.synchronize(dev)

    results = {}
    clk = Clocks(dev)
    with clk:
        for mode in ("alg2", "none"):
            h = handles[mode]
            for _ in range(args.warmup):
                flush.zero_()
                h.solve(bd, xd, EPS, KMAX)
            barrier()
            ms, ks = [], []
            t0 = time.perf_counter()
            for _ in range(args.steps):
                flush.zero_()                       # L2 flush between steps (256 MiB > 126 MB L2)
                _, info = h.solve(bd, xd, EPS, KMAX)
                assert info["status"] == 0, info
                ms.append(info["iter_phase_ms"])
                ks.append(info["iterations"])
            barrier()
            wall = (time.perf_counter() - t0) * 1e3
            # e2e through the public API with HOST buffers (H2D b, solve, D2H x inside the call)
            e2e = []
            bh = torch.from_numpy(b).pin_memory()
            xh = torch.empty_like(bh).pin_memory()
            for _ in range(max(3, args.steps // 2)):
                flush.zero_()
                torch.cuda.synchronize(dev)
                te = time.perf_counter()
                h.solve_host(bh, EPS, KMAX, out=xh)
                e2e.append((time.perf_counter() - te) * 1e3)
            results[mode] = dict(ms=float(np.mean(ms)), ms_max=float(np.max(ms)), k=int(ks[-1]), wall=wall,
                                 e2e=float(np.mean(e2e)), info=h.info)
    clocks = clk.summary()
    calib = spcg.calibrate(dev)
    # C4 sparsification sweep, fixed t beside Alg. 2's choice and PCG (t = 0)
    sweep_spec = args.sweep if args.sweep is not None else ("1,5,10" if name == "C4" else "")
    sweep = []
    for t in [float(v) for v in sweep_spec.split(",") if v.strip()]:
        hs = spcg.SPCG(A, mode="fixed", fixed_pct=t, K=K, sptrsv=args.sptrsv, parts=args.parts, device=dev,
                       stream=stream, setup=setup_kind)
        hs.solve(bd, xd, EPS, KMAX)
        tms, tk = [], 0
        for _ in range(max(1, min(args.steps, 3))):
            flush.zero_()
            _, inf = hs.solve(bd, xd, EPS, KMAX)
            tms.append(inf["iter_phase_ms"])
            tk = inf["iterations"]
        sweep.append({"t_pct": t, "ms": float(np.mean(tms)), "iterations": tk, "ms_per_iter": float(np.mean(tms)) / max(tk, 1),
                      "levels_L": hs.info["levels_L"], "m_t": hs.info["m_t"], "status": inf["status"],
                      "partition": hs.info["partition_name"],
                      "hbm_gbs_per_iter": hs.info["algo_bytes_per_iter"] * tk / (float(np.mean(tms)) * 1e-3) / 1e9})
        hs.close()

    # NEXT-2: fp32 factors with fp64 vectors (the paper's preconditioner precision,
    # P:L827-828) on the same workload: M = fl32(L) fl32(U), 4-byte record values
    f32 = None
    if name == "C4" and not args.no_f32:
        hf = spcg.SPCG(A, mode="alg2", K=K, sptrsv=args.sptrsv, parts=args.parts, device=dev, stream=stream,
                       setup=setup_kind, factors="f32")
        hf.solve(bd, xd, EPS, KMAX)
        fms, fk = [], 0
        for _ in range(max(1, min(args.steps, 3))):
            flush.zero_()
            _, inf = hf.solve(bd, xd, EPS, KMAX)
            fms.append(inf["iter_phase_ms"])
            fk = inf["iterations"]
        fb = hf.info["algo_bytes_per_iter"]
        f32 = {"ms": float(np.mean(fms)), "iterations": fk, "ms_per_iter": float(np.mean(fms)) / max(fk, 1),
               "algo_bytes_per_iter": fb, "record_value_bytes": hf.info["record_value_bytes"],
               "hbm_gbs_per_iter": fb * fk / (float(np.mean(fms)) * 1e-3) / 1e9, "status": inf["status"]}
        hf.close()

    # NEXT-4: four right-hand sides of the same system in one launch (spcg_solve_multi):
    # the matrix and factor streams are read once for all four
    mrhs = None
    if name == "C4" and not args.no_multi_rhs:
        try:
            Bh = np.stack([gen.rhs(A, seed=sd)[0] for sd in (99, 100, 101, 102)])
            Bd = torch.from_numpy(Bh).to(f"cuda:{dev}")
            h = handles["alg2"]
            h.solve_multi(Bd, eps=EPS, kmax=KMAX)
            mms, mk = [], None
            for _ in range(max(1, min(args.steps, 3))):
                flush.zero_()
                _, infs = h.solve_multi(Bd, eps=EPS, kmax=KMAX)
                mms.append(infs[0]["iter_phase_ms"])
                mk = [i["iterations"] for i in infs]
                assert all(i["status"] == 0 for i in infs), infs
            mt = float(np.mean(mms))
            mrhs = {"nrhs": 4, "ms": mt, "iterations": mk, "ms_per_rhs": mt / 4,
                    "rhs_per_s": 4 / (mt * 1e-3), "single_rhs_ms": results["alg2"]["ms"],
                    "throughput_vs_single": results["alg2"]["ms"] / (mt / 4),
                    "ms_per_iter_all_rhs": mt / max(max(mk), 1),
                    "note": "NEXT-4: 4 independent CGs, matrix/factor streams shared; right-hand sides "
                            "b_j = A x_j with x_j from seeds 99..102"}
        except Exception as e:        # a layout the multi-RHS kernel does not cover
            mrhs = {"unavailable": str(e)[:200]}

    def mx(v):
        if ws == 1:
            return v
        t = torch.tensor([v], dtype=torch.float64, device=f"cuda:{dev}")
        torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
        return float(t.item())

    s, p = results["alg2"], results["none"]
    s_ms, p_ms = mx(s["ms"]), mx(p["ms"])
    s_e2e = mx(s["e2e"])
    if rank != 0:
        torch.distributed.destroy_process_group()
        return
    peak, peak_src = _peaks()
    si, pi = s["info"], p["info"]
    s_bi, p_bi = si["algo_bytes_per_iter"], pi["algo_bytes_per_iter"]
    s_gbs = s_bi * s["k"] / (s_ms * 1e-3) / 1e9
    p_gbs = p_bi * p["k"] / (p_ms * 1e-3) / 1e9
    traffic = _ncu_traffic(name, "spcg", s["k"])
    l2_hit = None
    try:
        l2_hit = json.load(open(os.path.join(ROOT, "profiles", "ncu_summary.json")))[name]["spcg"].get("l2_hit_pct")
    except Exception:
        pass
    l2_resident = s_bi < 100e6
    cpu = cpu_mc = None
    if not args.no_cpu_baseline:
        o = run_oracle(name, A, b, 1, 0, budget_s=24.0)
        cpu = _cpu_line(name, o, 1, "single thread (the oracle as it stands)")
        om = run_oracle(name, A, b, 1, 0, budget_s=24.0, multicore=True)
        cpu_mc = _cpu_line(name, om, om["alg2"]["threads"], "OpenMP level-scheduled solve phase on all host cores "
                                                            "(oracle/spcg_oracle_omp.c)")
    line = {
        "metric": "SPCG iter-phase ms to eps=1e-8 + HBM GB/s per iter vs unsparsified PCG",
        "value": s_ms, "unit": "ms", "n_gpus": ws, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": s_ms, "higher_is_better": False, "scaling": "weak", "vs_baseline": None,
        "dtype": "f64", "data": "synthetic",
        "config": {"workload": WORKLOADS[name], "n": A.n, "nnz": A.nnz, "K": K, "eps": EPS,
                   "drop": "Algorithm 2 (tau=1, omega=10%, ratios 10/5/1)", "chosen_pct": si["chosen_pct"],
                   "sptrsv": si["sptrsv_name"], "ctas": si["parts"], "partition": si["partition_name"],
                   "l2": "flushed between steps (256 MiB write); timed region = the solve kernel only",
                   "replicas": ws},
        "iterations": s["k"], "ms_per_iter": s_ms / max(s["k"], 1),
        "hbm_gbs_per_iter": s_gbs, "algo_bytes_per_iter": s_bi,
        "levels": {"L": si["levels_L"], "U": si["levels_U"], "w_A": si["w_A"], "w_Ahat": si["w_Ahat"]},
        "nnz": {"A": si["nnz_A"], "Ahat": si["nnz_Ahat"], "L_s": si["nnz_L"], "U": si["nnz_U"]},
        "ncu_dram_gbs": None if traffic is None else traffic / (s_ms * 1e-3) / 1e9,
        "pcg": {"value": p_ms, "iterations": p["k"], "ms_per_iter": p_ms / max(p["k"], 1), "hbm_gbs_per_iter": p_gbs,
                "algo_bytes_per_iter": p_bi, "levels": {"L": pi["levels_L"], "U": pi["levels_U"]}},
        "sweep": sweep or None,
        "multi_rhs": mrhs,
        "fp32_factors": None if f32 is None else dict(f32, frac=f32["hbm_gbs_per_iter"] / peak,
                                                       note="NEXT-2: M = fl32(L) fl32(U) applied in fp64"),
        "spcg_vs_pcg": {"iter_phase_speedup": p_ms / s_ms,
                        "per_iter_speedup": (p_ms / max(p["k"], 1)) / (s_ms / max(s["k"], 1))},
        "paper_context": PAPER_CONTEXT,
        "roofline": {"bound": "hbm", "achieved": s_gbs, "peak": peak, "unit": "GB/s", "frac": s_gbs / peak,
                     "traffic": traffic,
                     "kernel": ("spcg_resident_kernel (one CTA, whole Alg. 1)" if si["sptrsv_name"] == "resident"
                                else "spcg_pcg_kernel (persistent, whole Alg. 1)"),
                     "peak_source": peak_src,
                     "achieved_def": "B_iter (DESIGN.md §4) x iterations / CUDA-event time of the launch",
                     "l2_hit_pct": l2_hit, "l2_resident": l2_resident,
                     "note": ("working set L2-resident (B_iter < 126 MB L2; ncu DRAM traffic << algorithmic): "
                              "frac is algorithmic bytes over the HBM peak, not an HBM utilisation"
                              if l2_resident else "working set >> L2: algorithmic bytes over the measured HBM peak")},
        "cpu_baseline": cpu,
        "cpu_baseline_multicore": cpu_mc,
        "chain_floor": chain_floor(calib, si, s_bi, peak, s_ms / max(s["k"], 1)),
        "e2e": {"value": s_e2e, "unit": "ms", "h2d_bytes_per_step": 8 * A.n, "d2h_bytes_per_step": 8 * A.n,
                "path": "spcg_solve with SPCG_HOST_PTRS (pinned host b, x; H2D + solve + D2H inside the call, wall clock)"},
        "gpu_launches": args.steps,
        "clocks": clocks,
        "setup_ms": {k: si[k] for k in si if k.startswith("setup_ms")},
        # NEXT-1 / §4.3: end to end = setup (on the GPU for ILU(0)) + iterative phase
        "end_to_end": {
            "setup": setup_kind,
            "spcg_setup_ms": si["setup_ms_total"], "pcg_setup_ms": pi["setup_ms_total"],
            "spcg_host_setup_ms": host_setup_ms,
            "spcg_ms": si["setup_ms_total"] + s_ms, "pcg_ms": pi["setup_ms_total"] + p_ms,
            "speedup_spcg_vs_pcg": (pi["setup_ms_total"] + p_ms) / (si["setup_ms_total"] + s_ms),
            "paper_context": "1.68x (ILU(0)) / 3.73x (ILU(K)) end to end, A100 fp32 (P:L56-58)"},
    }
    print(json.dumps(line))
    if ws > 1:
        torch.distributed.destroy_process_group()


def chain_floor(calib: dict, info: dict, bytes_per_iter: float, peak_gbs: float, ms_per_iter: float) -> dict:
    """chain floor = (levels_L + levels_U) x handoff cost, beside the HBM floor.
    Handoffs measured by spcg_calibrate on this box; the executor's own is named."""
    lv = info["levels_L"] + info["levels_U"]
    per = {"grid_sync": calib["grid_sync_ns"], "graph_kernel": calib["graph_kernel_ns"],
           "flag_same_die": calib["flag_same_die_ns"], "flag_cross_die": calib["flag_cross_die_ns"],
           "ll_flag_same_die": calib["flag_relaxed_same_die_ns"], "ll_flag_cross_die": calib["flag_relaxed_cross_die_ns"],
           "syncthreads": calib["syncthreads_ns"], "cluster_sync": calib["cluster_sync_ns"]}
    floors = {k: lv * v * 1e-3 for k, v in per.items()}              # us per iteration
    own = {"level": "grid_sync", "syncfree": "ll_flag_same_die", "chunked": "ll_flag_same_die"}.get(
        info["sptrsv_name"], "ll_flag_same_die")
    hbm_us = bytes_per_iter / (peak_gbs * 1e9) * 1e6
    return {"levels": lv, "handoff_ns": per, "floor_us_per_iter": floors, "executor_handoff": own,
            "chain_floor_us_per_iter": floors[own], "hbm_floor_us_per_iter": hbm_us,
            "binds": "chain" if floors[own] > hbm_us else "hbm", "measured_us_per_iter": ms_per_iter * 1e3,
            "note": "chunked: per-wavefront dependencies inside a CTA go through shared memory; cross-CTA ones "
                    "through flags (pipelined), so its true floor lies between the syncthreads and flag rows"}


def batch_cpu_baseline(systems, results, budget_s: float = 20.0):
    """The oracle (single thread) on a bounded sample of C5: the systems in index order
    until ~budget_s of CPU work, each solved to eps; the batch figure is projected by
    the GPU iteration counts and the oracle's measured time per iteration per row."""
    import oracle
    t_used, rates, done = 0.0, {}, []
    for s in systems:
        if t_used > budget_s:
            break
        A = gen.make(s.family, *s.params)
        if A.n > 300000:
            continue
        b, _ = gen.rhs(A)
        L, U, _ = oracle.setup(A, mode="alg2", K=s.K)
        r = oracle.pcg(A, L, U, b, EPS, 20000)
        t_used += r["seconds"]
        rates.setdefault(s.family, []).append(r["seconds"] / max(r["k"] + 1, 1) / A.nnz)
        done.append(s.index)
    if not rates:
        return None
    # s per (iteration x stored entry of A), per family (ILU(2) factors cost more per entry of A)
    fam_rate = {f: float(np.median(v)) for f, v in rates.items()}
    any_rate = float(np.median([x for v in rates.values() for x in v]))
    fam = {s.index: s.family for s in systems}
    nnz = {s.index: gen.make(s.family, *s.params).nnz for s in systems}
    proj = sum(fam_rate.get(fam[r.index], any_rate) * (r.iterations + 1) * nnz[r.index] for r in results) * 1e3
    return {"value": proj, "unit": "ms", "cores": 1, "kind": "oracle",
            "sample": f"{len(done)} of {len(systems)} systems solved to eps by the oracle ({t_used:.1f} s); the "
                      f"batch is projected with the median s per (iteration x nnz(A)) and the GPU iteration "
                      f"counts, single thread, {_cpu_info()}"}


def run_batch(args, ws, rank, local):
    """C5: independent systems spread over the ranks by LPT; no collective on the data path.

    A step = every system of the rank solved once (device time of each solve summed:
    the systems run back to back on the rank's GPU); value = max over ranks (makespan)."""
    import torch
    import paper_conf_sc_maacsh25_b200 as spcg
    from paper_conf_sc_maacsh25_b200 import batch
    if ws > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl")
    torch.cuda.set_device(local)
    systems = batch.batch_systems(args.batch_count)
    plan, load = batch.lpt_assign(systems, ws)
    sms = torch.cuda.get_device_properties(local).multi_processor_count
    hs = batch.setup_rank(plan[rank], device=local, lanes=args.lanes, sms=sms)

    def timed(hs_):
        order = {}

        def step():
            if args.lanes > 1 and args.sched == "dynamic":
                r, mk = batch.solve_rank_dynamic(hs_, args.lanes, order=order or None)
                order.update({x.index: x.iter_phase_ms for x in r})      # longest first next time
                return r, mk
            if args.lanes > 1:
                return batch.solve_rank_concurrent(hs_)
            r = batch.solve_rank(hs_)
            return r, sum(x.iter_phase_ms for x in r)

        last = None
        for _ in range(max(1, args.warmup)):
            last = step()
        if args.lanes > 1 and args.sched == "static":
            # static lanes re-planned by LPT over the warm-up step's measured per-system times
            batch.replan_lanes(hs_, {x.index: x.iter_phase_ms for x in last[0]}, args.lanes)
            step()
        t_dev_ = []
        res_ = None
        for _ in range(args.steps):
            torch.cuda.synchronize()
            if ws > 1:
                torch.distributed.barrier()
            res_, mk = step()
            t_dev_.append(mk)
        return res_, t_dev_

    clk = Clocks(local)
    with clk:
        res, t_dev = timed(hs)
    # the unsparsified PCG on the same batch (metric: "... vs unsparsified PCG")
    hs_pcg = batch.setup_rank(plan[rank], device=local, mode="none", lanes=args.lanes, sms=sms)
    res_pcg, t_pcg = timed(hs_pcg)
    ms_pcg = float(np.mean(t_pcg))
    pcg_bytes = sum(h.info["algo_bytes_per_iter"] * r.iterations for (_, _, _, h, _), r in zip(hs_pcg, res_pcg))
    for it in hs_pcg:
        it[3].close()
    ms = float(np.mean(t_dev))
    # e2e through the public API with host buffers (H2D b, solve, D2H x inside each call)
    te = time.perf_counter()
    e2e_res = batch.solve_rank(hs, host=True)
    e2e_ms = (time.perf_counter() - te) * 1e3
    h2d = sum(8 * r.n for r in e2e_res)
    bytes_rank = sum(h.info["algo_bytes_per_iter"] * r.iterations for (_, _, _, h, _), r in zip(hs, res))
    allr = batch.gather(res, ws)
    if ws > 1:
        t = torch.tensor([ms, e2e_ms, ms_pcg], dtype=torch.float64, device=f"cuda:{local}")
        torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
        ms, e2e_ms, ms_pcg = float(t[0].item()), float(t[1].item()), float(t[2].item())
        b = torch.tensor([bytes_rank, pcg_bytes], dtype=torch.float64, device=f"cuda:{local}")
        torch.distributed.all_reduce(b)
        bytes_rank, pcg_bytes = float(b[0].item()), float(b[1].item())
    allp = batch.gather(res_pcg, ws)
    if rank == 0:
        peak, peak_src = _peaks()
        gbs = bytes_rank / (ms * 1e-3) / 1e9
        # LPT makespans at g = 1, 2, 4, 8 from the MEASURED per-system times (projection, labelled)
        meas = {r.index: r.iter_phase_ms for r in allr}
        proj = {}
        for g in (1, 2, 4, 8):
            for s in systems:
                s.cost = meas[s.index]
            _, ld = batch.lpt_assign(systems, g)
            proj[str(g)] = max(ld)
        line = {"metric": "SPCG iter-phase ms to eps=1e-8 + HBM GB/s per iter vs unsparsified PCG",
                "value": ms, "unit": "ms", "n_gpus": ws, "steps": args.steps, "warmup": args.warmup,
                "ms_per_step": ms, "higher_is_better": False, "scaling": "strong", "vs_baseline": None,
                "dtype": "f64", "data": "synthetic",
                "config": {"workload": WORKLOADS["C5"], "systems": len(systems), "eps": EPS, "lanes": args.lanes,
                           "makespan": (f"device events fork/join around the rank's solves ({args.sched} lanes: "
                                        f"{args.lanes} streams x {sms // args.lanes} CTAs"
                                        + ("; lanes re-planned by LPT over the warm-up step's measured per-system times)"
                                           if args.sched == "static" else ")") if args.lanes > 1 else
                                        "sum of the rank's device-timed solves (back to back)") +
                                       "; max over ranks",
                           "l2": "no flush: 64 different systems run back to back (working set >> L2)"},
                "systems_per_s": len(systems) / (ms * 1e-3),
                "pcg": {"value": ms_pcg, "unit": "ms", "hbm_gbs": pcg_bytes / (ms_pcg * 1e-3) / 1e9,
                        "iterations_total": sum(r.iterations for r in allp),
                        "note": "the same batch, same lanes and schedule, Ahat = A (no sparsification)"},
                "spcg_vs_pcg": {"makespan_speedup": ms_pcg / ms},
                "roofline": {"bound": "hbm", "achieved": gbs, "peak": peak, "unit": "GB/s", "frac": gbs / peak,
                             "traffic": None, "kernel": "spcg_pcg_kernel (one launch per system)",
                             "peak_source": peak_src,
                             "achieved_def": "sum over systems of B_iter x iterations / makespan"},
                "cpu_baseline": None if args.no_cpu_baseline else batch_cpu_baseline(systems, allr),
                "e2e": {"value": e2e_ms, "unit": "ms", "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": h2d,
                        "path": "spcg_solve with SPCG_HOST_PTRS per system (wall clock of the rank's loop)"},
                "gpu_launches": len(systems) * args.steps,
                "clocks": clk.summary(),
                "lpt_makespan_ms_projected": proj,
                "lpt_projection_note": "LPT over the measured per-system solve times (concurrent lanes: each "
                                       "system's own event time); the largest system bounds the 8-GPU makespan",
                "largest_system_ms": max(meas.values()),
                # the largest system alone bounds the 8-GPU makespan, so strong scaling
                # cannot beat T_N / (8 max_i T_i) with T_N this run's makespan at N GPUs
                "efficiency_bound_8gpu": (ms * ws) / (8.0 * max(meas.values())),
                "per_system": [[r.index, r.family, r.n, r.iterations, round(r.iter_phase_ms, 3), r.chosen_pct,
                                r.status] for r in allr],
                "lpt_load_balance": max(load) / (sum(load) / ws)}
        print(json.dumps(line))
    if ws > 1:
        torch.distributed.destroy_process_group()


if __name__ == "__main__":
    main()
