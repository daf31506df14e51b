"""Multi-GPU batch of independent systems.

A single system does not shard (the triangular-solve chain is serial across
wavefronts), so multi-GPU use is data-parallel over *independent systems*: the
batch is split across ranks by LPT (longest processing time first) on a cost
estimate, every rank sets up and solves its own systems on its own GPU, and the
only communication is a host-side gather of the per-system results (no
collective on the solve path).  Launch one process per GPU (torchrun); ranks use
``torch.distributed`` only for the final gather and the timing barrier.
"""
from __future__ import annotations

import math
import time
from dataclasses import dataclass, field

import numpy as np

import gen

from . import SPCG


@dataclass
class System:
    index: int
    family: str
    params: tuple
    K: int
    cost: float = 0.0


def batch_systems(count: int = 64):
    """C5: system i of the seeded mixed batch."""
    out = []
    for i in range(count):
        s = gen.batch_spec(i)
        out.append(System(i, s["family"], tuple(s["params"]), s["K"]))
    return out


def estimate_cost(s: System) -> float:
    """Relative solve cost ~ bytes per iteration x expected iterations.

    Rows from the grid sides; stored entries per row by stencil (x ~2.5 for
    ILU(2) fill); iterations ~ grid side (CG on Laplacian-like systems)."""
    dims = [p for p in s.params if isinstance(p, (int, np.integer))][: 3 if s.family in ("poisson3d", "fem_q1") else 2]
    n = float(np.prod(dims))
    per_row = {"poisson2d": 5, "aniso_layered": 5, "poisson3d": 7, "fem_q1": 27}[s.family]
    fill = 2.5 if s.K >= 2 else 1.0
    side = max(dims)
    return n * (12.0 * per_row * (1.0 + fill) + 120.0) * side


def lpt_assign(systems, world: int):
    """Longest-processing-time-first: each system (largest cost first) goes to the
    currently least-loaded rank.  Deterministic (ties: lowest rank, then index)."""
    for s in systems:
        if s.cost == 0.0:
            s.cost = estimate_cost(s)
    order = sorted(systems, key=lambda s: (-s.cost, s.index))
    load = [0.0] * world
    plan = [[] for _ in range(world)]
    for s in order:
        r = min(range(world), key=lambda k: (load[k], k))
        plan[r].append(s)
        load[r] += s.cost
    for p in plan:
        p.sort(key=lambda s: s.index)
    return plan, load


@dataclass
class Result:
    index: int
    family: str
    n: int
    iterations: int = 0
    iter_phase_ms: float = 0.0
    rnorm: float = 0.0
    status: int = 0
    chosen_pct: float = 0.0
    levels_L: int = 0
    x_checksum: float = 0.0
    setup_s: float = 0.0


def setup_rank(systems, device: int, mode: str = "alg2", lanes: int = 1, sms: int = 148, **kw):
    """Host setup (+ upload when device >= 0) of this rank's systems.

    lanes > 1: the GPU is split into `lanes` concurrent streams of sms // lanes CTAs
    each (one persistent CTA per SM, so the cooperative solves in flight always fit
    the device together); systems go to lanes by LPT on their cost estimate."""
    handles = []
    lane_of = {}
    streams = None
    if lanes > 1 and device >= 0:
        import torch
        streams = [torch.cuda.Stream(device) for _ in range(lanes)]
        for s in systems:
            if s.cost == 0.0:
                s.cost = estimate_cost(s)
        plan, _ = lpt_assign(list(systems), lanes)
        for li, part in enumerate(plan):
            for s in part:
                lane_of[s.index] = li
    for s in systems:
        A = gen.make(s.family, *s.params)
        b, _ = gen.rhs(A)
        t0 = time.perf_counter()
        extra = dict(kw)
        if streams is not None:
            extra["stream"] = streams[lane_of[s.index]]
            # narrow systems: one CTA up to 4096 rows (resident), 16 up to 16384 (chunked,
            # DESIGN.md §5); larger ones and wide ILU(K) rows (sync-free) take the lane's CTAs
            lane_ctas = max(1, sms // lanes)
            if A.n <= 16384 and s.K == 0:
                extra["parts"] = 1 if A.n <= 4096 else min(16, lane_ctas)
            else:
                extra["parts"] = lane_ctas
        if device >= 0 and s.K == 0:
            extra.setdefault("setup", "gpu")      # NEXT-1: ILU(0) setups on the GPU
        h = SPCG(A, mode=mode, K=s.K, device=device, **extra)
        h.lane = lane_of.get(s.index, 0)
        handles.append((s, A, b, h, time.perf_counter() - t0))
    return handles


def solve_rank_dynamic(handles, lanes: int, eps: float = 1e-8, kmax: int = 20000, order=None):
    """List scheduling over `lanes` concurrent streams: the systems, longest first
    (`order`: expected solve ms per system index, e.g. the previous step's), go to
    whichever lane frees up first (spcg_set_stream + spcg_solve_async; lane
    completion seen through an event query).  Every handle was set up with
    sms // lanes CTAs, so the cooperative solves in flight always fit the GPU
    together.  Returns (results, device makespan ms from fork/join events)."""
    import torch
    dev = handles[0][3].device
    main = torch.cuda.current_stream(dev)
    streams = [torch.cuda.Stream(dev) for _ in range(lanes)]
    bufs = {}
    for s, A, b, h, st in handles:       # inputs resident before the timed region
        bd = torch.from_numpy(b).to(f"cuda:{dev}")
        bufs[s.index] = (bd, torch.empty_like(bd))
    torch.cuda.synchronize(dev)
    for s, A, b, h, st in handles:
        h.set_stream(streams[0])
    key = (lambda it: -order[it[0].index]) if order else (lambda it: -(it[0].cost or estimate_cost(it[0])))
    queue = sorted(handles, key=key)
    t0 = torch.cuda.Event(enable_timing=True)
    t1 = torch.cuda.Event(enable_timing=True)
    t0.record(main)
    for st_ in streams:
        st_.wait_event(t0)
    running = {}
    out = []

    def launch(item, lane):
        s, A, b, h, st = item
        h.set_stream(streams[lane])
        bd, xd = bufs[s.index]
        h.solve_async(bd, xd, eps=eps, kmax=kmax)
        ev = torch.cuda.Event()
        ev.record(streams[lane])
        running[lane] = (item, ev)

    for lane in range(min(lanes, len(queue))):
        launch(queue.pop(0), lane)
    while running:
        done = [lane for lane, (_, ev) in running.items() if ev.query()]
        if not done:
            time.sleep(2e-5)
            continue
        for lane in done:
            (s, A, b, h, st), _ = running.pop(lane)
            info = h.solve_wait()
            out.append(Result(s.index, s.family, A.n, info["iterations"], info["iter_phase_ms"], info["rnorm"],
                              info["status"], h.info["chosen_pct"], h.info["levels_L"],
                              float(bufs[s.index][1].double().sum().item()), st))
            if queue:
                launch(queue.pop(0), lane)
    for st_ in streams:
        e = torch.cuda.Event()
        e.record(st_)
        main.wait_event(e)
    t1.record(main)
    t1.synchronize()
    return sorted(out, key=lambda r: r.index), float(t0.elapsed_time(t1))


def replan_lanes(handles, measured_ms, lanes: int):
    """LPT of this rank's systems over its lanes by MEASURED solve times (SURVEY
    §8(e): the cost estimates refined by the measured per-system times, here those
    of a warm-up step).  Handles are rebound with spcg_set_stream (device-side
    ordering, the host does not block).  Returns the per-lane load (ms)."""
    by_lane = {}
    for item in handles:
        by_lane.setdefault(item[3].lane, item[3].stream)
    streams = [by_lane[k] for k in sorted(by_lane)]
    load = [0.0] * len(streams)
    for it in sorted(handles, key=lambda it: (-measured_ms[it[0].index], it[0].index)):
        k = min(range(len(streams)), key=lambda j: (load[j], j))
        load[k] += measured_ms[it[0].index]
        h = it[3]
        if h.stream is not streams[k]:
            h.set_stream(streams[k])
        h.lane = k
    return load


def solve_rank_concurrent(handles, eps: float = 1e-8, kmax: int = 20000):
    """All of this rank's systems in flight at once, one stream per lane
    (spcg_solve_async / spcg_solve_wait).  Returns (results, device makespan ms):
    events on the default stream fork to every lane and join after the last solve."""
    import torch
    dev = handles[0][3].device
    main = torch.cuda.current_stream(dev)
    lanes = {}
    for item in handles:
        lanes.setdefault(id(item[3].stream), item[3].stream)
    bufs = []
    for s, A, b, h, st in handles:       # inputs resident before the timed region
        with torch.cuda.stream(h.stream):
            bd = torch.from_numpy(b).to(f"cuda:{dev}", non_blocking=False)
            bufs.append((bd, torch.empty_like(bd)))
    torch.cuda.synchronize(dev)
    t0 = torch.cuda.Event(enable_timing=True)
    t1 = torch.cuda.Event(enable_timing=True)
    t0.record(main)
    for st_ in lanes.values():
        st_.wait_event(t0)
    for (s, A, b, h, st), (bd, xd) in zip(handles, bufs):
        h.solve_async(bd, xd, eps=eps, kmax=kmax)
    for st_ in lanes.values():
        e = torch.cuda.Event()
        e.record(st_)
        main.wait_event(e)
    t1.record(main)
    out = []
    for (s, A, b, h, st), (bd, xd) in zip(handles, bufs):
        info = h.solve_wait()
        out.append(Result(s.index, s.family, A.n, info["iterations"], info["iter_phase_ms"], info["rnorm"],
                          info["status"], h.info["chosen_pct"], h.info["levels_L"],
                          float(xd.double().sum().item()), st))
    t1.synchronize()
    return out, float(t0.elapsed_time(t1))


def solve_rank(handles, eps: float = 1e-8, kmax: int = 20000, host: bool = False):
    """Solve this rank's systems on its GPU; returns per-system results.
    host=True: the public host-pointer path (H2D of b and D2H of x inside each call)."""
    import torch
    out = []
    for s, A, b, h, st in handles:
        if host:
            xh, info = h.solve_host(b, eps=eps, kmax=kmax)
            out.append(Result(s.index, s.family, A.n, info["iterations"], info["iter_phase_ms"], info["rnorm"],
                              info["status"], h.info["chosen_pct"], h.info["levels_L"], float(np.sum(xh)), st))
            continue
        bd = torch.from_numpy(b).to(f"cuda:{h.device}")
        x, info = h.solve(bd, eps=eps, kmax=kmax)
        out.append(Result(s.index, s.family, A.n, info["iterations"], info["iter_phase_ms"], info["rnorm"],
                          info["status"], h.info["chosen_pct"], h.info["levels_L"],
                          float(x.double().sum().item()), st))
    return out


def gather(results, world: int):
    """Host-side gather of every rank's results onto all ranks (gloo or nccl)."""
    if world == 1:
        return sorted(results, key=lambda r: r.index)
    import torch.distributed as dist
    allr = [None] * world
    dist.all_gather_object(allr, results)
    return sorted([r for part in allr for r in part], key=lambda r: r.index)
