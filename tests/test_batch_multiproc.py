"""C5 batch driver host logic: LPT plan and the multi-process gather (gloo,
world_size 2 and 4, CPU), with host-only setups (device = -1)."""
import os
import socket

import pytest
import torch.multiprocessing as mp

import gen
from paper_conf_sc_maacsh25_b200 import batch


def test_batch_spec_matches_survey():
    S = batch.batch_systems(64)
    fams = [s.family for s in S]
    assert fams[:4] == ["poisson2d", "poisson3d", "fem_q1", "aniso_layered"]
    assert all(s.K == (2 if s.family == "fem_q1" else 0) for s in S)
    # n ~ 2^s with s in [12, 20]
    for s in S:
        dims = s.params[:3] if s.family in ("poisson3d", "fem_q1") else s.params[:2]
        n = 1
        for d in dims:
            n *= d
        assert 2 ** 11 < n < 2 ** 21


def test_lpt_plan_is_balanced_and_complete():
    S = batch.batch_systems(64)
    for world in (1, 2, 4, 8):
        plan, load = batch.lpt_assign(S, world)
        idx = sorted(s.index for p in plan for s in p)
        assert idx == list(range(64))
        # LPT bound: makespan <= 4/3 OPT and <= mean + max job
        mean = sum(load) / world
        assert max(load) <= mean + max(s.cost for s in S) + 1e-9


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    S = [s for s in batch.batch_systems(8) if s.family in ("poisson2d", "aniso_layered")][:4]
    # shrink to CPU-test sizes (same families)
    for s in S:
        s.params = (40 + 3 * s.index, 30) + tuple(s.params[2:])
    plan, _ = batch.lpt_assign(S, world)
    hs = batch.setup_rank(plan[rank], device=-1)
    res = [batch.Result(s.index, s.family, A.n, levels_L=h.info["levels_L"], chosen_pct=h.info["chosen_pct"])
           for s, A, b, h, st in hs]
    allr = batch.gather(res, world)
    if rank == 0:
        q.put([(r.index, r.n, r.levels_L, r.chosen_pct) for r in allr])
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 4])
def test_gather_ranks_gloo(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    # every system appears once, with the levels a single-process setup gives
    assert [o[0] for o in out] == sorted(o[0] for o in out)
    S = [s for s in batch.batch_systems(8) if s.family in ("poisson2d", "aniso_layered")][:4]
    for s, o in zip(sorted(S, key=lambda s: s.index), out):
        A = gen.make(s.family, 40 + 3 * s.index, 30, *s.params[2:])
        import paper_conf_sc_maacsh25_b200 as lib
        h = lib.SPCG(A, K=s.K, device=-1)
        assert o[1] == A.n and o[2] == h.info["levels_L"] and o[3] == h.info["chosen_pct"]


def test_replan_lanes_lpt_by_measured_times():
    """C5 re-planning: systems go, longest measured time first, to the
    least-loaded lane; handles whose lane changes are rebound with set_stream."""
    from types import SimpleNamespace
    from paper_conf_sc_maacsh25_b200 import batch

    class H:
        def __init__(self, lane, stream):
            self.lane, self.stream, self.rebound = lane, stream, 0

        def set_stream(self, st):
            self.stream, self.rebound = st, self.rebound + 1

    streams = [object(), object()]
    ms = {0: 10.0, 1: 9.0, 2: 6.0, 3: 5.0, 4: 1.0}
    handles = [(SimpleNamespace(index=i), None, None, H(0, streams[0]), 0.0) for i in ms]   # all on lane 0
    handles[1][3].lane, handles[1][3].stream = 1, streams[1]
    load = batch.replan_lanes(handles, ms, 2)
    assert sorted(load) == [15.0, 16.0]                       # LPT: {10, 5, 1} / {9, 6}
    lanes = {it[0].index: it[3].lane for it in handles}
    assert lanes[0] == 0 and lanes[1] == 1 and lanes[2] == 1 and lanes[3] == 0 and lanes[4] == 0
    for it in handles:
        assert it[3].stream is streams[it[3].lane]
    assert handles[2][3].rebound == 1 and handles[0][3].rebound == 0
