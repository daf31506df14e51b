"""Host logic of the warp-chain executor (no GPU): the inspector's chain layout,
decoded independently here and checked against the factors the library exports
(themselves bit-exact against the oracle in test_setup_parity.py).

Layout (chain_layout.cpp): position pos = 32 * step + lane; chain c
owns steps [chain_step[c], chain_step[c+1]); L walks them ascending, U descending.
A record per step (lane-major, W a power of two): u32 tag[32][W], f64 val[32][W],
(U) f64 1/u_ii[32], then {u32 publish mask, u32 flags}.  Tag kinds: PREV 0 (the
lane of the previous pass step; padding = PREV lane 0 with value 0), HIST 1 (lane,
distance in pass steps), GLOB 2 (position), EXT 3 (position, prefetch ordinal),
EXTS 4 (position).

Checked for every case and both factors:
  * perm is a bijection rows <-> non-padding positions; a step holds rows of one
    wavefront level, steps of a chain are in non-decreasing level (Fig. 1);
  * the entries of each row, resolved to dependency rows through their tags, are
    exactly the row's off-diagonal factor entries in CSR order with the same values;
  * every dependency resolved through a tag is EARLIER in the pass (the chain's own
    previous steps, or another chain); EXT sources are published (mask bit set);
  * a step's flags say SLOW iff it has a non-PREV/PAD entry, EXT iff it has an EXT;
  * U records carry 1/u_ii; the SpMV layout over positions reproduces A row by row.
"""
import numpy as np
import pytest

import gen
import paper_conf_sc_maacsh25_b200 as lib

PREV, HIST, GLOB, EXT, EXTS = 0, 1, 2, 3, 4
CASES = [("poisson2d", (32, 32), 0, "alg2"), ("poisson2d", (70, 37), 0, "none"), ("poisson3d", (13, 11, 9), 0, "alg2"),
         ("poisson3d", (16, 16, 16), 0, "none"), ("aniso_layered", (150, 67, 4), 0, "alg2"),
         ("aniso_layered", (96, 64, 4), 0, "none"), ("fem_q1", (6, 5, 4, 3), 0, "alg2"),
         ("poisson2d", (40, 33), 1, "alg2")]


def _decode(h, A):
    perm = h.export("dbg_chain_perm")
    cstep = h.export("dbg_chain_step")
    recs = {False: h.export("dbg_chain_recl"), True: h.export("dbg_chain_recu")}
    nsteps = int(cstep[-1])
    return perm, cstep, recs, nsteps


@pytest.mark.parametrize("fam,params,K,mode", CASES)
def test_chain_records_cover_factors(fam, params, K, mode):
    A = gen.make(fam, *params)
    h = lib.SPCG(A, mode=mode, K=K, sptrsv="wchain", device=-1)
    assert h.info["sptrsv_name"] == "wchain" and h.info["chains"] >= 1
    perm, cstep, recs, nsteps = _decode(h, A)
    n = A.n
    npos = 32 * nsteps
    assert len(perm) == npos == h.info["positions"]
    rows = perm[perm >= 0]
    assert len(rows) == n and np.array_equal(np.sort(rows), np.arange(n))
    pos_of = np.zeros(n, np.int64)
    pos_of[perm[perm >= 0]] = np.nonzero(perm >= 0)[0]
    chain_of_step = np.zeros(nsteps, np.int64)
    for c in range(len(cstep) - 1):
        chain_of_step[cstep[c]:cstep[c + 1]] = c
    levL = h.export("level_l")
    # grid partitions (chains that depend on each other): steps hold one wavefront level
    # each, non-decreasing inside a chain (deadlock freedom).  Packed components may mix
    # levels of independent components in one step (checked below: every dependency is
    # strictly earlier in its chain's pass).
    for c in range(len(cstep) - 1 if h.info["partition_name"] != "chain-components" else 0):
        last = -1
        for s in range(cstep[c], cstep[c + 1]):
            r = perm[32 * s:32 * s + 32]
            lv = set(int(levL[i]) for i in r if i >= 0)
            assert len(lv) == 1
            lv = lv.pop()
            assert lv >= last
            last = lv
    counts = {}
    for upper in (False, True):
        rp, col, val = (h.export("u_rowptr"), h.export("u_col"), h.export("u_val")) if upper else \
            (h.export("l_rowptr"), h.export("l_col"), h.export("l_val"))
        R = recs[upper]
        rb = len(R) // nsteps
        W = (rb - 16 - (256 if upper else 0)) // 384
        assert rb == 384 * W + 16 + (256 if upper else 0) and W & (W - 1) == 0
        tr = 384 * W + (256 if upper else 0)
        published = np.zeros(npos, bool)
        needs_pub = []
        for s in range(nsteps):
            rec = R[s * rb:(s + 1) * rb]
            tags = np.frombuffer(rec[:128 * W].tobytes(), np.uint32).reshape(32, W).T
            vals = np.frombuffer(rec[128 * W:384 * W].tobytes(), np.float64).reshape(32, W).T
            pub, flags = np.frombuffer(rec[tr:tr + 8].tobytes(), np.uint32)
            for l in range(32):
                if (pub >> l) & 1:
                    published[32 * s + l] = True
            c = chain_of_step[s]
            s0, s1 = int(cstep[c]), int(cstep[c + 1])
            u = (s1 - 1 - s) if upper else (s - s0)          # pass step
            any_slow = any_ext = False
            for l in range(32):
                i = perm[32 * s + l]
                kinds = tags[:, l] >> 29
                if i < 0:
                    assert np.all(tags[:, l] == 0) and np.all(vals[:, l] == 0.0)
                    continue
                q0 = rp[i] + (1 if upper else 0)
                cols, vv = col[q0:rp[i + 1]], val[q0:rp[i + 1]]
                assert len(cols) <= W
                for k in range(W):
                    tg, kind = int(tags[k, l]), int(kinds[k])
                    counts[kind] = counts.get(kind, 0) + 1
                    if k >= len(cols):
                        assert tg == 0 and vals[k, l] == 0.0          # padding: PREV lane 0, value 0
                        continue
                    if kind == PREV:
                        sj = (s + 1) if upper else (s - 1)
                        assert s0 <= sj < s1
                        pj = 32 * sj + (tg & 31)
                    elif kind == HIST:
                        d = (tg >> 5) & 255
                        assert 2 <= d < 32
                        sj = (s + d) if upper else (s - d)
                        assert s0 <= sj < s1
                        pj = 32 * sj + (tg & 31)
                        any_slow = True
                    elif kind == GLOB:
                        pj = tg & 0x1FFFFFFF
                        assert chain_of_step[pj // 32] == c
                        any_slow = True
                    elif kind in (EXT, EXTS):
                        pj = tg & (0x0FFFFFFF if kind == EXT else 0x1FFFFFFF)
                        assert chain_of_step[pj // 32] != c
                        needs_pub.append(pj)
                        any_slow = any_ext = True
                    else:
                        raise AssertionError(f"bad tag kind {kind}")
                    if kind in (PREV, HIST, GLOB):               # own chain: strictly earlier pass step
                        sj = pj // 32
                        uj = (s1 - 1 - sj) if upper else (sj - s0)
                        assert uj < u
                    assert perm[pj] == cols[k], (i, k)
                    assert vals[k, l] == vv[k]
                if upper:
                    dinv = np.frombuffer(rec[384 * W:384 * W + 256].tobytes(), np.float64)
                    assert dinv[l] == 1.0 / val[rp[i]]
            assert bool(flags & 1) == any_slow and bool(flags & 2) == any_ext
        assert all(published[p] for p in needs_pub)
    assert h.info["chain_entries"][0] <= counts.get(PREV, 0)       # PREV tags include the padding
    # SpMV over positions: row perm[p] of A with columns as positions, CSR order
    eoff = h.export("dbg_chain_a_eoff")
    acol = h.export("dbg_chain_a_col")
    aval = h.export("dbg_chain_a_val")
    for s in range(0, nsteps, max(1, nsteps // 50)):
        w = eoff[s + 1] - eoff[s]
        for l in range(32):
            i = perm[32 * s + l]
            es = [(acol[(eoff[s] + k) * 32 + l], aval[(eoff[s] + k) * 32 + l]) for k in range(w)]
            if i < 0:
                assert all(v == 0.0 for _, v in es)
                continue
            lo, hi = A.row_ptr[i], A.row_ptr[i + 1]
            got = [(perm[c], v) for c, v in es[:hi - lo]]
            assert got == list(zip(A.col[lo:hi], A.val[lo:hi]))
            assert all(v == 0.0 for _, v in es[hi - lo:])
    h.close()


def test_chain_partitions_chosen():
    """The inspector's partition on the paper-shaped families: the layered field after
    Algorithm 2 decouples into strips (components: no cross-chain entry at all); the
    unsparsified field and Poisson 2-D take 32-column blocks; 3-D grids line tiles."""
    h = lib.SPCG(gen.make("aniso_layered", 256, 96, 4), mode="alg2", sptrsv="wchain", device=-1)
    assert h.info["partition_name"] == "chain-components" and h.info["chain_entries"][3] == 0
    h = lib.SPCG(gen.make("aniso_layered", 256, 96, 4), mode="none", sptrsv="wchain", device=-1)
    assert h.info["partition_name"] == "chain-grid2d" and h.info["chains"] == 8
    h = lib.SPCG(gen.make("poisson3d", 16, 16, 16), mode="none", sptrsv="wchain", device=-1)
    assert h.info["partition_name"] == "chain-grid3d"
    # a connected system no wider than a warp (Poisson 32 x 32, 32 rows on the longest
    # anti-diagonal; a tridiagonal matrix): one component, one chain
    h = lib.SPCG(gen.make("poisson2d", 32, 32), mode="none", sptrsv="wchain", device=-1)
    assert h.info["partition_name"] == "chain-components" and h.info["chains"] == 1
    with pytest.raises(lib.SpcgError):          # 27-point ILU(2): rows wider than the chain records
        lib.SPCG(gen.make("fem_q1", 8, 8, 8, 3), K=2, sptrsv="wchain", device=-1)
