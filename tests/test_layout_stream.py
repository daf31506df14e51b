"""Host logic of the chunked executor (no GPU): the record stream the inspector
emits, parsed independently here and checked against the factors the library
exports (themselves bit-exact against the oracle in test_setup_parity.py).

For every partition candidate (forced with spcg_options_t.chunk_partition) and each
section (L, U):
  * every row of the part appears in exactly one FIRST record, every row of the
    matrix in exactly one part;
  * rows come in non-decreasing wavefront level inside a part (the wavefront
    order of Fig. 1);
  * a row's entries over its records are exactly its off-diagonal factor entries:
    cross-CTA entries name the column (-(j+1)) and carry l_ij / u_ij; ring entries
    carry the remaining values (multiset), and the ring slot of a dependency is
    that row's part-local slot;
  * U records carry 1/u_ii of their rows.
Record layout (layout.cpp emit_section): 16-byte header
{u16 w, u16 flags, u8 warp, u8 side, u16 bytes, u32 publish, u32 active}, 32 lane
words {i32 row, u32 len | ne << 8 | publish << 16 | slot << 17}, i32 src[w][32],
f64 val[w][32], f64 1/u_ii[32] (U, last record of a row).
"""

import numpy as np
import pytest

import gen
import paper_conf_sc_maacsh25_b200 as lib

REC_FIRST, REC_LAST, REC_UPPER, REC_EXT, REC_WIDE = 1, 2, 8, 16, 32


def _records(stream, c0, c1, CHUNK):
    for c in range(c0, c1):
        ch = stream[c * CHUNK:(c + 1) * CHUNK]
        nrec = int(np.frombuffer(ch[:2].tobytes(), np.uint16)[0])
        offs = np.frombuffer(ch[8:8 + 2 * nrec].tobytes(), np.uint16)
        for o in offs:
            o = int(o)
            w, fl = np.frombuffer(ch[o:o + 4].tobytes(), np.uint16)
            lanes = np.frombuffer(ch[o + 16:o + 272].tobytes(), np.int32).reshape(32, 2)
            src = np.frombuffer(ch[o + 272:o + 272 + 128 * w].tobytes(), np.int32).reshape(w, 32)
            val = np.frombuffer(ch[o + 272 + 128 * w:o + 272 + 384 * w].tobytes(), np.float64).reshape(w, 32)
            dinv = None
            if (fl & REC_UPPER) and (fl & REC_LAST) and not (fl & REC_WIDE):
                dinv = np.frombuffer(ch[o + 272 + 384 * w:o + 272 + 384 * w + 256].tobytes(), np.float64)
            yield int(w), int(fl), lanes, src, val, dinv


def _csr_rows(rp, col, val, i):
    return col[rp[i]:rp[i + 1]], val[rp[i]:rp[i + 1]]


CASES = [("poisson3d", (16, 16, 16), 0, 8), ("poisson3d", (13, 11, 9), 0, 7), ("aniso_layered", (150, 67, 4), 0, 8),
         ("poisson2d", (40, 33), 0, 5), ("fem_q1", (7, 6, 5, 3), 2, 4)]


@pytest.mark.parametrize("fam,params,K,parts", CASES)
@pytest.mark.parametrize("part", ["contiguous", "strided", "affinity", "components", "tiles"])
def test_record_stream_covers_factors(fam, params, K, parts, part):
    A = gen.make(fam, *params)
    idx = ["contiguous", "strided", "affinity", "components", "tiles"].index(part)
    h = lib.SPCG(A, mode="alg2", K=K, sptrsv="chunked", parts=parts, device=-1, chunk_partition=idx)
    if h.info["partition_name"] != part:
        pytest.skip(f"{part} is not a candidate for {fam}{params}")
    stream = h.export("dbg_stream")
    pch = h.export("dbg_part_chunk")
    puc = h.export("dbg_part_uchunk")
    Lrp, Lcol, Lval = h.export("l_rowptr"), h.export("l_col"), h.export("l_val")
    Urp, Ucol, Uval = h.export("u_rowptr"), h.export("u_col"), h.export("u_val")
    levL, levU = h.export("level_l"), h.export("level_u")
    chunk = len(stream) // int(pch[-1])             # bytes per chunk (a build constant)
    assert chunk % 1024 == 0 and chunk * int(pch[-1]) == len(stream)
    n = A.n
    seen = {"L": np.zeros(n, np.int32), "U": np.zeros(n, np.int32)}
    for c in range(parts):
        for sec, (c0, c1) in (("L", (pch[c], puc[c])), ("U", (puc[c], pch[c + 1]))):
            upper = sec == "U"
            lev = levU if upper else levL
            rp, col, val = (Urp, Ucol, Uval) if upper else (Lrp, Lcol, Lval)
            rows_part, last_level = [], -1
            entries = {}                                    # row -> list of (src, val)
            for w, fl, lanes, src, vv, dinv in _records(stream, c0, c1, chunk):
                assert bool(fl & REC_UPPER) == upper
                for l in range(32):
                    r, meta = int(lanes[l, 0]), int(lanes[l, 1]) & 0xFFFFFFFF
                    if r < 0:
                        continue
                    ln, ne = meta & 0xFF, (meta >> 8) & 0xFF
                    assert ne <= ln <= w
                    if fl & REC_FIRST:
                        seen[sec][r] += 1
                        rows_part.append(r)
                        assert lev[r] >= last_level, "wavefront order inside a part"
                        last_level = lev[r]
                        entries[r] = []
                    for k in range(ln):
                        entries[r].append((int(src[k, l]), float(vv[k, l]), k < ne))
                    if dinv is not None:
                        assert dinv[l] == 1.0 / val[rp[r]]            # U: diagonal first in its row
            part_rows = set(rows_part)
            lidx = {r: i for i, r in enumerate(sorted(part_rows))} if not upper else lidx_L
            if not upper:
                lidx_L = lidx
            slots = []
            for r, es in entries.items():
                cols, vals = _csr_rows(rp, col, val, r)
                off = cols != r
                cols, vals = cols[off], vals[off]
                assert len(es) == len(cols)
                ext = {(-s - 1): v for s, v, is_ext in es if is_ext}
                for j, v in ext.items():                           # cross-CTA: the column itself
                    k = np.nonzero(cols == j)[0]
                    assert len(k) == 1 and vals[k[0]] == v
                # ring entries follow in CSR order: pair them with the remaining columns
                ring_es = [(s, v) for s, v, is_ext in es if not is_ext]
                rest = [(j, v) for j, v in zip(cols, vals) if j not in ext]
                assert [v for _, v in ring_es] == [v for _, v in rest]
                for (s, _), (j, _) in zip(ring_es, rest):
                    assert j in part_rows, "ring dependency inside the part"
                    slots.append((s, lidx[int(j)]))
            # one power-of-two ring size R >= 16 explains every slot: slot = lidx & (R - 1)
            if slots:
                R = 16
                while R < 1 << 20 and not all(s == (li & (R - 1)) for s, li in slots):
                    R <<= 1
                assert all(s == (li & (R - 1)) for s, li in slots)
    assert np.all(seen["L"] == 1) and np.all(seen["U"] == 1)
