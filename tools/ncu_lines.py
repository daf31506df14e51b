#!/usr/bin/env python
"""Map ncu SASS-level stall samples to CUDA source lines via nvdisasm -gi.

usage: tools/ncu_lines.py REPORT.ncu-rep LIB.so KERNEL_SUBSTR [top]
"""
import csv, io, os, re, subprocess, sys, tempfile, collections

rep, so, kname = sys.argv[1], os.path.abspath(sys.argv[2]), sys.argv[3]
top = int(sys.argv[4]) if len(sys.argv) > 4 else 30
tmp = tempfile.mkdtemp()
subprocess.run(["cuobjdump", "-xelf", "all", so], cwd=tmp, capture_output=True)
cub = [f for f in os.listdir(tmp) if f.endswith(".cubin")]
line_of = {}
for c in cub:
    dis = subprocess.run(["nvdisasm", "-gi", "-c", os.path.join(tmp, c)], capture_output=True, text=True).stdout
    cur_fn, cur_line, fresh = None, None, True
    for l in dis.splitlines():
        m = re.match(r"\s*\.text\.(\S+):", l)
        if m:
            cur_fn = m.group(1)
            continue
        m = re.search(r'//## File ".*?([^/"]+)", line (\d+)', l)
        if m:
            if fresh:
                cur_line = f"{m.group(1)}:{m.group(2)}"
                fresh = False
            continue
        m = re.match(r"\s*/\*([0-9a-f]{4,})\*/", l)
        if m:
            fresh = True
            if cur_fn and kname in cur_fn:
                line_of[int(m.group(1), 16)] = cur_line
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hi = next(i for i, r in enumerate(rows) if "Address" in r)
h = rows[hi]
ia, iw, isrc = h.index("Address"), h.index("Warp Stall Sampling (All Samples)"), h.index("Source")
base = None
agg = collections.Counter()
srcl = {}
for r in rows[hi + 1:]:
    if len(r) <= iw or not r[ia].startswith("0x"):
        continue
    a = int(r[ia], 16)
    if base is None:
        base = a
    n = int(r[iw]) if r[iw].isdigit() else 0
    if os.environ.get("DBG") and n: print(hex(a - base), n, r[isrc][:40])
    ln = line_of.get(a - base, "?")
    agg[ln] += n
tot = sum(agg.values()) or 1
src = {}
for f in set(k.split(":")[0] for k in agg if ":" in k):
    for root, _, files in os.walk(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))):
        if f in files:
            src[f] = open(os.path.join(root, f)).read().splitlines()
            break
for ln, n in agg.most_common(top):
    text = ""
    if ":" in ln:
        f, k = ln.split(":")
        if f in src and int(k) - 1 < len(src[f]):
            text = src[f][int(k) - 1].strip()
    print(f"{100 * n / tot:5.1f}%  {ln:18s} {text[:100]}")
