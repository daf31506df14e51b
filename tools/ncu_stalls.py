#!/usr/bin/env python
"""Per-source-line stall-reason breakdown for a line range (ncu --page source + nvdisasm -gi).
usage: tools/ncu_stalls.py REPORT LIB.so KERNEL_SUBSTR LINE_FROM LINE_TO"""
import csv, io, os, re, subprocess, sys, tempfile, collections
rep, so, kname, lo, hi = sys.argv[1], os.path.abspath(sys.argv[2]), sys.argv[3], int(sys.argv[4]), int(sys.argv[5])
tmp = tempfile.mkdtemp()
subprocess.run(["cuobjdump", "-xelf", "all", so], cwd=tmp, capture_output=True)
line_of = {}
for c in [f for f in os.listdir(tmp) if f.endswith(".cubin")]:
    dis = subprocess.run(["nvdisasm", "-gi", "-c", os.path.join(tmp, c)], capture_output=True, text=True).stdout
    cur_fn, cur, fresh = None, None, True
    for l in dis.splitlines():
        m = re.match(r"\s*\.text\.(\S+):", l)
        if m: cur_fn = m.group(1); continue
        if "//## File" in l:
            m = re.search(r"line (\d+)", l)
            if fresh: cur = int(m.group(1)); fresh = False
            continue
        m = re.match(r"\s*/\*([0-9a-f]{4,})\*/", l)
        if m:
            fresh = True
            if cur_fn and kname in cur_fn: line_of[int(m.group(1), 16)] = cur
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hi_ = next(i for i, r in enumerate(rows) if "Address" in r)
h = rows[hi_]
stall_cols = [i for i, x in enumerate(h) if x.startswith("stall_") and "Not Issued" not in x]
ia = h.index("Address"); iex = h.index("Instructions Executed")
base = None
per = collections.defaultdict(collections.Counter)
execd = collections.Counter()
for r in rows[hi_ + 1:]:
    if len(r) <= max(stall_cols) or not r[ia].startswith("0x"): continue
    a = int(r[ia], 16)
    if base is None: base = a
    ln = line_of.get(a - base)
    if ln is None or not (lo <= ln <= hi): continue
    for i in stall_cols:
        if r[i].isdigit(): per[ln][h[i]] += int(r[i])
    if r[iex].isdigit(): execd[ln] += int(r[iex])
tot = collections.Counter()
for ln in sorted(per):
    t = sum(per[ln].values())
    tot.update(per[ln])
    if t: print(f"L{ln}: {t:6d} samples, {execd[ln]:8d} warp-instrs |", ", ".join(f"{k[6:]}={v}" for k, v in per[ln].most_common(4)))
print("TOTAL", sum(tot.values()), dict(tot.most_common(8)))
