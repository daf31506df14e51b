#!/usr/bin/env python
"""Summarise an ncu report (--set full) and a launch list into profiles/.

usage: tools/ncu_summary.py REPORT.ncu-rep|RAW.csv LAUNCHES.csv OUT.md --workload C2 --impl spcg [--json profiles/ncu_summary.json]
"""
import argparse, csv, io, json, os, subprocess, sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_bytes.sum",
        "lts__t_sector_hit_rate.pct", "l1tex__t_sector_hit_rate.pct", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size", "sm__cycles_elapsed.avg.per_second"]
UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}


def raw(rep):
    """REPORT.ncu-rep, or the CSV of its raw page (`ncu -i REP --page raw --csv`)."""
    if rep.endswith(".csv"):
        out = open(rep).read()
    else:
        out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    out = "".join(l + "\n" for l in out.splitlines() if not l.startswith("=="))
    rows = list(csv.reader(io.StringIO(out)))
    return rows[0], rows[1], rows[2:]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("rep"); ap.add_argument("launches"); ap.add_argument("out")
    ap.add_argument("--workload", default="C2"); ap.add_argument("--impl", default="spcg")
    ap.add_argument("--json", default="profiles/ncu_summary.json")
    ap.add_argument("--note", default="")
    ap.add_argument("--iterations", type=int, default=0,
                    help="forced-k iterations of the captured launch (per-iteration DRAM bytes = launch / (k + 1))")
    a = ap.parse_args()
    h, units, data = raw(a.rep)
    lines = [f"# ncu summary — {a.workload} ({a.impl})", "", a.note, "", f"report: `{os.path.basename(a.rep)}` (ncu --set full --clock-control none)", ""]
    per = []
    for v in data:
        d = {}
        for k in KEYS:
            if k in h:
                i = h.index(k)
                d[k] = (v[i], units[i])
        per.append(d)
        lines.append("| metric | value | unit |\n|---|---|---|")
        for k, (val, u) in d.items():
            lines.append(f"| {k} | {val} | {u} |")
        stalls = [(h[i], float(v[i])) for i in range(len(h)) if h[i].startswith("smsp__pcsamp_warps_issue_stalled_")
                  and not h[i].endswith("not_issued") and v[i].replace('.', '').isdigit()]
        stalls.sort(key=lambda x: -x[1])
        tot = sum(s for _, s in stalls) or 1
        lines.append("\nTop stall reasons (pc sampling):\n")
        for n, s in stalls[:6]:
            lines.append(f"- {n.replace('smsp__pcsamp_warps_issue_stalled_', '')}: {100 * s / tot:.1f}%")
        lines.append("")
    # launch list
    txt = "".join(l for l in open(a.launches) if not l.startswith("=="))
    rows = list(csv.reader(io.StringIO(txt)))
    hh = rows[0]
    ki, vi, ui = hh.index("Kernel Name"), hh.index("Metric Value"), hh.index("Metric Unit")
    tot = {}
    for r in rows[1:]:
        name = r[ki].split("(")[0][:80]
        val = float(r[vi].replace(",", ""))
        scale = {"nsecond": 1e-6, "usecond": 1e-3, "msecond": 1.0, "second": 1e3}.get(r[ui], 1e-6)
        tot.setdefault(name, [0, 0.0])
        tot[name][0] += 1
        tot[name][1] += val * scale
    allms = sum(v[1] for v in tot.values())
    lines.append(f"## launch list (`{os.path.basename(a.launches)}`, gpu__time_duration, serialised, cold cache)\n")
    lines.append("| kernel | launches | total ms | share |\n|---|---|---|---|")
    for k, (c, ms) in sorted(tot.items(), key=lambda x: -x[1][1]):
        lines.append(f"| `{k}` | {c} | {ms:.3f} | {100 * ms / allms:.1f}% |")
    open(a.out, "w").write("\n".join(lines) + "\n")
    # json for bench.py roofline.traffic
    d = per[0]
    rd = float(d["dram__bytes_read.sum"][0]) * UNIT.get(d["dram__bytes_read.sum"][1], 1)
    wr = float(d["dram__bytes_write.sum"][0]) * UNIT.get(d["dram__bytes_write.sum"][1], 1)
    js = json.load(open(a.json)) if os.path.exists(a.json) else {}
    e = {"dram_bytes_per_launch": rd + wr, "report": os.path.basename(a.rep), "summary": os.path.basename(a.out)}
    if a.iterations > 0:
        e["iterations_in_launch"] = a.iterations
        e["dram_bytes_per_iter"] = (rd + wr) / (a.iterations + 1)
    if "lts__t_sector_hit_rate.pct" in d:
        e["l2_hit_pct"] = float(d["lts__t_sector_hit_rate.pct"][0])
    js.setdefault(a.workload, {})[a.impl] = e
    json.dump(js, open(a.json, "w"), indent=1)
    print(open(a.out).read())


if __name__ == "__main__":
    main()
