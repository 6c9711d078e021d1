#!/usr/bin/env python3
"""Summarise ncu output into profiles/: launch list shares + per-kernel full-set metrics.

usage: ncu_summary.py <launches.csv> <prof.ncu-rep> <out_prefix> <capture key, e.g. config5/fused>
Writes <out_prefix>_launches.md, <out_prefix>_kernels.md and merges the capture into
profiles/ncu_summary.json under "captures"/<key> (dram bytes per launch per kernel;
bench.py reads the capture of its own workload and round-0 mode for roofline.traffic).
"""
import csv
import io
import json
import os
import subprocess
import sys
from collections import defaultdict


def launches(path):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    h = rows[hi]
    ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
    agg = defaultdict(list)
    for r in rows[hi + 1:]:
        if len(r) <= vi:
            continue
        v = float(r[vi].replace(",", ""))
        u = r[ui]
        v = v / 1e3 if u in ("nsecond", "ns") else v * 1e3 if u in ("msecond", "ms") else v
        name = r[ki].split("(")[0].replace("void ", "").split("<")[0].split("::")[-1]
        agg[name].append(v)
    return agg


def full(rep):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    h, units = rows[0], rows[1]
    want = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
            "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
            "launch__registers_per_thread", "lts__t_sector_hit_rate.pct", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
            "smsp__inst_executed.sum", "launch__grid_size", "launch__block_size"]
    out = defaultdict(list)
    for r in rows[2:]:
        name = r[h.index("Kernel Name")].split("(")[0].replace("void ", "").split("<")[0].split("::")[-1]
        d = {}
        for w in want:
            if w in h:
                i = h.index(w)
                try:
                    v = float(r[i].replace(",", ""))
                except ValueError:
                    continue
                u = units[i]
                scale = {"Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3, "byte": 1, "msecond": 1e-3, "usecond": 1e-6, "ms": 1e-3, "us": 1e-6, "ns": 1e-9, "s": 1.0,
                         "nsecond": 1e-9}.get(u, 1)
                d[w] = v * scale
        out[name].append(d)
    return out


def main():
    lpath, rep, prefix, key = sys.argv[1:5]
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    agg = launches(lpath)
    tot = sum(sum(v) for v in agg.values())
    lines = ["| kernel | launches | total us | mean us | share |", "|---|---|---|---|---|"]
    for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
        lines.append(f"| {k} | {len(v)} | {sum(v):.1f} | {sum(v) / len(v):.1f} | {sum(v) / tot * 100:.1f}% |")
    open(prefix + "_launches.md", "w").write(
        f"# ncu launch list ({os.path.basename(lpath)}; gpu__time_duration.sum, --clock-control none, cold/serialised)\n\n"
        + "\n".join(lines) + "\n")
    k = full(rep)
    lines = ["| kernel | ms | DRAM read GB | DRAM write GB | DRAM % peak | L2 hit % | warps active % | regs | SM % |",
             "|---|---|---|---|---|---|---|---|---|"]
    summ = {}
    for name, ds in k.items():
        d = max(ds, key=lambda x: x.get("gpu__time_duration.sum", 0))   # the kernel's dominant launch
        rb, wb = d.get("dram__bytes_read.sum", 0), d.get("dram__bytes_write.sum", 0)
        lines.append(f"| {name} | {d.get('gpu__time_duration.sum', 0) * 1e3:.3f} | {rb / 1e9:.3f} | {wb / 1e9:.3f} | "
                     f"{d.get('gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed', 0):.1f} | "
                     f"{d.get('lts__t_sector_hit_rate.pct', 0):.1f} | {d.get('sm__warps_active.avg.pct_of_peak_sustained_active', 0):.1f} | "
                     f"{d.get('launch__registers_per_thread', 0):.0f} | {d.get('sm__throughput.avg.pct_of_peak_sustained_elapsed', 0):.1f} |")
        summ[name.split("::")[-1]] = {"dram_bytes_per_launch": rb + wb, "dram_read": rb, "dram_write": wb,
                                      "ms": d.get("gpu__time_duration.sum", 0) * 1e3,
                                      "source": os.path.basename(rep)}
    open(prefix + "_kernels.md", "w").write(
        f"# ncu --set full ({os.path.basename(rep)}; longest captured launch per kernel)\n\n" + "\n".join(lines) + "\n")
    jpath = os.path.join(root, "profiles", "ncu_summary.json")
    try:
        doc = json.load(open(jpath))
    except Exception:
        doc = {}
    caps = doc.get("captures", {})
    caps[key] = {"kernels": summ}
    json.dump({"captures": caps, "note": "ncu --set full --clock-control none; per launch; key = config<k>/<round-0 mode>"},
              open(jpath, "w"), indent=1)
    print(open(prefix + "_launches.md").read())
    print(open(prefix + "_kernels.md").read())


if __name__ == "__main__":
    main()
