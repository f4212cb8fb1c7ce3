#!/usr/bin/env python
"""Per-CUDA-source-line totals from
`ncu -i X.ncu-rep --page source --csv --print-source cuda,sass > X.csv`
(a metric column, default L2 theoretical sectors, plus stall samples), top N.
Usage: python tools/ncu_lines.py X.csv [N] [metric]"""
import csv
import sys
from collections import defaultdict

path = sys.argv[1]
N = int(sys.argv[2]) if len(sys.argv) > 2 else 25
metric = sys.argv[3] if len(sys.argv) > 3 else "L2 Theoretical Sectors Global"
agg = defaultdict(lambda: [0.0, 0.0, ""])
f = hdr = line = None
src = ""
for r in csv.reader(open(path)):
    if not r:
        continue
    if r[0] == "File Path":
        f = r[1].split("/")[-1]
        continue
    if r[0] == "Line No":
        hdr = r
        continue
    if r[0] == "Function Name" or hdr is None:
        continue
    if r[0]:
        line, src = r[0], r[1]
    if len(r) < len(hdr):
        continue
    d = dict(zip(hdr[2:], r[2:]))
    try:
        m = float((d.get(metric) or "0").replace(",", ""))
        smp = float((d.get("Warp Stall Sampling (All Samples)") or "0").replace(",", ""))
    except ValueError:
        continue
    a = agg[(f, line)]
    a[0] += m
    a[1] += smp
    a[2] = src
tot_m = sum(v[0] for v in agg.values()) or 1
tot_s = sum(v[1] for v in agg.values()) or 1
print(f"{'file:line':24s} {metric[:18]:>18s} {'%':>6s} {'samples%':>8s}  source")
for (f, l), (m, s, src) in sorted(agg.items(), key=lambda kv: -kv[1][0])[:N]:
    print(f"{f + ':' + str(l):24s} {m:18.0f} {m / tot_m:6.1%} {s / tot_s:8.1%}  {src.strip()[:90]}")
print("-- by stall samples")
for (f, l), (m, s, src) in sorted(agg.items(), key=lambda kv: -kv[1][1])[:N]:
    print(f"{f + ':' + str(l):24s} {m:18.0f} {m / tot_m:6.1%} {s / tot_s:8.1%}  {src.strip()[:90]}")
