#!/usr/bin/env python
"""Summarise ncu outputs for profiles/: a launch list CSV (gpu__time_duration)
and/or a --set full report (.ncu-rep) -> a short text file."""
import csv
import subprocess
import sys
from collections import defaultdict

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_bytes.sum",
        "launch__grid_size", "launch__block_size", "launch__registers_per_thread",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
        "gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed"]


def launches(path):
    rows = list(csv.reader(open(path)))
    h = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    H = rows[h]
    ki, vi = H.index("Kernel Name"), H.index("Metric Value")
    agg = defaultdict(list)
    for r in rows[h + 1:]:
        if len(r) > vi and r[vi]:
            agg[r[ki].split("(")[0]].append(float(r[vi].replace(",", "")) / 1e3)
    tot = sum(sum(v) for v in agg.values())
    out = [f"launch list: {path}", f"{'kernel':60s} {'n':>4s} {'mean_us':>10s} {'total_us':>10s} {'share':>6s}"]
    for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
        out.append(f"{k[:60]:60s} {len(v):4d} {sum(v)/len(v):10.1f} {sum(v):10.1f} {sum(v)/tot:6.1%}")
    return out


def full(path):
    raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(raw.splitlines()))
    H, U = rows[0], rows[1]
    out = [f"ncu --set full: {path}"]
    for r in rows[2:]:
        name = r[H.index("Kernel Name")] if "Kernel Name" in H else "?"
        out.append(f"kernel {name.split('(')[0]}")
        for k in KEYS:
            if k in H:
                out.append(f"  {k} = {r[H.index(k)]} {U[H.index(k)]}")
        st = [(float(r[i].replace(",", "")), H[i]) for i in range(len(H))
              if "average_warps_issue_stalled" in H[i] and H[i].endswith("per_issue_active.ratio") and r[i] not in ("", "n/a")]
        st.sort(reverse=True)
        out.append("  top stall reasons (warps per issue): " +
                   ", ".join(f"{n.split('stalled_')[1].split('_per')[0]}={v:.1f}" for v, n in st[:6]))
    return out


if __name__ == "__main__":
    lines = []
    for p in sys.argv[1:]:
        lines += launches(p) if p.endswith(".csv") else full(p)
        lines.append("")
    print("\n".join(lines))
