#!/usr/bin/env python
"""One-line summary of a bench.py JSON line read from stdin (tag in argv[1])."""
import json
import sys

d = json.loads(sys.stdin.read())
tag = sys.argv[1] if len(sys.argv) > 1 else ""
cb = d.get("cpu_baseline") or {}
print(tag, "ms/step %.4f" % d["ms_per_step"], "value %.3g" % d["value"], d.get("kernel_ms"),
      "e2e %.4f" % (d.get("e2e") or {}).get("ms_per_step", float("nan")), "parity", cb.get("parity_cut_match"),
      "p50 %.4f" % d["iteration"]["ms_p50"])
