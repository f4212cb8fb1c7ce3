#!/usr/bin/env python
"""Build an A/B variant of libigk.so with extra compile definitions into
paper_conf_dac_leejlczcshh25_b200/ab/libigk_<tag>.so (load it with IGK_LIB=...).
Usage: python tools/build_ab.py <tag> -DNAME=VALUE ..."""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_dac_leejlczcshh25_b200 import build as b  # noqa: E402

tag, defs = sys.argv[1], sys.argv[2:]
out_dir = os.path.join(b.HERE, "ab")
os.makedirs(out_dir, exist_ok=True)
so = os.path.join(out_dir, f"libigk_{tag}.so")
cmd = [b.NVCC, *b.FLAGS, *defs, *[os.path.join(b.HERE, s) for s in b.SRCS], "-o", so]
r = subprocess.run(cmd, capture_output=True, text=True)
if r.returncode != 0:
    sys.exit("nvcc failed:\n" + r.stdout + r.stderr)
for line in r.stderr.splitlines():
    if "registers" in line or "spill" in line:
        pass
print(so)
