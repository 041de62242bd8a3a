#!/usr/bin/env python3
"""Warp-stall samples per CUDA source line of an ncu report (`--page source --print-source cuda,sass`).
Usage: ncu_lines.py report.ncu-rep [N] [kernel-regex]"""
import csv
import io
import subprocess
import sys

args = ["ncu", "-i", sys.argv[1], "--page", "source", "--csv", "--print-source", "cuda,sass"]
if len(sys.argv) > 3:
    args += ["-k", "regex:" + sys.argv[3]]
N = int(sys.argv[2]) if len(sys.argv) > 2 else 30
out = subprocess.run(args, capture_output=True, text=True).stdout
agg, tot, fname = {}, 0.0, ""


def f(x):
    try:
        return float(x)
    except ValueError:
        return 0.0


for r in csv.reader(io.StringIO(out)):
    if len(r) >= 2 and r[0] == "File Path":
        fname = r[1].split("/")[-1]
    if len(r) < 5 or r[0] in ("", "Line No"):
        continue
    k = (fname, r[0], r[1][:100])
    v = f(r[4])
    agg[k] = agg.get(k, 0) + v
    tot += v
for k, v in sorted(agg.items(), key=lambda x: -x[1])[:N]:
    print(f"{100 * v / max(tot, 1):5.1f}%  {k[0]}:{k[1]:<5} {k[2]}")
