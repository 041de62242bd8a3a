#!/usr/bin/env python3
"""Top SASS instructions of an ncu report by warp-stall samples (reads `ncu --page source --csv
--print-source sass`). Usage: ncu_hot.py report.ncu-rep [N] [kernel-regex]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
N = int(sys.argv[2]) if len(sys.argv) > 2 else 40
args = ["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"]
if len(sys.argv) > 3:
    args += ["-k", "regex:" + sys.argv[3]]
out = subprocess.run(args, capture_output=True, text=True).stdout
lines = out.splitlines()
# skip the kernel-name header block
start = next(i for i, l in enumerate(lines) if l.startswith('"Address"'))
rows = list(csv.DictReader(io.StringIO("\n".join(lines[start:]))))
stalls = [k for k in rows[0] if k.startswith("stall_") and "Not Issued" not in k]
tot = sum(float(r["Warp Stall Sampling (All Samples)"] or 0) for r in rows)
print(f"total samples {tot:.0f}")
agg = {k: sum(float(r[k] or 0) for r in rows) for k in stalls}
print("by reason:", ", ".join(f"{k[6:]} {100*v/tot:.1f}%" for k, v in sorted(agg.items(), key=lambda x: -x[1])[:10]))
rows.sort(key=lambda r: -float(r["Warp Stall Sampling (All Samples)"] or 0))
for r in rows[:N]:
    s = float(r["Warp Stall Sampling (All Samples)"] or 0)
    top = sorted(((float(r[k] or 0), k[6:]) for k in stalls), reverse=True)[:3]
    print(f"{100*s/tot:5.1f}% {r['Address']:>6} {r['Source'][:70]:70s} " + " ".join(f"{n}:{100*v/max(s,1):.0f}" for v, n in top if v))
