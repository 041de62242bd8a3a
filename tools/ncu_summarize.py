#!/usr/bin/env python
"""Summarize an `ncu --set full` report (.ncu-rep) into a small JSON + markdown block for profiles/.

  python tools/ncu_summarize.py gpurun_out/prof_C2.ncu-rep --config C2 --rows 100000000 \
      --bytes-per-row 36 --out profiles/ncu_C2_summary.json

The JSON carries `dram_bytes_per_launch` (dram__bytes_read.sum + dram__bytes_write.sum) and
`rows_per_launch`, which bench.py reads for the roofline `traffic` field.
"""
import argparse
import csv
import json
import subprocess
import sys


def ncu_csv(rep, page, extra=()):
    out = subprocess.run(["ncu", "-i", rep, "--page", page, "--csv", *extra], capture_output=True, text=True).stdout
    return list(csv.reader(out.splitlines()))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("rep")
    ap.add_argument("--config", required=True)
    ap.add_argument("--rows", type=int, required=True)
    ap.add_argument("--bytes-per-row", type=int, required=True)
    ap.add_argument("--out", required=True)
    ap.add_argument("--note", default="")
    a = ap.parse_args()
    raw = ncu_csv(a.rep, "raw")
    hdr, units, vals = raw[0], raw[1], raw[2]
    d = dict(zip(hdr, vals))
    u = dict(zip(hdr, units))

    def num(k):
        v = d.get(k, "")
        try:
            x = float(v.replace(",", ""))
        except ValueError:
            return None
        unit = u.get(k, "")
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12, "ns": 1e-9, "us": 1e-6,
                 "ms": 1e-3, "s": 1.0, "usecond": 1e-6, "msecond": 1e-3, "nsecond": 1e-9}.get(unit, 1)
        return x * scale

    dur = num("gpu__time_duration.sum")
    rd, wr = num("dram__bytes_read.sum"), num("dram__bytes_write.sum")
    stalls = {k.replace("smsp__pcsamp_warps_issue_stalled_", ""): float(v) for k, v in d.items()
              if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued") and v not in ("", "0")}
    tot = sum(stalls.values()) or 1
    top = sorted(stalls.items(), key=lambda kv: -kv[1])[:6]
    alg = a.rows * a.bytes_per_row
    summary = {
        "config": a.config, "kernel": d.get("Kernel Name", ""), "report": a.rep,
        "rows_per_launch": a.rows, "bytes_per_row": a.bytes_per_row, "algorithmic_bytes": alg,
        "duration_s": dur, "dram_bytes_read": rd, "dram_bytes_write": wr,
        "dram_bytes_per_launch": (rd or 0) + (wr or 0),
        "traffic_over_algorithmic": ((rd or 0) + (wr or 0)) / alg if alg else None,
        "algorithmic_gbs": alg / dur / 1e9 if dur else None,
        "dram_throughput_pct": num("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed"),
        "l2_hit_rate_pct": num("lts__t_sector_hit_rate.pct"),
        "registers_per_thread": num("launch__registers_per_thread"),
        "achieved_occupancy_pct": num("sm__warps_active.avg.pct_of_peak_sustained_active"),
        "shared_atom_inst": num("smsp__inst_executed_op_shared_atom.sum"),
        "shared_atom_bank_conflicts": num("l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_atom.sum"),
        "global_red_inst": num("smsp__inst_executed_op_global_red.sum"),
        "inst_executed": num("smsp__inst_executed.sum"),
        "lsu_data_pipe_pct": num("l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed"),
        "shared_wavefronts": num("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum"),
        "shared_ld_wavefronts": num("l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum"),
        "shared_atom_wavefronts": num("l1tex__data_pipe_lsu_wavefronts_mem_shared_op_atom.sum"),
        "global_ld_sectors": num("l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum"),
        "top_stalls_pct": {k: round(100 * v / tot, 1) for k, v in top},
        "sm_clock_hz": num("gpc__cycles_elapsed.avg.per_second"),
        "note": a.note,
    }
    json.dump(summary, open(a.out, "w"), indent=1)
    print(json.dumps(summary, indent=1))


if __name__ == "__main__":
    sys.exit(main())
