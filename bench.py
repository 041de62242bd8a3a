#!/usr/bin/env python
"""bench.py — GROUP BY throughput of libblugby on B200 (BASELINE.json metric).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config C2] [--impl blugby|reference]

One "step" is one whole GROUP BY of one batch of synthetic fact-table rows (SURVEY.md §8(a) S0-S8:
init, aggregate, CTA merge, compaction, the host read of n_groups; plus the NCCL merge at N > 1).
The default workload is BASELINE.json configs[1] = C2 (100M rows, 2 i32 dictionary keys, 4 value
columns, COUNT/SUM/MIN/MAX/AVG, path (a)). At N > 1 every rank aggregates its own 100M rows (weak
scaling) and the dense states are combined with NCCL all-reduces.

Timing: inputs generated in HBM before timing; between steps L2 is flushed (a 512 MB memset, outside
the per-step CUDA events); each step is bracketed by CUDA events on the launching stream; K steps are
bracketed by a barrier + synchronize; the max over ranks is reported. `--impl reference` times the
CPU oracle (oracle/, plain single-threaded std::map) on a bounded sample of the same workload.
"""
import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "GROUP BY rows/s and HBM GB/s (% of B200 peak) at 1/2/4/8 GPUs vs CPU oracle"
PEAKS_FALLBACK = {"hbm_gbs": 6650.0}  # B200_PROFILING.md fallback (used only if MEASURED_PEAKS.json is absent)


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy read+write)"
    return PEAKS_FALLBACK["hbm_gbs"], "fallback (B200_PROFILING.md)"


def load_traffic(config, phase=None):
    """Per-launch DRAM traffic (read + write bytes) of the aggregation kernel (or of one phase of the
    partitioned path) from the committed ncu --set full summary (profiles/), or None."""
    p = os.path.join(ROOT, "profiles", f"ncu_{config}_{phase + '_' if phase else ''}summary.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return d.get("dram_bytes_per_launch"), d.get("rows_per_launch")
    return None, None


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled DURING the timed region (B200_PROFILING.md)."""

    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.proc = None
        self.lines = []

    def start(self):
        if self.index < 0:
            return
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                                          "-i", str(self.index), "-lms", "50"], stdout=subprocess.PIPE,
                                         stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.06)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=2)
        except Exception:
            self.proc.kill()
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [x.strip() for x in ln.split(",")]
            if len(parts) < 6:
                continue
            try:
                sm.append(float(parts[0]))
                mx.append(float(parts[1]))
            except ValueError:
                continue
            for n, v in zip(names, parts[2:6]):
                if v.lower() == "active":
                    reasons.add(n)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm)}


def workload_for(config, rank, world):
    import blugen
    w = blugen.workload(config)
    return w


def result_bytes(res):
    n = 0
    for t in list(res.keys) + list(res.aggs or []):
        n += t.numel() * t.element_size()
    return n


# ----------------------------------------------------------------------------------------------
# CPU oracle leg (cpu_baseline and --impl reference)
# ----------------------------------------------------------------------------------------------
def oracle_rate(config, rows, row0=0):
    import blugen
    import oracle
    w = blugen.workload(config)
    t0 = time.perf_counter()
    o = oracle.groupby_generated(w, row0=row0, n=rows)
    dt = time.perf_counter() - t0
    return rows / dt, dt, o.n_groups


def cpu_baseline(config, seconds=10.0):
    """The oracle as it stands, single-threaded, on a bounded sample (first rows of the workload)."""
    r, dt, _ = oracle_rate(config, 200_000)
    rows = int(min(max(r * seconds, 200_000), 10**9))
    rows = min(rows, 50_000_000 if config in ("C1", "C2") else rows)
    rate, dt, ng = oracle_rate(config, rows)
    return {"value": rate, "unit": "rows/s", "cores": 1, "kind": "oracle",
            "sample": f"{config} rows [0, {rows}) ({dt:.1f} s, {ng} groups), plain single-threaded std::map, "
                      f"host {os.cpu_count()} cores visible"}


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import blugen
    w = blugen.workload(args.config)
    r0, _, _ = oracle_rate(args.config, 100_000)
    budget = float(os.environ.get("BLU_BENCH_REF_BUDGET_S", "90"))
    rows = int(max(50_000, min(10_000_000, r0 * budget / max(1, args.steps + args.warmup))))
    for i in range(args.warmup):
        oracle_rate(args.config, rows, row0=i * rows)
    times = []
    for i in range(args.steps):
        _, dt, _ = oracle_rate(args.config, rows, row0=(args.warmup + i) * rows % max(1, w.n_rows - rows))
        times.append(dt)
    tot = sum(times)
    value = rows * args.steps / tot
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": "rows/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1000 * tot / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "int64+f64",
            "data": "synthetic",
            "config": {"workload": f"{args.config}: {w.note}", "rows_per_step": rows, "full_rows": w.n_rows},
            "cpu_baseline": {"value": value, "unit": "rows/s", "cores": 1, "kind": "oracle",
                             "sample": f"{rows} rows per step of {args.config}, single-threaded std::map oracle"},
            "e2e": {"value": value, "unit": "rows/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


# ----------------------------------------------------------------------------------------------
# S1: the sort offload (§3) — a second workload, not the
# BASELINE metric: 10^8 rows of 16-byte binary-sortable keys shaped like an ORDER BY over
# store_sales (sold date, store, item/ticket), sorted into a stable permutation.
# ----------------------------------------------------------------------------------------------
SORT_METRIC = "sort offload rows/s (partial-key radix sort + duplicate-range jobs, P:76-88)"
SORT_N, SORT_W = 100_000_000, 16


def sort_cpu(rows_np, n):
    import oracle
    t0 = time.perf_counter()
    oracle.sort_rows(rows_np[:n])
    return n / (time.perf_counter() - t0)


def run_sort_reference(args):
    if int(os.environ.get("RANK", "0")) != 0:
        return 0
    import blugen
    n = int(os.environ.get("BLU_BENCH_SORT_REF_ROWS", "2000000"))
    rows = blugen.sort_rows(n, SORT_W)
    for _ in range(args.warmup):
        sort_cpu(rows, n // 4)
    rates = [sort_cpu(rows, n) for _ in range(args.steps)]
    value = statistics.mean(rates)
    line = {"impl": "reference", "metric": SORT_METRIC, "value": value, "unit": "rows/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1000 * n / value, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": {"workload": f"S1: {SORT_W}-byte keys, rows per step {n} of {SORT_N}"},
            "cpu_baseline": {"value": value, "unit": "rows/s", "cores": 1, "kind": "oracle",
                             "sample": f"{n} rows of S1, std::stable_sort + memcmp oracle, single thread"},
            "e2e": {"value": value, "unit": "rows/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def init_dist(torch, dist):
    """One process per GPU (torchrun env), NCCL process group for N > 1. Test-only overrides:
    BLU_BENCH_DIST_BACKEND=gloo and BLU_BENCH_DEVICE=<index> run every rank on one GPU, to exercise the
    N > 1 code path (partition, exchange, merge, max-over-ranks timing) where only one GPU exists."""
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("BLU_BENCH_DEVICE", os.environ.get("LOCAL_RANK", "0")))
    torch.cuda.set_device(local)
    if world > 1:
        backend = os.environ.get("BLU_BENCH_DIST_BACKEND", "nccl")
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
    return world, rank, local


def run_sort(args):
    import torch
    import torch.distributed as dist

    import blugen
    from paper_conf_sigmod_merajispcksygnk16_b200 import blugby as bg

    world, rank, local = init_dist(torch, dist)
    dev = torch.device("cuda", local)
    stream = torch.cuda.current_stream(dev)
    n = args.rows or SORT_N
    rows_np = blugen.sort_rows(n, SORT_W, seed=blugen.SORT_SEED + rank)  # every rank its own rows (weak)
    rows = torch.from_numpy(rows_np).to(dev)
    flush = torch.empty(512 * 2**20, dtype=torch.uint8, device=dev)
    for _ in range(args.warmup):
        flush.zero_()
        perm, stats = bg.blu_sort_rows(rows, stream=stream)
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    sampler = ClockSampler(local if not args.no_clocks else -1)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    sampler.start()
    time.sleep(1.0)  # nvidia-smi (NVML) start-up stalls the driver for ~0.5 s: let it finish first
    c0 = bg.blu_gby_launch_count()
    ds_ms, ds_bytes, ds_launch = [], [], []
    for i in range(args.steps):
        flush.zero_()
        ev[i][0].record(stream)
        perm, stats = bg.blu_sort_rows(rows, stream=stream)
        ev[i][1].record(stream)
        ds_ms.append(stats["downsweep_ms"])
        ds_bytes.append(stats["downsweep_bytes"])
        ds_launch.append(stats["downsweep_launches"])
    torch.cuda.synchronize()
    launches = bg.blu_gby_launch_count() - c0
    if world > 1:
        dist.barrier()
    clocks = sampler.stop()
    tot_ms = sum(a.elapsed_time(b) for a, b in ev)
    if world > 1:
        t = torch.tensor([tot_ms], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        tot_ms = float(t.item())
    value = n * world * args.steps / (tot_ms / 1000.0)
    peak, peak_src = load_peaks()
    per_launch_ms = sum(ds_ms) / max(1, sum(ds_launch))
    per_launch_bytes = sum(ds_bytes) / max(1, sum(ds_launch))
    achieved = per_launch_bytes / (per_launch_ms / 1000.0) / 1e9
    traffic = None
    sp = os.path.join(ROOT, "profiles", "ncu_S1_summary.json")
    if os.path.exists(sp):  # DRAM bytes / algorithmic bytes of the captured downsweep, per average launch
        traffic = json.load(open(sp)).get("traffic_over_algorithmic", 0) * per_launch_bytes or None
    roofline = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                "traffic": traffic,
                "kernel": "k_rs_downsweep + k_seg_window_sort (sort passes: read + write of key, payload)",
                "algorithmic_bytes_per_launch": per_launch_bytes, "avg_launch_ms": per_launch_ms,
                "launches_per_step": sum(ds_launch) / args.steps,
                "share_of_step": sum(ds_ms) / tot_ms, "peak_source": peak_src,
                "levels": stats["levels"], "active_rows_per_level": stats["active"], "ms_per_level": stats["ms"]}
    e2e = None
    if not args.no_e2e and world == 1:
        hrows = rows.cpu().pin_memory()
        hperm = torch.empty(n, dtype=torch.int32).pin_memory()
        e_steps = min(3, args.steps)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for _ in range(e_steps):
            d = hrows.to(dev, non_blocking=True)
            p, _ = bg.blu_sort_rows(d, stream=stream)
            hperm.copy_(p, non_blocking=True)
            torch.cuda.synchronize()
        dt = (time.perf_counter() - t0) / e_steps
        e2e = {"value": n / dt, "unit": "rows/s", "h2d_bytes_per_step": n * SORT_W, "d2h_bytes_per_step": n * 4,
               "ms_per_step": dt * 1000, "note": "pinned host rows -> device, blu_sort_rows, permutation -> host"}
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        m = 2_000_000
        cpu = {"value": sort_cpu(rows_np, m), "unit": "rows/s", "cores": 1, "kind": "oracle",
               "sample": f"first {m} rows of S1, std::stable_sort + memcmp oracle, single thread"}
    if rank == 0:
        line = {"metric": SORT_METRIC, "value": value, "unit": "rows/s", "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": tot_ms / args.steps, "higher_is_better": True,
                "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
                "config": {"workload": f"S1: sort offload, {n} rows x {SORT_W}-byte keys (date 1823, store 502, "
                                       f"8 random bytes), stable permutation", "rows_per_gpu": n,
                           "parallelism": f"replicas x{world}",
                           "l2": "flushed between steps (512 MB memset, outside step events); inputs > L2"},
                "input_gbs": value * SORT_W / 1e9, "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e,
                "gpu_launches": launches, "clocks": clocks}
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0


# ----------------------------------------------------------------------------------------------
# GPU leg
# ----------------------------------------------------------------------------------------------
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--config", default="C2", choices=["C1", "C2", "C3", "C4", "C5", "S1"],
                    help="C1-C5: GROUP BY configs (BASELINE.json); S1: the sort offload (NEXT-4, P:76-88)")
    ap.add_argument("--impl", default="blugby", choices=["blugby", "reference"])
    ap.add_argument("--rows", type=int, default=None, help="override rows per rank (testing only)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-clocks", action="store_true", help="do not sample nvidia-smi (diagnostics)")
    args = ap.parse_args()
    args.warmup = max(3, args.warmup)
    if args.impl == "reference":
        return run_sort_reference(args) if args.config == "S1" else run_reference(args)
    if args.config == "S1":
        return run_sort(args)

    import torch
    import torch.distributed as dist

    import blugen
    from paper_conf_sigmod_merajispcksygnk16_b200 import blugby as bg
    from paper_conf_sigmod_merajispcksygnk16_b200 import dist as bdist

    world, rank, local = init_dist(torch, dist)
    bg.blu_gby_bind_device(local)
    dev = torch.device("cuda", local)
    stream = torch.cuda.current_stream(dev)

    w = blugen.workload(args.config, n_rows=args.rows) if args.rows else blugen.workload(args.config)
    if args.config == "C5" and world > 1:
        # C5 is 4B rows sharded over the GPUs (strong scaling of one query)
        per = w.n_rows // world
        row0, n = rank * per, (per if rank < world - 1 else w.n_rows - rank * per)
        scaling = "strong"
    else:
        row0, n = rank * w.n_rows, w.n_rows  # every rank its own rows (weak scaling)
        scaling = "weak"
    kc = [blugen.gen_device(c, w.seed, row0, n, dev) for c in w.key_cols]
    vc = [blugen.gen_device(c, w.seed, row0, n, dev) for c in w.val_cols]
    torch.cuda.synchronize()
    plan = bg.plan_for(w.schema, w.est_groups, w.n_rows if scaling == "strong" else n)
    info = plan.info()
    flush = torch.empty(512 * 2**20, dtype=torch.uint8, device=dev)

    def step():
        if world == 1:
            return bg.blu_gby_execute(plan, kc, vc, stream=stream)
        res, _ = bdist.dist_execute(plan, kc, vc, stream=stream)
        return res

    bg.blu_gby_set_timing(True)
    for _ in range(args.warmup):
        flush.zero_()
        r = step()
    n_groups = r.n_groups
    del r
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    agg_ms = []
    part_t = []
    agg_kernel = ""
    sampler = ClockSampler(local if not args.no_clocks else -1)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    sampler.start()
    time.sleep(1.0)  # nvidia-smi (NVML) start-up stalls the driver for ~0.5 s: let it finish first
    c0 = bg.blu_gby_launch_count()
    for i in range(args.steps):
        flush.zero_()
        ev[i][0].record(stream)
        r = step()
        ev[i][1].record(stream)
        t = getattr(r, "agg_timing", None) or bg.blu_gby_last_timing()  # N > 1: the rank-local aggregation
        agg_ms.append(t["aggregate_ms"] / max(1, t["aggregate_launches"]))
        agg_kernel = t["kernel"]
        part_t.append((t["scatter_ms"], t["pass2_ms"], t["part_chunks"]))
        del r
    torch.cuda.synchronize()
    launches = bg.blu_gby_launch_count() - c0
    if world > 1:
        dist.barrier()
    clocks = sampler.stop()
    step_ms = [a.elapsed_time(b) for a, b in ev]
    tot_ms = sum(step_ms)
    if world > 1:
        t = torch.tensor([tot_ms], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        tot_ms = float(t.item())
    rows_total = (w.n_rows if scaling == "strong" else n * world) * args.steps
    value = rows_total / (tot_ms / 1000.0)
    bpr = w.bytes_per_row
    input_gbs = value * bpr / 1e9
    peak, peak_src = load_peaks()

    # dominant kernel: the aggregation kernel (S5), timed with CUDA events on its launch stream
    agg_avg_ms = statistics.mean(agg_ms)
    rows_per_launch = n  # one aggregate launch per execute (rows < grid * 2^30)
    alg_bytes = rows_per_launch * bpr
    traffic, traffic_rows = load_traffic(args.config)
    phases = None
    chunks = max(c for _, _, c in part_t) if part_t else 0
    if chunks:
        # partitioned path (b): two kernels per chunk — the scatter (reads the input columns, writes
        # the bucket records) and pass 2 (reads the records); the longer one is the dominant kernel
        rec_bytes = 8 + sum(v.element_size() for v in vc)
        sc_ms = statistics.mean(a for a, _, _ in part_t) / chunks
        p2_ms = statistics.mean(b for _, b, _ in part_t) / chunks
        rows_per_launch = n / chunks
        # shared-memory bucket tables with >= 256 buckets: the scatter phase is two scatters (input ->
        # 32 buckets, then each bucket -> its sub-buckets), i.e. the records are written twice
        two_level = (info["part_smem"] == 1 and info["partitions"] >= 256
                     and os.environ.get("BLU_GBY_PART_2LEVEL", "1") != "0")
        sc_alg = rows_per_launch * (bpr + rec_bytes + (2 * rec_bytes if two_level else 0))
        p2_alg = rows_per_launch * rec_bytes
        tr_sc, tr_rows_sc = load_traffic(args.config, "scatter2" if two_level else "scatter")
        tr_p2, tr_rows_p2 = load_traffic(args.config, "pass2")
        phases = {
            "scatter": {"avg_launch_ms": sc_ms, "algorithmic_bytes_per_launch": sc_alg,
                        "achieved_gbs": sc_alg / (sc_ms / 1e3) / 1e9,
                        "traffic": tr_sc * rows_per_launch / tr_rows_sc if tr_sc and tr_rows_sc else None},
            "pass2": {"avg_launch_ms": p2_ms, "algorithmic_bytes_per_launch": p2_alg,
                      "achieved_gbs": p2_alg / (p2_ms / 1e3) / 1e9,
                      "traffic": tr_p2 * rows_per_launch / tr_rows_p2 if tr_p2 and tr_rows_p2 else None},
            "launches_per_step": chunks,
        }
        dom = "pass2" if p2_ms >= sc_ms else "scatter"
        agg_avg_ms = phases[dom]["avg_launch_ms"]
        alg_bytes = phases[dom]["algorithmic_bytes_per_launch"]
        traffic = phases[dom]["traffic"]
        agg_kernel = f"{dom}: " + (agg_kernel if dom == "pass2" else
                                   "blu_jit_scatter x2 levels" if two_level else "blu_jit_scatter")
        achieved = alg_bytes / (agg_avg_ms / 1000.0) / 1e9
    else:
        achieved = alg_bytes / (agg_avg_ms / 1000.0) / 1e9
        if traffic is not None and traffic_rows:
            traffic = traffic * rows_per_launch / traffic_rows
    # SURVEY §8(d) denominator (i): the same input columns streamed read-only by our own kernel with the
    # aggregation kernels' load instructions (L2 flushed before each launch, like the steps)
    rr_out = torch.zeros(1, dtype=torch.int64, device=dev)
    rr_ms = []
    for i in range(13):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        bg.blu_gby_read_roofline(kc + vc, rr_out, stream=stream)
        b.record(stream)
        b.synchronize()
        if i >= 3:
            rr_ms.append(a.elapsed_time(b))
    read_gbs = n * bpr / (statistics.median(rr_ms) / 1000.0) / 1e9
    roofline = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                "traffic": traffic, "kernel": agg_kernel,
                "algorithmic_bytes_per_launch": alg_bytes, "avg_launch_ms": agg_avg_ms, "phases": phases,
                "peak_source": peak_src, "share_of_step": agg_avg_ms / (tot_ms / args.steps),
                "read_only_ceiling_gbs": read_gbs, "frac_of_read_only_ceiling": achieved / read_gbs,
                "spec_peak_gbs": 8000.0, "frac_of_spec": achieved / 8000.0}

    # e2e: same metric through the C ABI with pinned HOST columns (H2D + D2H inside the timed region)
    e2e = None
    if not args.no_e2e and world == 1:
        hk = [k.cpu().pin_memory() for k in kc]
        hv = [v.cpu().pin_memory() for v in vc]
        h2d = sum(t.numel() * t.element_size() for t in hk + hv)
        bg.blu_gby_execute_host(plan, hk, hv, stream=stream)
        e_steps = min(3, args.steps)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        d2h = 0
        for _ in range(e_steps):
            res = bg.blu_gby_execute_host(plan, hk, hv, stream=stream)
            d2h = sum(a.nbytes for a in list(res.keys) + list(res.aggs))
        torch.cuda.synchronize()
        dt = (time.perf_counter() - t0) / e_steps
        e2e = {"value": n / dt, "unit": "rows/s", "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
               "ms_per_step": dt * 1000, "note": "blu_gby_execute_host: pinned host columns, chunked H2D "
                                                 "overlapped with aggregation, host result"}
        del hk, hv

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        cpu = cpu_baseline(args.config)

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "rows/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": tot_ms / args.steps, "higher_is_better": True,
            "scaling": scaling, "vs_baseline": None, "dtype": "int64+f64", "data": "synthetic",
            "config": {"workload": f"{args.config}: {w.note}", "rows_per_gpu": n, "groups": n_groups,
                       "bytes_per_row": bpr, "path": info["path_name"], "hot_front": info["hot_front"],
                       "partitions": info["partitions"], "bucket_tables": info["part_smem"],
                       "grid": info["grid"], "block": info["block"], "smem_bytes": info["smem_bytes"],
                       "parallelism": f"rows sharded x{world}" + (" + NCCL allreduce" if world > 1 and info["path"] != 1 else
                                                                   " + NCCL all-to-all" if world > 1 else ""),
                       "l2": "flushed between steps (512 MB memset, outside step events); inputs > L2"},
            "input_gbs": input_gbs, "hbm_frac_input": input_gbs / peak,
            "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": launches, "clocks": clocks,
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
