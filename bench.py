#!/usr/bin/env python
"""bench.py — GROUP BY throughput of libblugby on B200 (BASELINE.json metric).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config C5] [--impl blugby|reference]

One "step" is one whole GROUP BY of one batch of synthetic fact-table rows (SURVEY.md §8(a) S0-S10:
init, aggregate, CTA merge, compaction, the host read of n_groups; at N > 1 plus the owner exchange
or the NCCL all-reduce and the merge). The headline workload is C5 (BASELINE.json configs[4]: 4e9
rows, one sparse i64 key, 5e7 groups, COUNT/SUM/AVG, path (b)), the largest configuration and the one
north_star quotes the 1 -> 8 GPU scaling on; at N > 1 its 4e9 rows are split over the ranks (strong
scaling) and the partial states are exchanged by owner with an NCCL all-to-all. At N = 1 the line
also carries sub-records for C3, C4 and C2, each with its own roofline object (--sub '' turns them
off). `--gpus N` without torchrun re-launches itself under torch.distributed.run with N ranks.

Timing: inputs generated in HBM before timing; between steps L2 is flushed (a 512 MB memset, outside
the per-step CUDA events); each step is bracketed by CUDA events on the launching stream; K steps are
bracketed by a barrier + synchronize; the max over ranks is reported. `--impl reference` times the
CPU oracle (oracle/, plain std::map) key-sliced over the host cores on bounded samples of the same
workload.
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
def _oracle_slice(job):
    """One key slice of the oracle over rows [row0, row0 + n) (a worker process)."""
    config, row0, n, p, P = job
    import blugen
    import oracle
    w = blugen.workload(config)
    t0 = time.perf_counter()
    o = oracle.groupby_generated(w, row0=row0, n=n, slice_p=p, slice_P=P)
    return o.n_groups, time.perf_counter() - t0


def cpu_model():
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.startswith("model name"):
                return ln.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def oracle_sliced(config, row0, n, P):
    """The oracle as it stands, key-sliced over P processes (slice p takes the rows with
    (k0 + 31 k1 + 961 k2) mod P == p; each regenerates the rows from the counter-based generator).
    Returns (rows/s over the whole sample, wall seconds, groups)."""
    import multiprocessing as mpc
    jobs = [(config, row0, n, p, P) for p in range(P)]
    t0 = time.perf_counter()
    if P == 1:
        out = [_oracle_slice(jobs[0])]
    else:
        with mpc.get_context("spawn").Pool(P) as pool:
            out = pool.map(_oracle_slice, jobs)
    dt = time.perf_counter() - t0
    return n / dt, dt, sum(g for g, _ in out)


def sample_rows(config, P, seconds):
    """Rows of a bounded sample that keeps the key-sliced oracle busy for about `seconds` (calibrated on
    growing samples so the worker start-up does not distort the rate)."""
    import blugen
    full = blugen.workload(config).n_rows
    n = 2_000_000
    while True:
        _, dt, _ = oracle_sliced(config, 0, n, P)
        if dt >= seconds / 4 or n >= full:
            return int(max(1, min(full, n * seconds / max(dt, 1e-3))))
        n = min(full, n * 4)


def cpu_baseline(config, seconds=12.0):
    """The oracle as it stands on the host cores (key-sliced, one process per core) on a bounded
    sample: the first R rows of the workload, R sized for ~`seconds` of wall time."""
    P = max(1, os.cpu_count() or 1)
    rows = sample_rows(config, P, seconds)
    rate, dt, ng = oracle_sliced(config, 0, rows, P)
    return {"value": rate, "unit": "rows/s", "cores": P, "kind": "oracle",
            "sample": f"{config} rows [0, {rows}) ({dt:.1f} s wall, {ng} groups), plain std::map oracle key-sliced "
                      f"over {P} processes ((k0 + 31 k1 + 961 k2) mod {P}), CPU: {cpu_model()}"}


def run_reference(args):
    """The reference arm: the oracle as it stands (there is no reference implementation; the reference
    is a paper), key-sliced over the host cores, each step a bounded sample of this workload's rows."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import blugen
    w = blugen.workload(args.config)
    P = max(1, os.cpu_count() or 1)
    budget = float(os.environ.get("BLU_BENCH_REF_BUDGET_S", "90"))
    rows = sample_rows(args.config, P, budget / max(1, args.steps + args.warmup))
    span = max(1, w.n_rows - rows)
    for i in range(args.warmup):
        oracle_sliced(args.config, (i * rows) % span, rows, P)
    times = []
    for i in range(args.steps):
        _, dt, _ = oracle_sliced(args.config, ((args.warmup + i) * rows) % span, rows, P)
        times.append(dt)
    tot = sum(times)
    value = rows * args.steps / tot
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": "rows/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1000 * tot / args.steps,
            "higher_is_better": True, "scaling": "strong" if args.config == "C5" else "weak", "vs_baseline": None,
            "dtype": "int64+f64", "data": "synthetic",
            "config": {"workload": f"{args.config}: {w.note}", "rows_per_step": rows, "full_rows": w.n_rows},
            "cpu_baseline": {"value": value, "unit": "rows/s", "cores": P, "kind": "oracle",
                             "sample": f"{rows} rows per step of {args.config}, std::map oracle key-sliced over {P} "
                                       f"processes, CPU: {cpu_model()}"},
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
def ncu_dram_frac(config, peak):
    """ncu achieved DRAM throughput of the committed capture of this config's dominant kernel(s)
    (profiles/ncu_<config>*_summary.json): dram bytes / duration / peak, per summary."""
    out = {}
    d = os.path.join(ROOT, "profiles")
    for fn in sorted(os.listdir(d)) if os.path.isdir(d) else []:
        if fn.startswith(f"ncu_{config}_") and fn.endswith("_summary.json") or fn == f"ncu_{config}_summary.json":
            try:
                s = json.load(open(os.path.join(d, fn)))
                b, t = s.get("dram_bytes_per_launch"), s.get("duration_s")
                if b and t:  # read + write bytes over the captured launch, against the same peak
                    out[fn[4:-13] or config] = {"dram_gbs": b / t / 1e9, "frac": b / t / 1e9 / peak,
                                                "ncu_dram_throughput_pct": s.get("dram_throughput_pct"),
                                                "kernel": s.get("kernel")}
            except (OSError, ValueError):
                pass
    return out or None


def measure(cfg, args, world, rank, local, torch, dist, bg, bdist, sampler_on):
    """Time K steps of one configuration on this rank; returns the record (rank 0 prints it)."""
    import blugen
    dev = torch.device("cuda", local)
    stream = torch.cuda.current_stream(dev)
    w = blugen.workload(cfg, n_rows=args.rows) if args.rows and cfg == args.config else blugen.workload(cfg)
    if cfg == "C5" and world > 1:
        # C5 is one 4e9-row query sharded over the GPUs (strong scaling)
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
    steps = args.steps if cfg == args.config else max(3, min(args.steps, args.sub_steps))
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(steps)]
    agg_ms, part_t, phase = [], [], {}
    agg_kernel = ""
    sampler = ClockSampler(local if sampler_on else -1)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    sampler.start()
    time.sleep(1.0 if sampler_on else 0.0)  # nvidia-smi (NVML) start-up stalls the driver for ~0.5 s
    c0 = bg.blu_gby_launch_count()
    for i in range(steps):
        flush.zero_()
        ev[i][0].record(stream)
        r = step()
        ev[i][1].record(stream)
        t = getattr(r, "agg_timing", None) or bg.blu_gby_last_timing()  # N > 1: the rank-local aggregation
        agg_ms.append(t["aggregate_ms"] / max(1, t["aggregate_launches"]))
        agg_kernel = t["kernel"]
        part_t.append((t["scatter_ms"], t["pass2_ms"], t["part_chunks"]))
        for k, v in (getattr(r, "phase_ms", None) or {}).items():
            phase[k] = phase.get(k, 0.0) + v / steps
        del r
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
    rows_total = (w.n_rows if scaling == "strong" else n * world) * steps
    value = rows_total / (tot_ms / 1000.0)
    bpr = w.bytes_per_row
    peak, peak_src = load_peaks()

    # dominant kernel, timed with CUDA events on its launch stream. SURVEY §8(d): the algorithmic
    # bytes are the input columns (bpr per row) the launch consumes; bytes the method itself moves
    # (partition records written and read back) are reported in `traffic` / `method_bytes_per_row`.
    agg_avg_ms = statistics.mean(agg_ms)
    rows_per_launch = n
    traffic, traffic_rows = load_traffic(cfg)
    phases = None
    chunks = max(c for _, _, c in part_t) if part_t else 0
    method_bpr = bpr
    if chunks:
        rec_bytes = 8 + sum(v.element_size() for v in vc)
        sc_ms = statistics.mean(a for a, _, _ in part_t) / chunks
        p2_ms = statistics.mean(b for _, b, _ in part_t) / chunks
        rows_per_launch = n / chunks
        levels = info.get("scatter_levels", 2 if (info["part_smem"] == 1 and info["partitions"] >= 256) else 1)
        method_bpr = bpr + rec_bytes * (2 * levels)  # each scatter level writes the records once, the next reads them
        # scatter traffic per launch: the first level's capture scaled to the chunk, plus (two levels)
        # one second-level launch's capture scaled to the chunk (the second level reads the first
        # level's output partly from L2)
        tr_sc, tr_rows_sc = load_traffic(cfg, "scatter")
        if levels == 2 and tr_sc and tr_rows_sc:
            tr_sc2, tr_rows_sc2 = load_traffic(cfg, "scatter2")
            if tr_sc2 and tr_rows_sc2:
                tr_sc, tr_rows_sc = (tr_sc / tr_rows_sc + tr_sc2 / tr_rows_sc2) * tr_rows_sc, tr_rows_sc
            else:
                tr_sc = None
        tr_p2, tr_rows_p2 = load_traffic(cfg, "pass2")
        alg = rows_per_launch * bpr
        phases = {
            "scatter": {"avg_launch_ms": sc_ms, "algorithmic_bytes_per_launch": alg,
                        "achieved_gbs": alg / (sc_ms / 1e3) / 1e9, "levels": levels,
                        "moved_bytes_per_row": bpr + rec_bytes * (2 * levels - 1),
                        "traffic": tr_sc * rows_per_launch / tr_rows_sc if tr_sc and tr_rows_sc else None},
            "pass2": {"avg_launch_ms": p2_ms, "algorithmic_bytes_per_launch": alg,
                      "achieved_gbs": alg / (p2_ms / 1e3) / 1e9, "moved_bytes_per_row": rec_bytes,
                      "traffic": tr_p2 * rows_per_launch / tr_rows_p2 if tr_p2 and tr_rows_p2 else None},
            "launches_per_step": chunks,
        }
        dom = "pass2" if p2_ms >= sc_ms else "scatter"
        agg_avg_ms = phases[dom]["avg_launch_ms"]
        traffic = phases[dom]["traffic"]
        agg_kernel = f"{dom}: " + (agg_kernel if dom == "pass2" else f"blu_jit_scatter x{levels} level(s)")
    elif traffic is not None and traffic_rows:
        traffic = traffic * rows_per_launch / traffic_rows
    alg_bytes = rows_per_launch * bpr
    achieved = alg_bytes / (agg_avg_ms / 1000.0) / 1e9
    # SURVEY §8(d) denominator (i): the same input columns streamed read-only by our own kernel with the
    # aggregation kernels' load instructions (L2 flushed before each launch, like the steps)
    rr_out = torch.zeros(1, dtype=torch.int64, device=dev)
    rr_ms = []
    for i in range(8):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        bg.blu_gby_read_roofline(kc + vc, rr_out, stream=stream)
        b.record(stream)
        b.synchronize()
        if i >= 3:
            rr_ms.append(a.elapsed_time(b))
    read_gbs = n * bpr / (statistics.median(rr_ms) / 1000.0) / 1e9
    step_ms = tot_ms / steps
    roofline = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                "traffic": traffic, "kernel": agg_kernel,
                "algorithmic_bytes_per_launch": alg_bytes, "algorithmic_bytes_per_row": bpr,
                "avg_launch_ms": agg_avg_ms, "phases": phases, "peak_source": peak_src,
                "share_of_step": agg_avg_ms * (chunks or 1) / step_ms,
                "read_only_ceiling_gbs": read_gbs, "frac_of_read_only_ceiling": achieved / read_gbs,
                "spec_peak_gbs": 8000.0, "frac_of_spec": achieved / 8000.0,
                "method_bytes_per_row": method_bpr,
                "frac_method": (n * method_bpr / (step_ms / 1e3) / 1e9) / peak,
                "ncu_dram_frac": ncu_dram_frac(cfg, peak)}
    input_gbs = value * bpr / 1e9
    rec = {"config": cfg, "value": value, "unit": "rows/s", "ms_per_step": step_ms, "steps": steps,
           "scaling": scaling, "workload": f"{cfg}: {w.note}", "rows": w.n_rows, "rows_per_gpu": n,
           "groups": n_groups, "bytes_per_row": bpr, "path": info["path_name"], "hot_front": info["hot_front"],
           "partitions": info["partitions"], "bucket_tables": info["part_smem"], "grid": info["grid"],
           "block": info["block"], "smem_bytes": info["smem_bytes"], "input_gbs": input_gbs,
           "hbm_frac_input": input_gbs / peak / (world if scaling == "strong" or world > 1 else 1),
           "roofline": roofline, "gpu_launches": launches, "clocks": clocks,
           "phase_ms": phase or None}
    # e2e: the same metric through the C ABI with pinned HOST columns (H2D + D2H inside the timed region),
    # on a prefix of the workload (the host-resident query is PCIe-bound: rows/s does not depend on size)
    rec["e2e"] = None
    if not args.no_e2e and world == 1 and cfg == args.config:
        m = min(n, int(os.environ.get("BLU_BENCH_E2E_ROWS", 250_000_000)))
        hk = [k[:m].cpu().pin_memory() for k in kc]
        hv = [v[:m].cpu().pin_memory() for v in vc]
        h2d = sum(t.numel() * t.element_size() for t in hk + hv)
        plan_m = bg.plan_for(w.schema, w.est_groups, m)
        for _ in range(2):  # warm-up: JIT, workspace and the pinned result blocks
            res = bg.blu_gby_execute_host(plan_m, hk, hv, stream=stream)
            del res
        e_steps = 3
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        d2h = 0
        for _ in range(e_steps):
            res = bg.blu_gby_execute_host(plan_m, hk, hv, stream=stream)
            d2h = sum(a.nbytes for a in list(res.keys) + list(res.aggs))
            del res  # the caller consumes the host result, then releases it
        torch.cuda.synchronize()
        dt = (time.perf_counter() - t0) / e_steps
        rec["e2e"] = {"value": m / dt, "unit": "rows/s", "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
                      "ms_per_step": dt * 1000, "rows_per_step": m,
                      "note": f"blu_gby_execute_host on rows [0, {m}) of {cfg}: pinned host columns -> device "
                              f"(whole, or chunked and overlapped with aggregation), host result in pinned "
                              f"memory (PCIe-bound)"}
        del hk, hv
    del kc, vc, flush
    bg.blu_gby_release_workspace()
    torch.cuda.empty_cache()
    return rec


def relaunch(args):
    """`bench.py --gpus N` outside torchrun: re-run this command under torch.distributed.run with N
    ranks on this node (127.0.0.1 rendezvous), so the driver's plain invocation spawns every rank."""
    import socket
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="C5", choices=["C1", "C2", "C3", "C4", "C5", "S1"],
                    help="C1-C5: GROUP BY configs (BASELINE.json); S1: the sort offload (NEXT-4, P:76-88)")
    ap.add_argument("--sub", default="C3,C4,C2", help="N = 1: configs measured as sub-records ('' = none)")
    ap.add_argument("--sub-steps", type=int, default=10)
    ap.add_argument("--impl", default="blugby", choices=["blugby", "reference"])
    ap.add_argument("--rows", type=int, default=None, help="override rows of --config (testing only)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-clocks", action="store_true", help="do not sample nvidia-smi (diagnostics)")
    args = ap.parse_args()
    args.warmup = max(3, args.warmup)
    if "WORLD_SIZE" not in os.environ and args.gpus > 1:
        return relaunch(args)
    if args.impl == "reference":
        return run_sort_reference(args) if args.config == "S1" else run_reference(args)
    if args.config == "S1":
        return run_sort(args)
    world = int(os.environ.get("WORLD_SIZE", "1"))
    assert world == args.gpus, f"--gpus {args.gpus} but WORLD_SIZE {world}"
    # the oracle's CPU baseline first, before this process holds GPU memory (spawned workers)
    cpu = None
    if int(os.environ.get("RANK", "0")) == 0 and world == 1 and not args.no_cpu:
        cpu = cpu_baseline(args.config)

    import torch
    import torch.distributed as dist

    from paper_conf_sigmod_merajispcksygnk16_b200 import blugby as bg
    from paper_conf_sigmod_merajispcksygnk16_b200 import dist as bdist

    world, rank, local = init_dist(torch, dist)
    bg.blu_gby_bind_device(local)
    head = measure(args.config, args, world, rank, local, torch, dist, bg, bdist, not args.no_clocks)
    subs = {}
    if world == 1 and args.sub:
        for c in [x for x in args.sub.split(",") if x and x != args.config]:
            r = measure(c, args, world, rank, local, torch, dist, bg, bdist, False)
            r.pop("clocks", None)
            subs[c] = r
    if rank == 0:
        par = f"rows sharded x{world}" + ("" if world == 1 else " + NCCL all-reduce" if head["path"][0] != "b" or
                                          head["path"].startswith("b'") else " + NCCL all-to-all")
        line = {
            "metric": METRIC, "value": head["value"], "unit": "rows/s", "n_gpus": world, "steps": head["steps"],
            "warmup": args.warmup, "ms_per_step": head["ms_per_step"], "higher_is_better": True,
            "scaling": head["scaling"], "vs_baseline": None, "dtype": "int64+f64", "data": "synthetic",
            "config": {"workload": head["workload"], "rows": head["rows"], "rows_per_gpu": head["rows_per_gpu"],
                       "groups": head["groups"], "bytes_per_row": head["bytes_per_row"], "path": head["path"],
                       "hot_front": head["hot_front"], "partitions": head["partitions"],
                       "bucket_tables": head["bucket_tables"], "grid": head["grid"], "block": head["block"],
                       "smem_bytes": head["smem_bytes"], "parallelism": par,
                       "l2": "flushed between steps (512 MB memset, outside step events); inputs > L2"},
            "input_gbs": head["input_gbs"], "hbm_frac_input": head["hbm_frac_input"],
            "roofline": head["roofline"], "cpu_baseline": cpu, "e2e": head["e2e"],
            "gpu_launches": head["gpu_launches"], "clocks": head["clocks"], "phase_ms": head["phase_ms"],
            "sub_records": subs or None,
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
