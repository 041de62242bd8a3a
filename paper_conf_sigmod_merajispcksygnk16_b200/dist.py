"""Multi-GPU GROUP BY over torch.distributed (NCCL over NVLink / NVSwitch; gloo for CPU tests).

One process per GPU; each rank aggregates its contiguous row range (the paper's range
partitioning, "the input data is partitioned ... sent to some number of available
GPU devices ... The results are then merged together in the final step"). The merge is chosen by
the plan's path:

  * dense state (paths a / b'): every rank holds the same D x fields state arrays; three
    all-reduces issued back to back (int64 SUM, f64 SUM, and int64 MIN over MIN ++ ~MAX) combine
    them; every rank finalizes the same replicated result;
  * hash path (b), partials mode (default when the rank's rows outnumber the estimated groups):
    each rank emits per-group partial states, buckets them by owner rank (mulhi(fmix64(key), P),
    bits independent of the slot bits), exchanges them with an all-to-all-v and merges what it
    owns; the result is distributed by key range;
  * hash path (b), rows mode (est_groups >= rows per rank: partial states would be as large as
    the rows): the raw rows are bucketed by owner, exchanged, and aggregated by their owner.

The collective orchestration (`allreduce_dense_state`, `alltoallv_records`) only moves tensors; all
GROUP BY arithmetic stays in libblugby.
"""
from __future__ import annotations

from typing import List, Sequence

import torch
import torch.distributed as dist


class _Phases:
    """CUDA events around the local, exchange and merge phases of one dist_execute (on the launching
    stream); read after the call's own synchronisation. Off unless timing is enabled."""

    def __init__(self, on: bool, stream):
        self.on = on
        self.stream = stream
        self.ev = []

    def mark(self, name: str):
        if self.on:
            e = torch.cuda.Event(enable_timing=True)
            e.record(self.stream)
            self.ev.append((name, e))

    def result(self) -> dict:
        if not self.on or len(self.ev) < 2:
            return {}
        self.ev[-1][1].synchronize()
        out = {}
        for (_, a), (name, b) in zip(self.ev, self.ev[1:]):
            out[name + "_ms"] = out.get(name + "_ms", 0.0) + a.elapsed_time(b)
        return out


def allreduce_dense_state(state_arrays: Sequence[torch.Tensor], group=None) -> None:
    """[int64 SUM group, f64 SUM group, int64 MIN group, int64 MAX group] in place, with three
    collectives issued back to back (no host wait between them): int64 SUM, f64 SUM, and one int64
    MIN over the MIN group concatenated with the bitwise complement of the MAX group (~ reverses the
    order of two's-complement integers, so max(x) = ~min(~x) with no overflow at INT64_MIN)."""
    isum, fsum, mn, mx = state_arrays
    works = []
    if isum.numel():
        works.append(dist.all_reduce(isum, op=dist.ReduceOp.SUM, group=group, async_op=True))
    if fsum.numel():
        works.append(dist.all_reduce(fsum, op=dist.ReduceOp.SUM, group=group, async_op=True))
    mm = None
    if mn.numel() or mx.numel():
        mm = torch.cat([mn.reshape(-1), torch.bitwise_not(mx.reshape(-1))])
        works.append(dist.all_reduce(mm, op=dist.ReduceOp.MIN, group=group, async_op=True))
    for w in works:
        w.wait()
    if mm is not None:
        a = mn.numel()
        if a:
            mn.copy_(mm[:a].reshape(mn.shape))
        if mx.numel():
            torch.bitwise_not(mm[a:], out=mm[a:])
            mx.copy_(mm[a:].reshape(mx.shape))


def alltoallv_records(send: torch.Tensor, send_counts: List[int], words: int, group=None) -> torch.Tensor:
    """Exchange variable-size buckets of fixed-width records (int64 words). send holds the buckets
    for ranks 0..P-1 back to back; send_counts[p] records go to rank p. Returns the received records
    (concatenated in source-rank order) as a 1-D int64 tensor of words."""
    P = dist.get_world_size(group)
    dev = send.device
    sc = torch.tensor(send_counts, dtype=torch.int64, device=dev)
    rc = torch.empty(P, dtype=torch.int64, device=dev)
    dist.all_to_all_single(rc, sc, group=group)
    recv_counts = [int(x) for x in rc.cpu().tolist()]
    recv = torch.empty(max(1, sum(recv_counts)) * words, dtype=torch.int64, device=dev)
    dist.all_to_all_single(recv[: sum(recv_counts) * words], send[: sum(send_counts) * words],
                           output_split_sizes=[c * words for c in recv_counts],
                           input_split_sizes=[c * words for c in send_counts], group=group)
    return recv[: sum(recv_counts) * words]


def owner_plan(plan, P: int):
    """The plan an owner aggregates its received records with. Owners hold ~1/P of the groups
    (owner = mulhi(fmix64(key), P)), so the owner-side table is sized from est_groups / P; the global
    estimate (reading A19) would give every owner a table P times too large (C5 at P = 8: 4.3 GB instead
    of 537 MB, with an 8x larger init and compaction). Cached per plan; P = 1 is the plan itself."""
    if P <= 1:
        return plan
    cache = plan.__dict__.setdefault("_owner_plans", {})
    if P not in cache:
        from . import blugby as bg
        info = plan.info()
        est = max(1, -(-int(info["est_groups"]) // P))
        cache[P] = bg.blu_gby_plan(plan.keys, plan.vals, plan.aggs, est, max(1, est))
    return cache[P]


def exchange_mode(plan, n_local: int, mode=None) -> str:
    """'rows' when the estimate says partial states would not be smaller than the
    rows (est_groups >= rows on this rank), else 'partials'; an explicit mode wins."""
    if mode in ("rows", "partials"):
        return mode
    return "rows" if plan.info()["est_groups"] >= max(1, n_local) else "partials"


def dist_execute(plan, key_cols, val_cols, group=None, stream=None, mode=None):
    """Whole-job GROUP BY of this rank's rows; returns (result, mode). Dense paths: replicated
    finalized result; hash path: this rank's owned groups (mode 'partials' or 'rows').
    With timing on (blu_gby_set_timing), res.agg_timing holds the rank-local aggregation's
    blu_gby_last_timing() and res.phase_ms the CUDA-event times of the local / exchange / merge
    phases on this rank."""
    from . import blugby as bg
    P = dist.get_world_size(group)
    info = plan.info()
    if stream is None:
        stream = torch.cuda.current_stream(key_cols[0].device) if key_cols[0].is_cuda else None
    ph = _Phases(bool(bg.timing_enabled()) and stream is not None, stream)
    ph.mark("start")
    if info["path"] != bg.BLU_PATH_HASH_GLOBAL:
        st = bg.dense_state_arrays(plan, device=key_cols[0].device)
        bg.blu_gby_execute_dense_state(plan, key_cols, val_cols, st, init=True, stream=stream)
        t = bg.blu_gby_last_timing()
        ph.mark("local")
        if P > 1:
            allreduce_dense_state(st, group)
        ph.mark("exchange")
        res = bg.blu_gby_finalize_dense_state(plan, st, stream=stream)
        ph.mark("merge")
        res.agg_timing = t
        res.phase_ms = ph.result()
        return res, "allreduce"
    n_local = int(len(key_cols[0]))
    if P > 1 and exchange_mode(plan, n_local, mode) == "rows":
        words = plan.row_record_bytes // 8
        send = torch.empty(max(1, n_local) * words, dtype=torch.int64, device=key_cols[0].device)
        counts = bg.blu_gby_partition_rows(plan, key_cols, val_cols, P, send, stream=stream)
        ph.mark("local")
        recv = alltoallv_records(send, counts, words, group)
        ph.mark("exchange")
        res = bg.blu_gby_execute_records(owner_plan(plan, P), recv, recv.numel() // words, stream=stream)
        res.agg_timing = bg.blu_gby_last_timing()
        ph.mark("merge")
        res.phase_ms = ph.result()
        return res, "rows"
    part = bg.blu_gby_execute_partial(plan, key_cols, val_cols, stream=stream)
    t = bg.blu_gby_last_timing()
    if P == 1:
        ph.mark("local")
        res = bg.blu_gby_merge(plan, [part], stream=stream)
        ph.mark("merge")
        res.agg_timing = t
        res.phase_ms = ph.result()
        return res, "local"
    words = plan.record_bytes // 8
    send = torch.empty(max(1, part.n_groups) * words, dtype=torch.int64, device=key_cols[0].device)
    counts = bg.blu_gby_partition(plan, part, P, send, stream=stream)
    del part
    ph.mark("local")
    recv = alltoallv_records(send, counts, words, group)
    del send
    ph.mark("exchange")
    res = bg.blu_gby_merge_records(owner_plan(plan, P), recv, recv.numel() // words, stream=stream)
    ph.mark("merge")
    res.agg_timing = t
    res.phase_ms = ph.result()
    return res, "partials"
