"""Multi-process (world_size 2, gloo, CPU) tests of the collective orchestration in dist.py: the
dense-state allreduce groups (SUM / SUM / MIN / MAX) and the all-to-all-v of fixed-width records.
The GPU library calls around them are covered by the single-GPU simulated-rank tests."""
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _dist_module():
    # dist.py imports only torch at module level; load it without importing the package __init__
    # (which loads libblugby and would not be needed here).
    import importlib.util
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    spec = importlib.util.spec_from_file_location("blu_dist", os.path.join(
        root, "paper_conf_sigmod_merajispcksygnk16_b200", "dist.py"))
    m = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(m)
    return m


def _worker(rank, world, port, q):
    try:
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=world)
        bd = _dist_module()
        # dense state: 4 groups with rank-dependent contents
        D = 7
        isum = torch.arange(2 * D, dtype=torch.int64) * (rank + 1)
        fsum = torch.full((D,), 0.5 * (rank + 1), dtype=torch.float64)
        mn = torch.tensor([10 - rank, -3 * rank, 2**62, 0, 5, 6, 7], dtype=torch.int64)
        mx = torch.tensor([rank, -rank, -(2**62), 0, 5, 6, 7 + rank], dtype=torch.int64)
        empty = torch.empty(0, dtype=torch.int64)
        bd.allreduce_dense_state([isum, fsum, mn, mx, ][:4])
        ok1 = (torch.equal(isum, torch.arange(2 * D, dtype=torch.int64) * 3) and torch.allclose(fsum, torch.full((D,), 1.5, dtype=torch.float64))
               and mn.tolist() == [9, -3, 2**62, 0, 5, 6, 7] and mx.tolist() == [1, 0, -(2**62), 0, 5, 6, 8])
        bd.allreduce_dense_state([empty, torch.empty(0, dtype=torch.float64), empty.clone(), empty.clone()])
        # all-to-all-v of records (words = 3): rank r sends (r+1)*(d+1) records to rank d,
        # record = [src, dst, i]
        words = 3
        counts = [(rank + 1) * (d + 1) for d in range(world)]
        send = torch.cat([torch.tensor([[rank, d, i] for i in range(c)], dtype=torch.int64).reshape(-1)
                          for d, c in enumerate(counts)])
        recv = bd.alltoallv_records(send, counts, words)
        rec = recv.reshape(-1, words).tolist()
        want = [[s, rank, i] for s in range(world) for i in range((s + 1) * (rank + 1))]
        ok2 = rec == want
        # zero records to send
        recv0 = bd.alltoallv_records(torch.empty(0, dtype=torch.int64), [0] * world, words)
        ok3 = recv0.numel() == 0
        q.put((rank, ok1, ok2, ok3))
        dist.destroy_process_group()
    except Exception as e:  # pragma: no cover
        q.put((rank, repr(e), False, False))


def test_dense_allreduce_and_alltoallv_world2():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    for rank, ok1, ok2, ok3 in res:
        assert ok1 is True, (rank, ok1)
        assert ok2 and ok3, rank


def test_bench_reference_arm_cpu():
    """`bench.py --impl reference` (the oracle on host cores) prints one valid JSON line."""
    import json
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, BLU_BENCH_REF_BUDGET_S="2")
    out = subprocess.run([sys.executable, os.path.join(root, "bench.py"), "--impl", "reference", "--steps", "2",
                          "--warmup", "1"], capture_output=True, text=True, env=env, timeout=300)
    assert out.returncode == 0, out.stderr[-2000:]
    line = json.loads(out.stdout.strip().splitlines()[-1])
    assert line["impl"] == "reference" and line["value"] > 0 and line["unit"] == "rows/s"
    assert line["cpu_baseline"]["kind"] == "oracle" and line["e2e"]["h2d_bytes_per_step"] == 0


def test_exchange_mode_rule():
    """rows mode when est_groups >= rows on this rank, partials otherwise; an
    explicit mode wins."""
    bd = _dist_module()

    class Stub:
        def __init__(self, est):
            self.est = est

        def info(self):
            return {"est_groups": self.est}

    assert bd.exchange_mode(Stub(50_000_000), 500_000_000) == "partials"   # C5 at P = 8
    assert bd.exchange_mode(Stub(50_000_000), 10_000_000) == "rows"        # as many groups as rows
    assert bd.exchange_mode(Stub(10), 10) == "rows"
    assert bd.exchange_mode(Stub(10**9), 5, mode="partials") == "partials"
    assert bd.exchange_mode(Stub(1), 10**9, mode="rows") == "rows"
