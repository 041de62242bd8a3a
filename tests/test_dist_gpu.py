"""End-to-end multi-rank GROUP BY through dist.dist_execute (the code bench.py runs at N > 1),
compared element by element with the CPU oracle.

P ranks (P = 2, 4) run as separate processes on ONE GPU over gloo (the only multi-process transport a
one-GPU box has; the collectives are the same torch.distributed calls the NCCL path issues). Each rank
generates its contiguous row range (the paper's range partitioning), runs
dist_execute, and sends its result to rank 0, which checks:
  * dense merge (paths a / b', C2 / C4 shapes): every rank holds the same replicated result, equal
    to the oracle over all rows ("merged together in the final step");
  * partials mode (C5 shape, rows per rank > est_groups) and rows mode (C3 shape, est_groups >= rows
    per rank): the owners' results are disjoint and their union equals the oracle (Table 1 fields,
    P:151; owner exchange SURVEY.md §8(e)).
"""
import os
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")

CASES = {
    # name: (config, rows, groups or None, expected mode)
    "dense_a_C2": ("C2", 600_001, None, "allreduce"),
    "dense_bprime_C4": ("C4", 800_003, None, "allreduce"),
    "partials_C5": ("C5", 1_200_007, 20_000, "partials"),
    "rows_C3": ("C3", 900_001, 600_000, "rows"),  # est 600K >= rows per rank (450K at P = 2)
}


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, case, q):
    try:
        import torch.distributed as dist

        import blugen
        from paper_conf_sigmod_merajispcksygnk16_b200 import blugby as bg
        from paper_conf_sigmod_merajispcksygnk16_b200 import dist as bdist

        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        torch.cuda.set_device(0)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        cfg, n, groups, want_mode = CASES[case]
        w = blugen.workload(cfg, n_rows=n, n_groups=groups) if groups else blugen.workload(cfg, n_rows=n)
        cuts = np.linspace(0, w.n_rows, world + 1).astype(np.int64)
        r0, r1 = int(cuts[rank]), int(cuts[rank + 1])
        kc = [blugen.gen_device(c, w.seed, r0, r1 - r0, "cuda") for c in w.key_cols]
        vc = [blugen.gen_device(c, w.seed, r0, r1 - r0, "cuda") for c in w.val_cols]
        plan = bg.plan_for(w.schema, w.est_groups, w.n_rows)
        bg.blu_gby_set_timing(True)
        res, mode = bdist.dist_execute(plan, kc, vc)
        keys = [k.cpu().numpy() for k in res.keys] if res.n_groups else []
        aggs = [a.cpu().numpy() for a in res.aggs] if res.n_groups else []
        payload = (rank, mode, int(res.n_groups), keys, aggs, sorted(getattr(res, "phase_ms", {}) or {}))
        out = [None] * world
        dist.all_gather_object(out, payload)
        if rank == 0:
            q.put(("ok", out))
        dist.barrier()
        dist.destroy_process_group()
    except Exception as e:  # pragma: no cover - reported to the parent
        import traceback
        q.put(("err", f"rank {rank}: {e!r}\n{traceback.format_exc()}"))


def _run(case, world):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, case, q)) for r in range(world)]
    for p in procs:
        p.start()
    try:
        status, out = q.get(timeout=600)
    finally:
        for p in procs:
            p.join(timeout=120)
            if p.is_alive():
                p.kill()
    assert status == "ok", out
    return out


def _sorted(keys, aggs):
    k = np.stack([x.astype(np.int64) for x in keys], axis=1)
    order = np.lexsort(k.T[::-1])
    return k[order], [a[order] for a in aggs]


@pytest.mark.parametrize("world", [2, 4])
@pytest.mark.parametrize("case", list(CASES))
def test_dist_execute_matches_oracle(case, world):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import blugen
    import oracle
    from parity_util import assert_parity

    cfg, n, groups, want_mode = CASES[case]
    w = blugen.workload(cfg, n_rows=n, n_groups=groups) if groups else blugen.workload(cfg, n_rows=n)
    o = oracle.groupby_generated(w)
    out = _run(case, world)
    modes = {m for _, m, _, _, _, _ in out}
    assert modes == {want_mode}, modes
    for _, _, _, _, _, phases in out:  # per-phase CUDA-event timing (bench.py's N > 1 line)
        assert "local_ms" in phases and "merge_ms" in phases, phases
    if want_mode == "allreduce":
        ref = None
        for rank, _, ng, keys, aggs, _ in out:  # replicated: every rank the full result
            gk, ga = _sorted(keys, aggs)
            assert_parity(gk, ga, o, w.schema)
            if ref is not None:
                assert np.array_equal(gk, ref)
            ref = gk
    else:
        allk = np.concatenate([np.stack([x.astype(np.int64) for x in keys], axis=1)
                               for _, _, ng, keys, _, _ in out if ng])
        alla = [np.concatenate([aggs[a] for _, _, ng, _, aggs, _ in out if ng]) for a in range(len(w.schema.aggs))]
        assert len(np.unique(allk, axis=0)) == len(allk)  # owners hold disjoint key ranges
        gk, ga = _sorted(list(allk.T), alla)
        assert_parity(gk, ga, o, w.schema)
