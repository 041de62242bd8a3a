"""bench.py's N > 1 path (one process per rank, max-over-ranks timing, partition / exchange / merge
through dist_execute) run with two ranks on one GPU over gloo (BLU_BENCH_DIST_BACKEND /
BLU_BENCH_DEVICE test overrides): launched the driver's way (torchrun) and as a plain
`python bench.py --gpus 2` (bench.py re-launches itself under torch.distributed.run). The JSON line
keeps the contract, reports n_gpus = 2, carries per-phase (local / exchange / merge) times, and the
roofline times the rank-local aggregation kernel."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.parametrize("launcher", ["torchrun", "self"])
@pytest.mark.parametrize("args", [["--config", "C2", "--rows", "4000000"], ["--config", "C5", "--rows", "8000000"]])
def test_bench_two_ranks_one_gpu(args, launcher):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    env = dict(os.environ, BLU_BENCH_DIST_BACKEND="gloo", BLU_BENCH_DEVICE="0")
    env.pop("WORLD_SIZE", None)
    bench = [os.path.join(ROOT, "bench.py"), "--gpus", "2", "--steps", "3", "--warmup", "3", "--no-e2e",
             "--no-clocks", *args]
    if launcher == "torchrun":
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
               "--master-addr", "127.0.0.1", "--master-port", "29561", *bench]
    else:
        cmd = [sys.executable, *bench]
    out = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=600)
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1  # rank 0 alone prints
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["steps"] == 3 and d["value"] > 0
    r = d["roofline"]
    assert r["avg_launch_ms"] > 0 and 0 < r["frac"] < 1.5, r
    assert d["gpu_launches"] > 0
    ph = d["phase_ms"]
    assert ph and ph["local_ms"] > 0 and "exchange_ms" in ph and ph["merge_ms"] > 0, ph
