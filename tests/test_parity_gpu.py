"""GPU parity: libblugby (through its C ABI) vs the CPU oracle on the same seeded inputs.

Sizes span many tiles and CTAs with ragged tails; configs C1..C5 are scaled down so the oracle
finishes in seconds (full-size checks live in test_fullsize_gpu.py). Integers, keys and the dyadic
f64 columns are compared bit-exactly (north_star; readings A12/A13)."""
import os

import numpy as np
import pytest

import blugen
import oracle
from blugen import AVG, COUNT, F64, I32, I64, MAX, MIN, REAL, SUM
from parity_util import assert_parity, gpu_sorted, host_sorted

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def bg():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sigmod_merajispcksygnk16_b200 import blugby
    return blugby


SCALED = {
    "C1": dict(n_rows=1_000_003),
    "C2": dict(n_rows=2_000_011),
    "C3": dict(n_rows=2_000_003, n_groups=60_000),
    "C4": dict(n_rows=3_000_017),
    "C5": dict(n_rows=2_500_001, n_groups=150_000),
    "K3": dict(n_rows=2_000_003, n_groups=1_000_000),
}


def run_gpu(bg, w, est=None, **env):
    kc, vc = blugen.device_columns(w)
    plan = bg.plan_for(w.schema, w.est_groups if est is None else est, w.n_rows)
    res = bg.blu_gby_execute(plan, kc, vc)
    return plan, res


@pytest.fixture(scope="module")
def oracles():
    cache = {}

    def get(name):
        if name not in cache:
            w = blugen.workload(name, **SCALED[name])
            cache[name] = (w, oracle.groupby_generated(w))
        return cache[name]
    return get


@pytest.mark.parametrize("jit", ["1", "0", "1-nopipe"])
@pytest.mark.parametrize("name", ["C1", "C2", "C3", "C4", "C5"])
def test_config_parity(bg, oracles, monkeypatch, name, jit):
    """The NVRTC-specialised kernels (default: software-pipelined row streams), the same without
    the pipelining, and the precompiled generic ones."""
    monkeypatch.setenv("BLU_GBY_JIT", jit[0])
    if jit.endswith("nopipe"):
        monkeypatch.setenv("BLU_GBY_PIPE", "0")
        monkeypatch.setenv("BLU_GBY_DENSE_PIPE", "0")
    w, o = oracles(name)
    plan, res = run_gpu(bg, w)
    assert res.n_groups == o.n_groups
    gk, ga = gpu_sorted(res, w.schema)
    assert_parity(gk, ga, o, w.schema)


@pytest.mark.parametrize("name,paths", [("C1", "abd"), ("C2", "abd"), ("C4", "bd"), ("C3", "b")])
@pytest.mark.parametrize("front", ["0", "1"])
def test_forced_paths_identical(bg, oracles, monkeypatch, name, paths, front):
    """Forced path (a) vs (b) vs (b'), hot-key front on/off: all equal the oracle."""
    w, o = oracles(name)
    kc, vc = blugen.device_columns(w)
    monkeypatch.setenv("BLU_GBY_HOT_FRONT", front)
    for p in paths:
        monkeypatch.setenv("BLU_GBY_FORCE_PATH", p)
        plan = bg.plan_for(w.schema, w.est_groups, w.n_rows)
        res = bg.blu_gby_execute(plan, kc, vc)
        gk, ga = gpu_sorted(res, w.schema)
        assert_parity(gk, ga, o, w.schema)


@pytest.mark.parametrize("rank", ["1", "1-hotreg", "0", "1-dedupe", "1-hotreg-dedupe"])
@pytest.mark.parametrize("dicts,n", [((13, 7), 200_003), ((64, 1024), 1_048_583), ((100, 20, 20), 700_001)])
def test_rank_front(bg, monkeypatch, rank, dicts, n):
    """Path (b') hot-key front as a rank image (bitmap + per-word prefix) vs the hash front: both equal
    the oracle. D = 91, D = 32 * S exactly (S = 2048 front entries for this schema), D = 4 * 10^4.
    Skewed keys so the seeded front fills up; rows of cold keys take the global REDs. "hotreg": the
    sample's hottest key summed in per-thread registers (BLU_GBY_HOT_REG=1) for every field kind of
    ALL(3) (i32/i64/f64 SUM, MIN, MAX, COUNT); "dedupe": lanes hitting the same front entry combined
    with __match_any_sync + a shuffle tree before the shared-memory update (BLU_GBY_DEDUPE=1)."""
    monkeypatch.setenv("BLU_GBY_HOT_REG", "1" if "hotreg" in rank else "0")
    monkeypatch.setenv("BLU_GBY_DEDUPE", "1" if "dedupe" in rank else "0")
    rng = np.random.default_rng(sum(dicts) + n)
    D = int(np.prod(dicts))
    sch = blugen.Schema([(I32, d) for d in dicts], [I32, I64, F64], ALL(3))
    r = np.minimum(rng.zipf(1.3, n) - 1, D - 1)          # heavy head, long tail, max code present
    perm = rng.permutation(D)
    g = perm[r]
    g[:3] = [0, D - 1, D // 2]
    kc, rem = [], g
    for d in dicts:
        kc.append((rem % d).astype(np.int32))
        rem = rem // d
    vc = [rng.integers(-(2**31), 2**31, n).astype(np.int32), rng.integers(-(2**62), 2**62, n).astype(np.int64),
          rng.integers(-(2**20), 2**20, n) / 64.0]
    o = oracle.groupby_arrays(sch, kc, vc)
    monkeypatch.setenv("BLU_GBY_FORCE_PATH", "d")
    monkeypatch.setenv("BLU_GBY_HOT_FRONT", "1")
    if rank == "0":
        monkeypatch.setenv("BLU_GBY_NO_RANK_FRONT", "1")
    plan = bg.plan_for(sch, D, n)
    info = plan.info()
    assert info["hot_front"] == 1 and info["path"] == bg.BLU_PATH_DIRECT_GLOBAL
    assert (D + 31) // 32 <= info["front_slots"]
    dk, dv = _mk(kc, vc)
    res = bg.blu_gby_execute(plan, dk, dv)
    gk, ga = gpu_sorted(res, sch)
    assert_parity(gk, ga, o, sch)


@pytest.mark.parametrize("est", [1, 1000, 60_000, 2_000_003])
def test_est_groups_invariance_and_regrow(bg, oracles, est):
    """Under-estimates take the error path: regrow and rerun, same exact result."""
    w, o = oracles("C3")
    plan, res = run_gpu(bg, w, est=est)
    gk, ga = gpu_sorted(res, w.schema)
    assert_parity(gk, ga, o, w.schema)
    if est == 1:
        assert plan.info()["retries_last"] >= 1


def _mk(keys_np, vals_np):
    return [torch.from_numpy(k).cuda() for k in keys_np], [torch.from_numpy(v).cuda() for v in vals_np]


ALL = lambda nv: [(COUNT, -1)] + [(op, c) for c in range(nv) for op in (SUM, MIN, MAX, AVG)]


@pytest.mark.parametrize("seed", [1, 2, 3, 4])
def test_hot_reg_key_outside_front(bg, monkeypatch, seed):
    """Hottest key in registers when the seeded front cannot hold every heavy hitter: a 64-entry rank
    front, 100 keys each far above the sample histogram's top bin, so the front takes 64 of them
    first come and the sample's argmax key may be left out; its register partial then goes straight
    to the dense state instead of a front entry. Either way the result equals the oracle."""
    rng = np.random.default_rng(seed)
    n, D = 2_000_003, 2048
    sch = blugen.Schema([(I32, D)], [I32, I64, F64], ALL(3))
    hot = rng.choice(D, 100, replace=False)
    g = hot[rng.integers(0, 100, n)]
    cold = rng.random(n) < 0.05
    g[cold] = rng.integers(0, D, int(cold.sum()))
    kc = [g.astype(np.int32)]
    vc = [rng.integers(-(2**31), 2**31, n).astype(np.int32), rng.integers(-(2**62), 2**62, n).astype(np.int64),
          rng.integers(-(2**20), 2**20, n) / 64.0]
    o = oracle.groupby_arrays(sch, kc, vc)
    monkeypatch.setenv("BLU_GBY_FORCE_PATH", "d")
    monkeypatch.setenv("BLU_GBY_HOT_FRONT", "1")
    monkeypatch.setenv("BLU_GBY_FRONT_SLOTS", "64")
    monkeypatch.setenv("BLU_GBY_HOT_REG", "1")
    plan = bg.plan_for(sch, D, n)
    info = plan.info()
    assert info["hot_front"] == 1 and info["front_slots"] == 64
    dk, dv = _mk(kc, vc)
    res = bg.blu_gby_execute(plan, dk, dv)
    gk, ga = gpu_sorted(res, sch)
    assert_parity(gk, ga, o, sch)


@pytest.mark.parametrize("mmb", ["2", "1", "0"])
@pytest.mark.parametrize("recipe", ["group-offset", "trend", "late-extremes"])
@pytest.mark.parametrize("path", ["a", "d-rank", "d-rank-hotreg"])
def test_minmax_skip_bounds(bg, monkeypatch, mmb, recipe, path):
    """MIN/MAX skip bounds of the shared-memory tables (BLU_GBY_MMBOUND): a row skips
    the read-before-atomic only when its value cannot beat the largest current MIN (smallest MAX) of
    any live entry. Adversarial value recipes: per-group offsets far apart (the bound is the highest
    group's MIN, so low groups must never be skipped), a monotone trend over the rows (every row is
    a new MIN of its group in one column and a new MAX in another), and the column extremes placed
    in the last 1% of the rows (after the bound has converged). i32 / i64 / f64 (negative values:
    the order-preserving encoding) MIN and MAX, on path (a) and the rank front with and without the
    register-held hottest key; equal to the oracle bit for bit with the bounds off (0), on path (a)
    only (1) and also on the rank front (2)."""
    monkeypatch.setenv("BLU_GBY_MMBOUND", mmb)
    monkeypatch.setenv("BLU_GBY_HOT_REG", "1" if "hotreg" in path else "0")
    rng = np.random.default_rng(len(recipe) * 7 + len(path))
    n = 3_000_017
    D = 1024 if path == "a" else 20_000
    if path == "a":
        g = rng.integers(0, D, n)
    else:
        g = np.minimum(rng.zipf(1.2, n) - 1, D - 1)
        g = rng.permutation(D)[g]
    i = np.arange(n, dtype=np.int64)
    if recipe == "group-offset":
        off = rng.permutation(D).astype(np.int64) * 1_000_000
        v1 = off[g] + rng.integers(0, 1000, n)
    elif recipe == "trend":
        v1 = -i * 3 + rng.integers(0, 2, n)
    else:
        v1 = rng.integers(-10**6, 10**6, n)
        late = rng.random(n) < 0.01
        late[: n * 99 // 100] = False
        v1[late] = rng.choice([-(10**9), 10**9], int(late.sum())) + rng.integers(-5, 5, int(late.sum()))
    v0 = np.clip(v1 // 1000, -(2**31), 2**31 - 1).astype(np.int32)
    if recipe == "trend":
        v0 = (i // 3 - 2**20).astype(np.int32)  # rising: every row a new MAX of its group
    v2 = (v1 % (2**20) - 2**19) / 64.0 - (i if recipe == "trend" else 0) / 2.0
    sch = blugen.Schema([(I32, D)], [I32, I64, F64], ALL(3))
    kc = [g.astype(np.int32)]
    vc = [v0, v1.astype(np.int64), v2]
    o = oracle.groupby_arrays(sch, kc, vc)
    if path == "a":
        monkeypatch.setenv("BLU_GBY_FORCE_PATH", "a")
        monkeypatch.setenv("BLU_GBY_NO_FUSE", "1")
    else:
        monkeypatch.setenv("BLU_GBY_FORCE_PATH", "d")
        monkeypatch.setenv("BLU_GBY_HOT_FRONT", "1")
    plan = bg.plan_for(sch, D, n)
    if path != "a":
        assert plan.info()["hot_front"] == 1
    dk, dv = _mk(kc, vc)
    res = bg.blu_gby_execute(plan, dk, dv)
    gk, ga = gpu_sorted(res, sch)
    assert_parity(gk, ga, o, sch)


@pytest.mark.parametrize("n", [0, 1, 3, 31, 33, 4095, 4097, 65_537])
@pytest.mark.parametrize("path", ["a", "a-nofuse", "b", "d"])
def test_small_and_ragged(bg, monkeypatch, n, path):
    """Tiny and ragged sizes on every path; "a-nofuse" takes the unfused, software-pipelined dense
    kernel (the one large inputs use) instead of the fused small-input one."""
    if path == "a-nofuse":
        monkeypatch.setenv("BLU_GBY_NO_FUSE", "1")
        path = "a"
    rng = np.random.default_rng(n + 7)
    sch = blugen.Schema([(I32, 13), (I64, 7)], [I32, I64, F64], ALL(3))
    kc = [rng.integers(0, 13, n).astype(np.int32), rng.integers(0, 7, n).astype(np.int64)]
    vc = [rng.integers(-(2**31), 2**31, n).astype(np.int32), rng.integers(-(2**62), 2**62, n).astype(np.int64),
          rng.integers(-(2**20), 2**20, n) / 64.0]
    o = oracle.groupby_arrays(sch, kc, vc)
    monkeypatch.setenv("BLU_GBY_FORCE_PATH", path)
    plan = bg.plan_for(sch, 91, n)
    dk, dv = _mk(kc, vc)
    res = bg.blu_gby_execute(plan, dk, dv, n_rows=n)
    gk, ga = gpu_sorted(res, sch)
    assert_parity(gk, ga, o, sch)


def test_single_group_and_all_distinct(bg):
    n = 300_001
    rng = np.random.default_rng(1)
    sch = blugen.Schema([(I64, 0)], [I64, F64, I32], ALL(3))
    v = [rng.integers(-(2**40), 2**40, n), rng.integers(-(2**20), 2**20, n) / 64.0,
         rng.integers(-(2**31), 2**31, n).astype(np.int32)]
    for kc in ([np.full(n, 12345, np.int64)], [rng.permutation(10**7)[:n].astype(np.int64)]):
        o = oracle.groupby_arrays(sch, kc, v)
        dk, dv = _mk(kc, v)
        plan = bg.plan_for(sch, 1 if kc[0][0] == kc[0][1] else n, n)
        res = bg.blu_gby_execute(plan, dk, dv)
        gk, ga = gpu_sorted(res, sch)
        assert_parity(gk, ga, o, sch)


def test_key_range_errors(bg):
    sch = blugen.Schema([(I32, 10)], [I64], [(SUM, 0)])
    plan = bg.plan_for(sch, 10, 1000)
    k = torch.arange(1000, dtype=torch.int32, device="cuda") % 10
    v = torch.ones(1000, dtype=torch.int64, device="cuda")
    for bad in (10, -1):
        k2 = k.clone()
        k2[777] = bad
        with pytest.raises(bg.BluError) as e:
            bg.blu_gby_execute(plan, [k2], [v])
        assert e.value.status == bg.BLU_E_KEY_RANGE
    sp = bg.plan_for(blugen.Schema([(I64, 0)], [I64], [(SUM, 0)]), 10, 1000)
    ks = torch.arange(1000, dtype=torch.int64, device="cuda")
    ks[5] = -3
    with pytest.raises(bg.BluError) as e:
        bg.blu_gby_execute(sp, [ks], [v])
    assert e.value.status == bg.BLU_E_KEY_RANGE
    # the valid maximum code dict_size - 1 is accepted
    k3 = k.clone()
    k3[:] = 9
    r = bg.blu_gby_execute(plan, [k3], [v])
    assert r.n_groups == 1 and int(r.aggs[0][0]) == 1000


@pytest.mark.parametrize("path,front", [("a", "0"), ("d", "1"), ("d", "0"), ("b", "0")])
def test_key_range_errors_large(bg, monkeypatch, path, front):
    """Out-of-range codes caught by the software-pipelined kernels (tile_unpack) at sizes that take
    the unfused, multi-tile launch; the bad row is the last one (ragged tail) or deep inside."""
    monkeypatch.setenv("BLU_GBY_NO_FUSE", "1")  # path (a): the pipelined kernel, not the fused one
    n = 5_000_011
    sch = blugen.Schema([(I32, 30), (I32, 40)], [I64], [(COUNT, -1), (SUM, 0)])
    monkeypatch.setenv("BLU_GBY_FORCE_PATH", path)
    monkeypatch.setenv("BLU_GBY_HOT_FRONT", front)
    plan = bg.plan_for(sch, 1200, n)
    k0 = torch.arange(n, dtype=torch.int64, device="cuda").remainder(30).to(torch.int32)
    k1 = torch.arange(n, dtype=torch.int64, device="cuda").remainder(37).to(torch.int32)
    v = torch.ones(n, dtype=torch.int64, device="cuda")
    for col, pos, bad in ((0, n - 1, 30), (1, 3_333_333, -1), (1, 0, 40)):
        ks = [k0.clone(), k1.clone()]
        ks[col][pos] = bad
        with pytest.raises(bg.BluError) as e:
            bg.blu_gby_execute(plan, ks, [v])
        assert e.value.status == bg.BLU_E_KEY_RANGE
    r = bg.blu_gby_execute(plan, [k0, k1], [v])
    assert r.n_groups == 30 * 37 and int(r.aggs[0].sum()) == n and int(r.aggs[1].sum()) == n


def test_general_f64_within_tolerance(bg):
    """Non-dyadic doubles: SUM/AVG within 1e-12 * sum|v| of the oracle (reading A13)."""
    n = 1_000_003
    w = blugen.Workload("real", n, 77, [blugen.Col(I32, blugen.UNIFORM, 0, 0, 500)],
                        [blugen.Col(F64, REAL, 1, lo=10**6)],
                        blugen.Schema([(I32, 500)], [F64], [(COUNT, -1), (SUM, 0), (AVG, 0), (MIN, 0), (MAX, 0)]),
                        500, 500)
    o = oracle.groupby_generated(w)
    for p in "ab":
        os.environ["BLU_GBY_FORCE_PATH"] = p
        try:
            plan, res = run_gpu(bg, w)
        finally:
            del os.environ["BLU_GBY_FORCE_PATH"]
        gk, ga = gpu_sorted(res, w.schema)
        assert_parity(gk, ga, o, w.schema, f64_tol=1e-12)


def test_misaligned_columns_scalar_path(bg, oracles):
    w, _ = oracles("C2")
    kc, vc = blugen.device_columns(w)
    # drop the first row: every column pointer is 4 or 8 bytes past a 16-byte boundary
    kc1, vc1 = [k[1:] for k in kc], [v[1:] for v in vc]
    hk, hv = blugen.host_columns(w)
    o = oracle.groupby_arrays(w.schema, [k[1:] for k in hk], [v[1:] for v in hv])
    plan = bg.plan_for(w.schema, w.est_groups, w.n_rows - 1)
    res = bg.blu_gby_execute(plan, kc1, vc1)
    gk, ga = gpu_sorted(res, w.schema)
    assert_parity(gk, ga, o, w.schema)


@pytest.mark.parametrize("name", ["C2", "C3", "C4"])
def test_partial_merge_equals_full(bg, oracles, name):
    """S9: execute_partial on 3 row shards, then merge (P:68 range partitions merged at the end)."""
    w, o = oracles(name)
    kc, vc = blugen.device_columns(w)
    plan = bg.plan_for(w.schema, w.est_groups, w.n_rows)
    cuts = [0, w.n_rows // 3 + 1, 2 * w.n_rows // 3 + 5, w.n_rows]
    parts = [bg.blu_gby_execute_partial(plan, [k[a:b] for k in kc], [v[a:b] for v in vc])
             for a, b in zip(cuts[:-1], cuts[1:])]
    res = bg.blu_gby_merge(plan, parts)
    gk, ga = gpu_sorted(res, w.schema)
    assert_parity(gk, ga, o, w.schema)
    # merge_partial then merge again is still exact
    mp = bg.blu_gby_merge_partial(plan, parts[:2])
    res2 = bg.blu_gby_merge(plan, [mp, parts[2]])
    gk, ga = gpu_sorted(res2, w.schema)
    assert_parity(gk, ga, o, w.schema)


@pytest.mark.parametrize("name", ["C3", "C2"])
def test_partition_records_exchange(bg, oracles, name):
    """S10 simulated on one GPU: each of P 'ranks' partitions its partial by owner; each owner merges
    the records it would receive. The union of owners' results equals the full result."""
    w, o = oracles(name)
    kc, vc = blugen.device_columns(w)
    plan = bg.plan_for(w.schema, w.est_groups, w.n_rows)
    P = 4
    cuts = np.linspace(0, w.n_rows, P + 1).astype(int)
    rb = plan.record_bytes
    inbox = [[] for _ in range(P)]
    for r in range(P):
        part = bg.blu_gby_execute_partial(plan, [k[cuts[r]:cuts[r + 1]] for k in kc],
                                          [v[cuts[r]:cuts[r + 1]] for v in vc])
        buf = torch.empty(max(1, part.n_groups) * rb // 8, dtype=torch.int64, device="cuda")
        counts = bg.blu_gby_partition(plan, part, P, buf)
        assert sum(counts) == part.n_groups
        off = 0
        for dst in range(P):
            inbox[dst].append(buf[off * rb // 8:(off + counts[dst]) * rb // 8])
            off += counts[dst]
    keys, aggs = [], []
    for dst in range(P):
        recs = torch.cat(inbox[dst])
        res = bg.blu_gby_merge_records(plan, recs, recs.numel() * 8 // rb)
        gk, ga = gpu_sorted(res, w.schema)
        keys.append(gk)
        aggs.append(ga)
    allk = np.concatenate(keys)
    order = np.lexsort(allk.T[::-1])
    assert_parity(allk[order], [np.concatenate([a[i] for a in aggs])[order] for i in range(len(w.schema.aggs))],
                  o, w.schema)


def _owner_np(keys: np.ndarray, P: int) -> np.ndarray:
    """S2 owner = mulhi(fmix64(key), P), uint64 arithmetic in numpy."""
    h = keys.astype(np.uint64)
    with np.errstate(over="ignore"):
        h ^= h >> np.uint64(33)
        h *= np.uint64(0xff51afd7ed558ccd)
        h ^= h >> np.uint64(33)
        h *= np.uint64(0xc4ceb9fe1a85ec53)
        h ^= h >> np.uint64(33)
    a = (h >> np.uint64(32)) * np.uint64(P)
    b = ((h & np.uint64(0xFFFFFFFF)) * np.uint64(P)) >> np.uint64(32)
    return ((a + b) >> np.uint64(32)).astype(np.int64)


@pytest.mark.parametrize("n", [1, 4097, 1_000_003])
@pytest.mark.parametrize("P", [1, 3, 8, 1024])
def test_partition_rows_layout(bg, n, P):
    """S10 owner partition (count / scan / scatter kernels): the send buffer holds owner 0's records,
    then owner 1's, ...; every record lands in its key's owner bucket (owner computed here in numpy),
    the counts match, and the records are exactly the input rows (as a multiset)."""
    rng = np.random.default_rng(n + P)
    sch = blugen.Schema([(I64, 0)], [I64, F64], [(COUNT, -1), (SUM, 0), (AVG, 1)])
    k = rng.integers(0, 2**62, n).astype(np.int64)
    v = [rng.integers(-(2**40), 2**40, n), rng.integers(-(2**20), 2**20, n) / 64.0]
    plan = bg.plan_for(sch, n, n)
    words = plan.row_record_bytes // 8
    assert words == 3
    dk, dv = _mk([k], v)
    send = torch.empty(n * words, dtype=torch.int64, device="cuda")
    counts = bg.blu_gby_partition_rows(plan, dk, dv, P, send)
    assert len(counts) == P and sum(counts) == n
    own = _owner_np(k, P)
    assert np.array_equal(np.bincount(own, minlength=P), np.array(counts))
    recs = send.cpu().numpy().reshape(n, words)
    starts = np.concatenate([[0], np.cumsum(counts)])
    for o in range(P):
        assert np.all(_owner_np(recs[starts[o]:starts[o + 1], 0], P) == o)
    got = recs[np.lexsort(recs.T[::-1])]
    exp = np.stack([k, v[0], v[1].view(np.int64)], axis=1)
    assert np.array_equal(got, exp[np.lexsort(exp.T[::-1])])


@pytest.mark.parametrize("name", ["C1", "C2", "C4"])
def test_dense_state_accumulate_and_finalize(bg, oracles, name):
    """Path (a)/(b') multi-GPU helpers on one GPU: 3 shards accumulate into one dense state."""
    w, o = oracles(name)
    kc, vc = blugen.device_columns(w)
    plan = bg.plan_for(w.schema, w.est_groups, w.n_rows)
    st = bg.dense_state_arrays(plan)
    cuts = [0, 1000, w.n_rows // 2, w.n_rows]
    for i, (a, b) in enumerate(zip(cuts[:-1], cuts[1:])):
        bg.blu_gby_execute_dense_state(plan, [k[a:b] for k in kc], [v[a:b] for v in vc], st, init=(i == 0))
    res = bg.blu_gby_finalize_dense_state(plan, st)
    gk, ga = gpu_sorted(res, w.schema)
    assert_parity(gk, ga, o, w.schema)


@pytest.mark.parametrize("name", ["C1", "C3", "C3-parts"])
def test_execute_host_columns(bg, oracles, monkeypatch, name):
    """Host columns in, host result out (pinned result blocks, reused after the result is released):
    chunked H2D overlapped with aggregation (C1, C3 one pass), or — for a partitioned plan — the whole
    input copied to the device and run through the scatter + pass 2 ('C3-parts'). Twice, so the second
    call reuses the first result's pinned blocks."""
    w, o = oracles(name.split("-")[0])
    if name.endswith("parts"):
        monkeypatch.setenv("BLU_GBY_PARTS", "16")
    hk, hv = blugen.host_columns(w)
    hk = [torch.from_numpy(k).pin_memory() for k in hk]
    hv = [torch.from_numpy(v).pin_memory() for v in hv]
    plan = bg.plan_for(w.schema, w.est_groups, w.n_rows)
    if name.endswith("parts"):
        assert plan.info()["partitions"] == 16
    for _ in range(2):
        res = bg.blu_gby_execute_host(plan, hk, hv)
        gk, ga = host_sorted(res, w.schema)
        assert_parity(gk, ga, o, w.schema)
        del res


def test_concurrent_executes_on_streams(bg, oracles, monkeypatch):
    """The header's concurrency promise: host threads running whole queries at the same time on their
    own streams — host-column queries (partitioned plan: staging, two-level scatter with its second
    stream, pinned result blocks) next to device-column queries — each equal to the oracle."""
    import threading
    w3, o3 = oracles("C3")
    w5, o5 = oracles("C5")
    monkeypatch.setenv("BLU_GBY_PARTS", "256")
    monkeypatch.setenv("BLU_GBY_PART_SMEM", "1")
    plan3 = bg.plan_for(w3.schema, w3.est_groups, w3.n_rows)
    assert plan3.info()["partitions"] == 256 and plan3.info()["part_smem"] == 1
    monkeypatch.delenv("BLU_GBY_PARTS")
    monkeypatch.delenv("BLU_GBY_PART_SMEM")
    plan5 = bg.plan_for(w5.schema, w5.est_groups, w5.n_rows)
    hk, hv = blugen.host_columns(w3)
    hk = [torch.from_numpy(k).pin_memory() for k in hk]
    hv = [torch.from_numpy(v).pin_memory() for v in hv]
    kc5, vc5 = blugen.device_columns(w5)
    torch.cuda.synchronize()
    errors = []

    def host_worker():
        try:
            s = torch.cuda.Stream()
            for _ in range(3):
                res = bg.blu_gby_execute_host(plan3, hk, hv, stream=s)
                gk, ga = host_sorted(res, w3.schema)
                assert_parity(gk, ga, o3, w3.schema)
                del res
        except Exception as e:  # noqa: BLE001 - reported below
            errors.append(e)

    def device_worker():
        try:
            s = torch.cuda.Stream()
            for _ in range(3):
                with torch.cuda.stream(s):
                    res = bg.blu_gby_execute(plan5, kc5, vc5, stream=s)
                    gk, ga = gpu_sorted(res, w5.schema)
                assert_parity(gk, ga, o5, w5.schema)
                del res
        except Exception as e:  # noqa: BLE001
            errors.append(e)

    ts = [threading.Thread(target=host_worker), threading.Thread(target=host_worker),
          threading.Thread(target=device_worker)]
    for t in ts:
        t.start()
    for t in ts:
        t.join()
    assert not errors, errors


def test_init_table_matches_table1(bg):
    """S4 on the device: every slot equals the Table 1 mask."""
    plan = bg.blu_gby_plan([(I64, 0)], [I64, I64, I32], [(SUM, 0), (MAX, 1), (MIN, 2)], 1000, 10**6)
    t = plan.slot_template()
    n = 4099
    buf = torch.zeros(n * len(t), dtype=torch.uint8, device="cuda")
    bg.blu_gby_init_table(plan, buf, n)
    torch.cuda.synchronize()
    got = buf.cpu().numpy().reshape(n, len(t))
    want = np.frombuffer(t, np.uint8)
    assert np.all(got == want[None, :])
    assert t[:8] == b"\xff" * 8 and int.from_bytes(t[16:24], "little", signed=True) == -(2**63)
    assert int.from_bytes(t[24:28], "little", signed=True) == 2**31 - 1


def test_cross_check_against_torch_library(bg):
    """Second reference independent of both libblugby and the oracle: torch.unique + scatter_reduce."""
    w = blugen.workload("C2", n_rows=20_000_000)
    kc, vc = blugen.device_columns(w)
    plan = bg.plan_for(w.schema, w.est_groups, w.n_rows)
    res = bg.blu_gby_execute(plan, kc, vc)
    packed = kc[0].long() + 32 * kc[1].long()
    uq, inv, cnt = torch.unique(packed, return_inverse=True, return_counts=True)
    G = uq.numel()
    s0 = torch.zeros(G, dtype=torch.int64, device="cuda").scatter_add_(0, inv, vc[0].long())
    mn = torch.full((G,), 2**62, dtype=torch.int64, device="cuda").scatter_reduce_(0, inv, vc[1], "amin")
    mx = torch.full((G,), -(2**62), dtype=torch.int64, device="cuda").scatter_reduce_(0, inv, vc[2], "amax")
    s3 = torch.zeros(G, dtype=torch.float64, device="cuda").scatter_add_(0, inv, vc[3])
    gp = res.keys[0].long() + 32 * res.keys[1].long()
    order = torch.argsort(gp)
    assert res.n_groups == G and torch.equal(gp[order], uq)
    assert torch.equal(res.aggs[0][order], cnt)
    assert torch.equal(res.aggs[1][order], s0)
    assert torch.equal(res.aggs[2][order], mn) and torch.equal(res.aggs[3][order], mx)
    assert torch.equal(res.aggs[4][order], s3 / cnt.double())


def test_launch_count_and_timing(bg):
    w = blugen.workload("C1", n_rows=100_000)
    kc, vc = blugen.device_columns(w)
    plan = bg.plan_for(w.schema, 16, w.n_rows)
    bg.blu_gby_set_timing(True)
    c0 = bg.blu_gby_launch_count()
    bg.blu_gby_execute(plan, kc, vc)
    c1 = bg.blu_gby_launch_count()
    t = bg.blu_gby_last_timing()
    bg.blu_gby_set_timing(False)
    assert c1 - c0 >= 1  # path (a): init and compaction fused into the one aggregation launch
    assert t["aggregate_ms"] > 0 and t["aggregate_launches"] == 1 and t["kernel"]
    assert t["kernel"].startswith("blu_jit_dense"), t["kernel"]  # the plan-specialised kernel ran
    os.environ["BLU_GBY_NO_FUSE"] = "1"
    try:
        c0 = bg.blu_gby_launch_count()
        r = bg.blu_gby_execute(plan, kc, vc)
        assert bg.blu_gby_launch_count() - c0 == 3  # init (+flags), aggregate, one-CTA compaction
        assert r.n_groups == 16
    finally:
        del os.environ["BLU_GBY_NO_FUSE"]


@pytest.mark.parametrize("smem", ["1", "0"])
@pytest.mark.parametrize("parts,chunk,div", [("8", None, None), ("16", "300000", None), ("64", "1000003", None),
                                             ("2", None, None), ("256", None, "7"), ("128", "700001", "64"),
                                             ("32", None, "2")])
def test_partitioned_two_pass(bg, oracles, monkeypatch, parts, chunk, div, smem):
    """Path (b) partitioned mode: scatter into buckets by slot bits, then bucket-by-bucket
    aggregation — in per-CTA shared-memory bucket tables merged once per piece (smem=1; with 2
    buckets most groups find no room and take the global path inside the same kernel; div cuts
    buckets into many pieces, so one bucket is merged from several CTAs) or directly into the
    bucket's L2-resident table slice (smem=0); several chunks; identical to the oracle."""
    w, o = oracles("C3")
    kc, vc = blugen.device_columns(w)
    monkeypatch.setenv("BLU_GBY_PARTS", parts)
    monkeypatch.setenv("BLU_GBY_PART_SMEM", smem)
    if chunk:
        monkeypatch.setenv("BLU_GBY_PART_CHUNK", chunk)
    if div:
        monkeypatch.setenv("BLU_GBY_PIECE_DIV", div)
    plan = bg.plan_for(w.schema, w.est_groups, w.n_rows)
    info = plan.info()
    assert info["partitions"] == int(parts) and info["part_smem"] == int(smem), info
    bg.blu_gby_set_timing(True)
    res = bg.blu_gby_execute(plan, kc, vc)
    t = bg.blu_gby_last_timing()
    bg.blu_gby_set_timing(False)
    assert t["part_chunks"] >= 1 and t["scatter_ms"] > 0 and t["pass2_ms"] > 0, t
    assert t["part_fallbacks"] == 0, t  # pass 2 ran (no bucket overflowed)
    gk, ga = gpu_sorted(res, w.schema)
    assert_parity(gk, ga, o, w.schema)


@pytest.mark.parametrize("tma", ["1", "0"])
@pytest.mark.parametrize("shape", [("C3", 3_000_017, 200_000, None), ("C3", 2_000_003, 30_000, "1"),
                                   ("C5", 4_000_037, 400_000, None)])
def test_scatter_tma_write_out(bg, monkeypatch, tma, shape):
    """Partitioned path (b) with the scatter's staged bucket runs leaving shared memory by TMA bulk
    copies (cp.async.bulk, runs padded to even lengths with empty-key records that pass 2 and the second
    scatter level skip) and with the per-element write-out: both equal the oracle, one level (L2-slice
    pass 2) and two levels (shared-memory bucket tables)."""
    name, n, G, smem = shape
    w = blugen.workload(name, n_rows=n, n_groups=G)
    o = oracle.groupby_generated(w)
    kc, vc = blugen.device_columns(w)
    monkeypatch.setenv("BLU_GBY_SCATTER_TMA", tma)
    monkeypatch.setenv("BLU_GBY_PARTS", "256" if smem else "64")
    if smem:
        monkeypatch.setenv("BLU_GBY_PART_SMEM", "1")
    plan = bg.plan_for(w.schema, w.est_groups, w.n_rows)
    assert plan.info()["partitions"] > 1
    bg.blu_gby_set_timing(True)
    res = bg.blu_gby_execute(plan, kc, vc)
    t = bg.blu_gby_last_timing()
    bg.blu_gby_set_timing(False)
    assert t["part_chunks"] >= 1 and t["part_fallbacks"] == 0, t
    gk, ga = gpu_sorted(res, w.schema)
    assert_parity(gk, ga, o, w.schema)


@pytest.mark.parametrize("n,parts,chunk", [(4097, "2", None), (65_537, "16", "8192"), (1_000_003, "64", "300001"),
                                          (300_007, "256", "65536")])
def test_scatter_tma_edges(bg, monkeypatch, n, parts, chunk):
    """TMA write-out edge cases: ragged sizes, 2 to 256 buckets, several chunks (padding records in every
    chunk's partition buffers), the smallest inputs the partitioned mode accepts; equal to the oracle."""
    w = blugen.workload("C5", n_rows=n, n_groups=max(16, n // 50))
    o = oracle.groupby_generated(w)
    kc, vc = blugen.device_columns(w)
    monkeypatch.setenv("BLU_GBY_SCATTER_TMA", "1")
    monkeypatch.setenv("BLU_GBY_PARTS", parts)
    if chunk:
        monkeypatch.setenv("BLU_GBY_PART_CHUNK", chunk)
    plan = bg.plan_for(w.schema, w.est_groups, w.n_rows)
    bg.blu_gby_set_timing(True)
    res = bg.blu_gby_execute(plan, kc, vc)
    t = bg.blu_gby_last_timing()
    bg.blu_gby_set_timing(False)
    if n >= 4096 * int(parts):
        assert t["part_chunks"] >= 1 and t["part_fallbacks"] == 0, t
    gk, ga = gpu_sorted(res, w.schema)
    assert_parity(gk, ga, o, w.schema)


def test_host_results_pinned_reuse(bg, oracles):
    """Host results of different sizes one after another, some kept alive while others are freed: each
    takes its own pinned blocks from the cache (never one still referenced) and stays intact."""
    held = []
    for name, n in (("C3", 400_003), ("C1", 10_007), ("C3", 900_001), ("C2", 50_001)):
        w = blugen.workload(name, n_rows=n)
        o = oracle.groupby_generated(w)
        hk, hv = blugen.host_columns(w)
        plan = bg.plan_for(w.schema, w.est_groups, w.n_rows)
        res = bg.blu_gby_execute_host(plan, [torch.from_numpy(k).pin_memory() for k in hk],
                                      [torch.from_numpy(v).pin_memory() for v in hv])
        held.append((res, o, w.schema))
        if len(held) == 3:
            held.pop(0)  # free one result while two stay alive
    for res, o, sch in held:
        gk, ga = host_sorted(res, sch)
        assert_parity(gk, ga, o, sch)


@pytest.mark.parametrize("parts", ["1024", "4096"])
def test_partitioned_l2_mode_max_buckets(bg, monkeypatch, parts):
    """The L2-slice pass 2 at its bucket limit (kMaxSegs = 1024): forced 1024 buckets, and a forced
    4096 clamped to 1024 by the planner (2048 once overran the pass's shared prefix array)."""
    w = blugen.workload("C3", n_rows=5_000_011, n_groups=300_000)
    o = oracle.groupby_generated(w)
    kc, vc = blugen.device_columns(w)
    monkeypatch.setenv("BLU_GBY_PART_SMEM", "0")
    monkeypatch.setenv("BLU_GBY_PARTS", parts)
    plan = bg.plan_for(w.schema, w.est_groups, w.n_rows)
    info = plan.info()
    assert info["part_smem"] == 0 and info["partitions"] == 1024, info
    bg.blu_gby_set_timing(True)
    res = bg.blu_gby_execute(plan, kc, vc)
    t = bg.blu_gby_last_timing()
    bg.blu_gby_set_timing(False)
    assert t["part_chunks"] == 1, t
    gk, ga = gpu_sorted(res, w.schema)
    assert_parity(gk, ga, o, w.schema)


@pytest.mark.parametrize("one", ["0", "1"])
def test_partitioned_two_level_128(bg, monkeypatch, one):
    """More than 4096 bucket tables: the two-level scatter splits 128 x B/128 (8192 buckets = 128 x 64
    here; C5's forced shared-memory mode is 128 x 128), per-bucket second-level launches or one
    segmented launch; 40M rows into 4M groups, against the oracle."""
    w = blugen.workload("C3", n_rows=40_000_003, n_groups=4_000_000)
    o = oracle.groupby_generated(w)
    kc, vc = blugen.device_columns(w)
    monkeypatch.setenv("BLU_GBY_PART_SMEM", "1")
    monkeypatch.setenv("BLU_GBY_PARTS", "8192")
    monkeypatch.setenv("BLU_GBY_2LEVEL_ONE", one)
    plan = bg.plan_for(w.schema, w.est_groups, w.n_rows)
    info = plan.info()
    assert info["part_smem"] == 1 and info["partitions"] == 8192, info
    bg.blu_gby_set_timing(True)
    res = bg.blu_gby_execute(plan, kc, vc)
    t = bg.blu_gby_last_timing()
    bg.blu_gby_set_timing(False)
    assert t["part_chunks"] == 1 and t["part_fallbacks"] == 0, t
    gk, ga = gpu_sorted(res, w.schema)
    assert_parity(gk, ga, o, w.schema)


@pytest.mark.parametrize("two_level", ["0", "1", "1-one"])
@pytest.mark.parametrize("parts", [None, "4096"])
def test_partitioned_wide_fanout(bg, monkeypatch, parts, two_level):
    """Shared-memory bucket tables as planned for 2M groups (several hundred buckets, the 1024-thread
    wide scatter) and with a forced 4096-way scatter, at 20M rows, against the oracle; in one B-way
    scatter or in two levels (32 first-level buckets, each scattered again into B / 32: one launch per
    first-level bucket, or '1-one': all of them in one launch over the segmented first-level output)."""
    w = blugen.workload("C3", n_rows=20_000_003, n_groups=2_000_000)
    o = oracle.groupby_generated(w)
    kc, vc = blugen.device_columns(w)
    monkeypatch.setenv("BLU_GBY_PART_SMEM", "1")
    monkeypatch.setenv("BLU_GBY_PART_2LEVEL", two_level[0])
    monkeypatch.setenv("BLU_GBY_2LEVEL_ONE", "1" if two_level.endswith("one") else "0")
    if parts:
        monkeypatch.setenv("BLU_GBY_PARTS", parts)
    plan = bg.plan_for(w.schema, w.est_groups, w.n_rows)
    info = plan.info()
    assert info["part_smem"] == 1 and info["partitions"] >= 256, info
    bg.blu_gby_set_timing(True)
    res = bg.blu_gby_execute(plan, kc, vc)
    t = bg.blu_gby_last_timing()
    bg.blu_gby_set_timing(False)
    assert t["part_chunks"] == 1 and t["part_fallbacks"] == 0, t
    gk, ga = gpu_sorted(res, w.schema)
    assert_parity(gk, ga, o, w.schema)


@pytest.mark.parametrize("smem", ["1", "0", "2level"])
def test_partitioned_skew_falls_back(bg, monkeypatch, smem):
    """A bucket overflow (every row in one bucket) takes the device-side fallback: still exact; with the
    two-level scatter the first level overflows and the second level sees truncated buckets (the
    partitioned path needs >= 4096 rows per bucket: 512 buckets -> 2.2M rows)."""
    n = 2_200_000 if smem == "2level" else 600_000
    rng = np.random.default_rng(3)
    sch = blugen.Schema([(I64, 0)], [I64, F64], [(COUNT, -1), (SUM, 0), (AVG, 1), (MIN, 0), (MAX, 1)])
    k = np.where(rng.random(n) < 0.9, 77, rng.integers(0, 5000, n)).astype(np.int64)
    v = [rng.integers(-(2**40), 2**40, n), rng.integers(-(2**20), 2**20, n) / 64.0]
    o = oracle.groupby_arrays(sch, [k], v)
    monkeypatch.setenv("BLU_GBY_PARTS", "512" if smem == "2level" else "16")
    monkeypatch.setenv("BLU_GBY_PART_SMEM", "1" if smem == "2level" else smem)
    dk, dv = _mk([k], v)
    plan = bg.plan_for(sch, 5000, n)
    bg.blu_gby_set_timing(True)
    res = bg.blu_gby_execute(plan, dk, dv)
    t = bg.blu_gby_last_timing()
    bg.blu_gby_set_timing(False)
    assert t["part_fallbacks"] == t["part_chunks"] == 1, t
    gk, ga = gpu_sorted(res, sch)
    assert_parity(gk, ga, o, sch)


@pytest.mark.parametrize("smem", ["1", "0", "2level"])
def test_partitioned_with_regrow(bg, oracles, monkeypatch, smem):
    w, o = oracles("C5")
    kc, vc = blugen.device_columns(w)
    monkeypatch.setenv("BLU_GBY_PARTS", "4" if smem != "2level" else "512")
    monkeypatch.setenv("BLU_GBY_PART_SMEM", "1" if smem == "2level" else smem)
    monkeypatch.setenv("BLU_GBY_PART_2LEVEL", "1" if smem == "2level" else "0")
    plan = bg.plan_for(w.schema, 1000, w.n_rows)  # under-estimate: partitioned + regrow
    res = bg.blu_gby_execute(plan, kc, vc)
    gk, ga = gpu_sorted(res, w.schema)
    assert_parity(gk, ga, o, w.schema)


@pytest.mark.parametrize("name", ["C3", "C2", "C4"])
def test_partition_rows_exchange(bg, oracles, name):
    """S10 rows mode simulated on one GPU: each of P 'ranks' buckets its raw rows
    by owner (blu_gby_partition_rows); each owner aggregates the row records it would receive
    (blu_gby_execute_records). The union of the owners' results equals the full result — sparse
    keys (C3) and dense composite keys (C2, C4: mixed-radix packed keys unpacked by the owner)."""
    w, o = oracles(name)
    kc, vc = blugen.device_columns(w)
    plan = bg.plan_for(w.schema, w.est_groups, w.n_rows)
    P = 4
    cuts = np.linspace(0, w.n_rows, P + 1).astype(int)
    rb = plan.row_record_bytes
    assert rb == 8 * (1 + len(w.schema.vals))
    inbox = [[] for _ in range(P)]
    for r in range(P):
        n = int(cuts[r + 1] - cuts[r])
        buf = torch.empty(max(1, n) * rb // 8, dtype=torch.int64, device="cuda")
        counts = bg.blu_gby_partition_rows(plan, [k[cuts[r]:cuts[r + 1]] for k in kc],
                                           [v[cuts[r]:cuts[r + 1]] for v in vc], P, buf)
        assert sum(counts) == n
        off = 0
        for dst in range(P):
            inbox[dst].append(buf[off * rb // 8:(off + counts[dst]) * rb // 8])
            off += counts[dst]
    keys, aggs = [], []
    for dst in range(P):
        recs = torch.cat(inbox[dst])
        res = bg.blu_gby_execute_records(plan, recs, recs.numel() * 8 // rb)
        gk, ga = gpu_sorted(res, w.schema)
        keys.append(gk)
        aggs.append(ga)
    allk = np.concatenate(keys)
    order = np.lexsort(allk.T[::-1])
    assert_parity(allk[order], [np.concatenate([a[i] for a in aggs])[order] for i in range(len(w.schema.aggs))],
                  o, w.schema)


def test_partition_rows_key_range(bg):
    sch = blugen.Schema([(I32, 10)], [I64], [(COUNT, -1), (SUM, 0)])
    k = np.array([1, 2, 10, 3], np.int32)  # 10 is outside the dictionary
    dk, dv = _mk([k], [np.arange(4, dtype=np.int64)])
    plan = bg.plan_for(sch, 4, 4)
    buf = torch.empty(16 * 4, dtype=torch.int64, device="cuda")
    with pytest.raises(bg.BluError) as e:
        bg.blu_gby_partition_rows(plan, dk, dv, 2, buf)
    assert e.value.status == bg.BLU_E_KEY_RANGE


@pytest.mark.parametrize("G,n,k", [(700, 200_000, 2048), (50_000, 3_000_000, 2048), (1_000_000, 4_000_000, 1024)])
def test_kmv_estimate(bg, G, n, k):
    """NEXT-3: on-GPU KMV estimate equals the numpy statement of the same definition,
    is exact below k distinct keys, and lands within 5 standard errors of the true count."""
    w = blugen.workload("C3", n_rows=n, n_groups=G)
    kc, _ = blugen.device_columns(w)
    est, exact = bg.blu_gby_estimate_groups(w.schema.keys, kc, k=k)
    host = kc[0].cpu().numpy()
    ref, ref_exact = oracle.kmv([host], [0], k)  # oracle/kmv_oracle.cpp: the plain definition
    true = len(np.unique(host))
    assert exact == ref_exact and est == ref
    if exact:
        assert est == true
    else:
        assert abs(est - true) <= 5 * true / np.sqrt(k - 2)
    # order invariance: the same key set in a different row order gives the same estimate
    perm = torch.randperm(n, device="cuda")
    est2, _ = bg.blu_gby_estimate_groups(w.schema.keys, [kc[0][perm].contiguous()], k=k)
    assert est2 == est


def test_kmv_dense_composite_keys(bg):
    w = blugen.workload("C4", n_rows=2_000_000)
    kc, _ = blugen.device_columns(w)
    est, exact = bg.blu_gby_estimate_groups(w.schema.keys, kc, k=2048)
    packed = kc[0].long() + 100 * kc[1].long() + 5000 * kc[2].long()
    ref, ref_exact = oracle.kmv([c.cpu().numpy() for c in kc], [d for _, d in w.schema.keys], 2048)
    assert est == ref and exact == ref_exact
    true = int(torch.unique(packed).numel())
    assert abs(est - true) <= 5 * true / np.sqrt(2046)


def test_plan_from_device_estimate(bg, oracles):
    """Estimate -> plan -> execute, the paper's runtime order."""
    w, o = oracles("C5")
    kc, vc = blugen.device_columns(w)
    plan = bg.plan_estimated(w.schema, kc)
    assert abs(plan.info()["est_groups"] - w.expected_groups) <= 0.15 * w.expected_groups
    res = bg.blu_gby_execute(plan, kc, vc)
    gk, ga = gpu_sorted(res, w.schema)
    assert_parity(gk, ga, o, w.schema)


@pytest.mark.parametrize("name,lock", [("K3", "rule"), ("K3", "0"), ("C3", "1"), ("C4", "1")])
def test_kernel3_row_lock(bg, oracles, monkeypatch, name, lock):
    """NEXT-1: kernel 3 locks the slot once and applies every aggregate. Chosen automatically
    for > 5 aggregates at a low rows/groups ratio (K3); forced on C3/C4 (hash path) for parity."""
    w, o = oracles(name)
    kc, vc = blugen.device_columns(w)
    if lock is not None:
        monkeypatch.setenv("BLU_GBY_ROW_LOCK", lock)
    if name == "C4":
        monkeypatch.setenv("BLU_GBY_FORCE_PATH", "b")
    plan = bg.plan_for(w.schema, w.est_groups, w.n_rows)
    assert plan.info()["row_lock"] == (0 if lock == "0" else 1)
    res = bg.blu_gby_execute(plan, kc, vc)
    gk, ga = gpu_sorted(res, w.schema)
    assert_parity(gk, ga, o, w.schema)


# ---- NEXT-2: wide keys (> 64-bit packed key) --------------------------------------------
WIDE = {
    # two sparse i64 columns: 128-bit key, heavy duplication
    "ss": lambda rng, n: ([(I64, 0), (I64, 0)],
                          [rng.integers(0, 2**62, 997)[rng.integers(0, 997, n)],
                           rng.integers(0, 2**40, 31)[rng.integers(0, 31, n)]]),
    # sparse + two dense columns (dense ones share word 1)
    "sdd": lambda rng, n: ([(I64, 0), (I32, 7), (I64, 1000)],
                           [rng.integers(0, 2**50, 5000)[rng.integers(0, 5000, n)],
                            rng.integers(0, 7, n).astype(np.int32), rng.integers(0, 1000, n)]),
    # dense tuple with domain 2^70: spills into the second word
    "dd": lambda rng, n: ([(I64, 2**40), (I64, 2**30)],
                          [rng.integers(0, 2**40, 3000)[rng.integers(0, 3000, n)],
                           rng.integers(2**30 - 5, 2**30, n)]),
}


@pytest.mark.parametrize("n", [0, 1, 33, 65_537, 1_000_003])
@pytest.mark.parametrize("kind", sorted(WIDE))
def test_wide_keys_parity(bg, kind, n):
    rng = np.random.default_rng(sorted(WIDE).index(kind) * 1000 + n)
    keys, kc = WIDE[kind](rng, n)
    kc = [k.astype(np.int32 if d == I32 else np.int64) for k, (d, _) in zip(kc, keys)]
    sch = blugen.Schema(keys, [I32, I64, F64], ALL(3))
    vc = [rng.integers(-(2**31), 2**31, n).astype(np.int32), rng.integers(-(2**40), 2**40, n),
          rng.integers(-(2**20), 2**20, n) / 64.0]
    o = oracle.groupby_arrays(sch, kc, vc)
    plan = bg.plan_for(sch, max(1, o.keys.shape[0] // 2), n)  # under-estimate: exercises regrow
    assert plan.info()["path"] == bg.BLU_PATH_HASH_GLOBAL
    dk, dv = _mk(kc, vc)
    res = bg.blu_gby_execute(plan, dk, dv, n_rows=n)
    gk, ga = gpu_sorted(res, sch)
    assert_parity(gk, ga, o, sch)


def test_wide_keys_partition_and_merge(bg):
    """Partial -> partition records (2 key words) -> merge_records, and partial merge, for wide keys."""
    rng = np.random.default_rng(5)
    n = 400_001
    keys, kc = WIDE["sdd"](rng, n)
    kc = [k.astype(np.int32 if d == I32 else np.int64) for k, (d, _) in zip(kc, keys)]
    sch = blugen.Schema(keys, [I64, F64], [(COUNT, -1), (SUM, 0), (MIN, 1), (MAX, 0), (AVG, 1)])
    vc = [rng.integers(-(2**40), 2**40, n), rng.integers(-(2**20), 2**20, n) / 64.0]
    o = oracle.groupby_arrays(sch, kc, vc)
    plan = bg.plan_for(sch, o.keys.shape[0], n)
    dk, dv = _mk(kc, vc)
    P = 3
    cuts = np.linspace(0, n, P + 1).astype(int)
    parts = [bg.blu_gby_execute_partial(plan, [k[cuts[r]:cuts[r + 1]] for k in dk],
                                        [v[cuts[r]:cuts[r + 1]] for v in dv]) for r in range(P)]
    gk, ga = gpu_sorted(bg.blu_gby_merge(plan, parts), sch)
    assert_parity(gk, ga, o, sch)
    rb = plan.record_bytes
    inbox = [[] for _ in range(P)]
    for part in parts:
        buf = torch.empty(max(1, part.n_groups) * rb // 8, dtype=torch.int64, device="cuda")
        counts = bg.blu_gby_partition(plan, part, P, buf)
        off = 0
        for dst in range(P):
            inbox[dst].append(buf[off * rb // 8:(off + counts[dst]) * rb // 8])
            off += counts[dst]
    keys_, aggs = [], []
    for dst in range(P):
        recs = torch.cat(inbox[dst])
        k, a = gpu_sorted(bg.blu_gby_merge_records(plan, recs, recs.numel() * 8 // rb), sch)
        keys_.append(k)
        aggs.append(a)
    allk = np.concatenate(keys_)
    order = np.lexsort(allk.T[::-1])
    assert_parity(allk[order], [np.concatenate([a[i] for a in aggs])[order] for i in range(len(sch.aggs))], o, sch)


def test_wide_keys_host_columns(bg):
    rng = np.random.default_rng(9)
    n = 300_007
    keys, kc = WIDE["ss"](rng, n)
    sch = blugen.Schema(keys, [I64], [(COUNT, -1), (SUM, 0), (MAX, 0)])
    vc = [rng.integers(-(2**40), 2**40, n)]
    o = oracle.groupby_arrays(sch, kc, vc)
    plan = bg.plan_for(sch, o.keys.shape[0], n)
    res = bg.blu_gby_execute_host(plan, kc, vc)
    gk, ga = host_sorted(res, sch)
    assert_parity(gk, ga, o, sch)


# ---- 128-bit integer payloads (NEXT-2; "128bit Integer or Decimal"; reading A18) ------
I128 = blugen.I128


def _i128(rng, n, kind):
    """(n, 2) int64 = (lo, hi) words of 128-bit values: the full range, the int64 range (sign
    extended) or values near +-2^126 so that group sums wrap mod 2^128."""
    lo = rng.integers(-(2**63), 2**63, n, dtype=np.int64)
    if kind == "full":
        hi = rng.integers(-(2**63), 2**63, n, dtype=np.int64)
    elif kind == "small":
        hi = lo >> 63
    else:
        hi = rng.choice(np.array([2**62, 2**62 - 1, -(2**62), -(2**62) - 1], np.int64), n)
    return np.ascontiguousarray(np.stack([lo, hi], axis=1))


def _i128_case(rng, n, kind):
    G = max(1, n // 40)
    codes = rng.integers(0, 2**62, G, dtype=np.int64)
    k = codes[rng.integers(0, G, n)] if n else np.zeros(0, np.int64)
    v64 = rng.integers(-(2**62), 2**62, n, dtype=np.int64)
    sch = blugen.Schema([(I64, 0)], [I128, I64],
                        [(COUNT, -1), (SUM, 0), (MIN, 0), (MAX, 0), (AVG, 0), (SUM, 1), (MAX, 1)])
    return sch, [k], [_i128(rng, n, kind), v64], G


@pytest.mark.parametrize("kind", ["full", "small", "wrap"])
@pytest.mark.parametrize("n", [0, 1, 33, 4097, 300_001])
def test_i128_payload_parity(bg, n, kind):
    """SUM mod 2^128, MIN/MAX (signed), AVG = RN(RN(sum)/count) of a 128-bit column beside an int64
    column, bit-exact against the oracle's __int128 arithmetic (path (b), one pass, k_agg_q)."""
    rng = np.random.default_rng(1000 + n)
    sch, kc, vc, G = _i128_case(rng, n, kind)
    o = oracle.groupby_arrays(sch, kc, vc)
    plan = bg.plan_for(sch, G, max(n, 1))
    info = plan.info()
    assert info["path"] == bg.BLU_PATH_HASH_GLOBAL and info["partitions"] == 1 and info["hot_front"] == 0
    dk, dv = _mk(kc, vc)
    bg.blu_gby_set_timing(True)
    res = bg.blu_gby_execute(plan, dk, dv, n_rows=n)
    t = bg.blu_gby_last_timing()
    bg.blu_gby_set_timing(False)
    if n:
        assert t["kernel"].startswith("k_agg_q"), t["kernel"]
    gk, ga = gpu_sorted(res, sch)
    if n:
        assert ga[1].shape == (res.n_groups, 2)
    assert_parity(gk, ga, o, sch)


def test_i128_regrow_partial_merge_and_host(bg):
    """Under-estimated groups (regrow), 3 partial shards merged on the device (128-bit states),
    and host columns through blu_gby_execute_host — all equal to the oracle."""
    rng = np.random.default_rng(77)
    n = 200_003
    sch, kc, vc, G = _i128_case(rng, n, "full")
    o = oracle.groupby_arrays(sch, kc, vc)
    dk, dv = _mk(kc, vc)
    plan = bg.plan_for(sch, 1, n)
    gk, ga = gpu_sorted(bg.blu_gby_execute(plan, dk, dv), sch)
    assert_parity(gk, ga, o, sch)
    assert plan.info()["retries_last"] >= 1
    plan = bg.plan_for(sch, G, n)
    cuts = [0, 70_001, 140_000, n]
    parts = [bg.blu_gby_execute_partial(plan, [k[a:b] for k in dk], [v[a:b] for v in dv], n_rows=b - a)
             for a, b in zip(cuts[:-1], cuts[1:])]
    assert parts[0].states[1].shape[1] == 2  # the 128-bit SUM state travels as (lo, hi)
    gk, ga = gpu_sorted(bg.blu_gby_merge(plan, parts), sch)
    assert_parity(gk, ga, o, sch)
    hk, ha = host_sorted(bg.blu_gby_execute_host(plan, [torch.from_numpy(k) for k in kc],
                                                 [torch.from_numpy(v) for v in vc]), sch)
    assert_parity(hk, ha, o, sch)


def test_i128_record_helpers_unsupported(bg):
    rng = np.random.default_rng(5)
    sch, kc, vc, G = _i128_case(rng, 1000, "small")
    plan = bg.plan_for(sch, G, 1000)
    dk, dv = _mk(kc, vc)
    part = bg.blu_gby_execute_partial(plan, dk, dv)
    buf = torch.empty(1 << 20, dtype=torch.uint8, device="cuda")
    with pytest.raises(bg.BluError) as e:
        bg.blu_gby_partition(plan, part, 2, buf)
    assert e.value.status == bg.BLU_E_UNSUPPORTED
