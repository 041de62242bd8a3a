"""Host-side tests of libblugby's C ABI: the library loads, exports every symbol the header declares,
and the planner (host only, no GPU) makes the documented decisions. No GPU needed."""
import ctypes
import json
import os
import re
import struct

import pytest

import blugen
from blugen import AVG, COUNT, F64, I32, I64, MAX, MIN, SUM

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def bg():
    from paper_conf_sigmod_merajispcksygnk16_b200 import blugby
    return blugby


def test_library_exports_every_header_symbol(bg):
    hdr = open(os.path.join(ROOT, "include", "blu_gby.h")).read()
    names = set(re.findall(r"\b(blu_gby_[a-z_0-9]+)\s*\(", hdr))
    assert len(names) >= 20
    lib = ctypes.CDLL(bg.LIB_PATH)
    missing = [n for n in sorted(names) if not hasattr(lib, n)]
    assert not missing, missing


def test_library_exports_sort_header_symbols(bg):
    """include/blu_sort.h (NEXT-4 sort offload): every declared entry point is exported;
    argument checks run without a GPU."""
    hdr = open(os.path.join(ROOT, "include", "blu_sort.h")).read()
    names = set(re.findall(r"\b(blu_sort_[a-z_0-9]+)\s*\(", hdr))
    assert names == {"blu_sort_partial_keys", "blu_sort_pairs", "blu_sort_dup_ranges", "blu_sort_rows"}
    lib = ctypes.CDLL(bg.LIB_PATH)
    assert all(hasattr(lib, n) for n in names)
    st = bg.lib.blu_sort_rows(None, 10, 6, None, None, None)       # W not a multiple of 4
    assert st == bg.BLU_E_INVALID
    st = bg.lib.blu_sort_rows(None, 0, 16, None, None, None)       # empty input: nothing to do
    assert st == bg.BLU_OK
    st = bg.lib.blu_sort_pairs(None, None, 5, None, None, None)    # NULL buffers
    assert st == bg.BLU_E_INVALID


def test_generator_library_exports():
    hdr = open(os.path.join(ROOT, "include", "blu_gen.h")).read()
    names = set(re.findall(r"^(?:int|void)\s+(blu_gen_[a-z_0-9]+)\s*\(", hdr, re.M))
    lib = ctypes.CDLL(blugen.LIB_PATH)
    assert names and all(hasattr(lib, n) for n in names)


def test_status_strings(bg):
    for s, name in bg.STATUS_NAMES.items():
        assert bg.lib.blu_gby_status_str(s).decode() == name


def test_table1_mask_matches_paper(bg):
    """S4 template == PAPER.md Table 1: SUM(C1), MAX(C2), MIN(C3) group by C1."""
    g = json.load(open(os.path.join(ROOT, "tests", "golden", "table1_mask.json")))
    dt = {"i32": I32, "i64": I64, "f64": F64}
    ops = {"COUNT": COUNT, "SUM": SUM, "MIN": MIN, "MAX": MAX, "AVG": AVG}
    keys = [(dt[d], n) for d, n in g["schema"]["keys"]]
    vals = [dt[d] for d in g["schema"]["vals"]]
    aggs = [(ops[o], c) for o, c in g["schema"]["aggs"]]
    plan = bg.blu_gby_plan(keys, vals, aggs, est_groups=1000, n_rows=10**6)
    assert plan.info()["path"] == bg.BLU_PATH_HASH_GLOBAL
    t = plan.slot_template()
    assert len(t) == g["row_bytes"] == 32
    for f in g["fields"]:
        raw = t[f["offset"]:f["offset"] + f["bytes"]]
        if "value_hex" in f:
            assert raw.hex().upper() == f["value_hex"]
        else:
            fmt = "<q" if f["bytes"] == 8 else "<i"
            assert struct.unpack(fmt, raw)[0] == f["value"], f["name"]


def _plan(bg, w, **kw):
    est = kw.pop("est", w.est_groups)
    return bg.plan_for(w.schema, est, kw.pop("n_rows", w.n_rows))


def test_planner_paths_for_the_five_configs(bg):
    """The moderator: small dense domain -> (a); dense 1e5 domain with a high
    rows/groups ratio -> direct-mapped (b') + hot-key front; sparse keys -> hash (b)."""
    c1 = _plan(bg, blugen.workload("C1")).info()
    c2 = _plan(bg, blugen.workload("C2")).info()
    c3 = _plan(bg, blugen.workload("C3")).info()
    c4 = _plan(bg, blugen.workload("C4")).info()
    c5 = _plan(bg, blugen.workload("C5")).info()
    assert c1["path"] == c2["path"] == bg.BLU_PATH_DENSE_SMEM
    assert c1["capacity"] == 16 and c2["capacity"] == 1024
    # C3: 537 MB at load 0.6 exceeds the L2 budget -> partitioned mode; its 10^7 groups fit 2048
    # shared-memory bucket tables (two-level scatter), so that mode is the default
    assert c3["path"] == bg.BLU_PATH_HASH_GLOBAL and c3["capacity"] == 2**24 and c3["slot_bytes"] == 32
    assert c3["part_smem"] == 1 and c3["partitions"] == 2048
    assert c3["hot_front"] == 0
    assert c4["path"] == bg.BLU_PATH_DIRECT_GLOBAL and c4["capacity"] == 100_000 and c4["hot_front"] == 1
    assert c5["path"] == bg.BLU_PATH_HASH_GLOBAL and c5["capacity"] == 2**27 and c5["partitions"] >= 64
    assert c1["partitions"] == c2["partitions"] == c4["partitions"] == 1


def test_planner_partitioned_l2_mode(bg, monkeypatch):
    """K3's 8-field states need more than the 16384 bucket tables a two-level scatter reaches: pass 2
    in L2-resident slices of the global table, sized at load <= 0.5. C5's 5*10^7 groups fit 16384
    tables behind a 128 x 128 scatter (the default, 141 vs 148 ms for the L2 mode at 4e9 rows);
    BLU_GBY_PART_SMEM=0 forces the L2 mode for C5 and C3."""
    c5 = _plan(bg, blugen.workload("C5")).info()
    assert c5["part_smem"] == 1 and c5["partitions"] == 16384
    k3 = _plan(bg, blugen.workload("K3")).info()
    assert k3["part_smem"] == 0 and k3["partitions"] > 1
    monkeypatch.setenv("BLU_GBY_PART_SMEM", "0")
    c5 = _plan(bg, blugen.workload("C5")).info()
    assert c5["part_smem"] == 0 and c5["partitions"] >= 64
    c3 = _plan(bg, blugen.workload("C3")).info()
    assert c3["path"] == bg.BLU_PATH_HASH_GLOBAL and c3["capacity"] == 2**25 and c3["slot_bytes"] == 32
    assert c3["part_smem"] == 0
    assert c3["partitions"] >= 16 and c3["capacity"] * 32 // c3["partitions"] <= 48 * 2**20


def test_planner_partitioned_smem_mode(bg, monkeypatch):
    """BLU_GBY_PART_SMEM=1: pass 2 in per-CTA shared-memory bucket tables; buckets hold <= 0.7 x the
    table's entries on average (C3: 10^7 / 2048 = 4883 of 8000); the global table keeps load <= 0.7;
    the two-level scatter (32 x 512; the second level one launch with 512 bins per tile) allows 16384
    buckets (C5), a one-level scatter at most 4096."""
    monkeypatch.setenv("BLU_GBY_PART_SMEM", "1")
    c3 = _plan(bg, blugen.workload("C3")).info()
    assert c3["part_smem"] == 1 and c3["capacity"] == 2**24
    assert c3["partitions"] == 2048 and c3["bucket_entries"] >= 7900
    assert 10**7 / c3["partitions"] <= 0.7 * c3["bucket_entries"]
    c5 = _plan(bg, blugen.workload("C5")).info()
    assert c5["part_smem"] == 1 and c5["partitions"] == 16384
    monkeypatch.setenv("BLU_GBY_PART_2LEVEL", "0")
    c5 = _plan(bg, blugen.workload("C5")).info()
    assert c5["part_smem"] == 1 and c5["partitions"] == 4096


@pytest.mark.parametrize("est,cap", [(1, 1024), (700, 1024), (716, 1024), (717, 2048), (10_000_000, 2**24),
                                     (50_000_000, 2**27)])
def test_capacity_rounding(bg, monkeypatch, est, cap):
    """cap = next_pow2(ceil(max(est,1)/0.7)), >= 1024 ("slightly larger", reading A5);
    one-pass mode and the shared-memory partitioned mode (the L2-slice partitioned mode sizes its
    buckets at load <= 0.5)."""
    monkeypatch.setenv("BLU_GBY_PART_MB", "0")
    p = bg.blu_gby_plan([(I64, 0)], [I64], [(SUM, 0)], est, 10**10)
    assert p.info()["capacity"] == cap and p.info()["partitions"] == 1
    monkeypatch.delenv("BLU_GBY_PART_MB")
    p2 = bg.blu_gby_plan([(I64, 0)], [I64], [(SUM, 0)], est, 10**10)
    if p2.info()["partitions"] > 1 and not p2.info()["part_smem"]:  # L2-resident slices: load <= 0.5
        assert p2.info()["capacity"] >= 2 * est
    if p2.info()["part_smem"]:  # default shared-memory bucket tables: the global table keeps load <= 0.7
        assert p2.info()["capacity"] == cap and p2.info()["partitions"] >= 256
    monkeypatch.setenv("BLU_GBY_PART_SMEM", "1")
    p3 = bg.blu_gby_plan([(I64, 0)], [I64], [(SUM, 0)], est, 10**10)
    if p3.info()["partitions"] > 1:  # shared-memory bucket tables: the global table keeps load <= 0.7
        assert p3.info()["part_smem"] == 1 and p3.info()["capacity"] == cap


def test_est_clamped_to_rows(bg):
    p = bg.blu_gby_plan([(I64, 0)], [I64], [(SUM, 0)], 10**9, 5000)
    assert p.info()["capacity"] == 8192


def test_state_fields_and_slot_sizes(bg):
    p = bg.plan_for(blugen.workload("C3").schema, 10**7, 10**9)
    i = p.info()
    # COUNT, SUM(v0) i64, SUM(v1) f64 (AVG shares COUNT + SUM): key 8 + 3 x 8 = 32 B
    assert i["n_states"] == 3 and i["state_dtypes"] == [I64, I64, F64] and i["slot_bytes"] == 32
    p4 = bg.plan_for(blugen.workload("C4").schema, 10**5, 10**9)
    i4 = p4.info()
    # COUNT, SUM v0, SUM v1 (+AVG v1), SUM v2, MIN v2, MAX v2
    assert i4["n_states"] == 6 and i4["slot_bytes"] == 64
    assert p4.dense_state_shape() == (4, 0, 1, 1, 100_000)


def test_schema_validation(bg):
    with pytest.raises(bg.BluError) as e:
        bg.blu_gby_plan([], [I64], [(SUM, 0)], 1, 1)
    assert e.value.status == bg.BLU_E_INVALID
    with pytest.raises(bg.BluError) as e:
        bg.blu_gby_plan([(I32, 4)], [I64], [(SUM, 3)], 1, 1)
    assert e.value.status == bg.BLU_E_INVALID
    with pytest.raises(bg.BluError) as e:
        bg.blu_gby_plan([(F64, 4)], [I64], [(SUM, 0)], 1, 1)
    assert e.value.status == bg.BLU_E_INVALID
    with pytest.raises(bg.BluError) as e:  # three sparse key columns: wider than 128 bits
        bg.blu_gby_plan([(I64, 0), (I64, 0), (I32, 0)], [I64], [(SUM, 0)], 1, 1)
    assert e.value.status == bg.BLU_E_UNSUPPORTED
    with pytest.raises(bg.BluError) as e:  # dense tuple of 2^120 codes does not fit two 2^62 words
        bg.blu_gby_plan([(I64, 2**40), (I64, 2**40), (I64, 2**40)], [I64], [(SUM, 0)], 1, 1)
    assert e.value.status == bg.BLU_E_UNSUPPORTED
    with pytest.raises(bg.BluError) as e:  # sparse + sparse + any dense column: no room
        bg.blu_gby_plan([(I64, 0), (I64, 0), (I32, 4)], [I64], [(SUM, 0)], 1, 1)
    assert e.value.status == bg.BLU_E_UNSUPPORTED
    with pytest.raises(bg.BluError) as e:
        bg.blu_gby_plan([(I32, 4)], [I64], [(7, 0)], 1, 1)
    assert e.value.status == bg.BLU_E_INVALID


def test_forced_path_env(bg, monkeypatch):
    w = blugen.workload("C2")
    monkeypatch.setenv("BLU_GBY_FORCE_PATH", "b")
    assert _plan(bg, w).info()["path"] == bg.BLU_PATH_HASH_GLOBAL
    monkeypatch.setenv("BLU_GBY_FORCE_PATH", "d")
    assert _plan(bg, w).info()["path"] == bg.BLU_PATH_DIRECT_GLOBAL
    monkeypatch.setenv("BLU_GBY_FORCE_PATH", "a")
    with pytest.raises(bg.BluError):
        _plan(bg, blugen.workload("C3"))


def test_record_bytes(bg):
    p = bg.plan_for(blugen.workload("C3").schema, 10**7, 10**9)
    assert p.record_bytes == 8 * (1 + 3)


def test_planner_kernel3_rule(bg, monkeypatch):
    """more than 5 aggregation functions and a low rows/groups ratio -> kernel 3 (row lock).
    Off by default on B200 (native 64-bit REDs measured faster); BLU_GBY_ROW_LOCK=rule applies it."""
    k3 = bg.plan_for(blugen.workload("K3").schema, 50_000_000, 100_000_000).info()
    assert k3["path"] == bg.BLU_PATH_HASH_GLOBAL and k3["row_lock"] == 0 and k3["n_states"] == 8
    monkeypatch.setenv("BLU_GBY_ROW_LOCK", "rule")
    k3 = bg.plan_for(blugen.workload("K3").schema, 50_000_000, 100_000_000).info()
    assert k3["row_lock"] == 1
    c3 = bg.plan_for(blugen.workload("C3").schema, 10**7, 10**9).info()
    assert c3["row_lock"] == 0  # 3 fields
    hi = bg.plan_for(blugen.workload("K3").schema, 1000, 100_000_000).info()
    assert hi["row_lock"] == 0  # 1e5 rows per group: contention, keep per-field atomics


@pytest.mark.parametrize("keys, n_fields", [
    ([(I64, 0), (I32, 4)], 1),                 # sparse + dense
    ([(I64, 2**40), (I64, 2**30)], 1),         # dense domain >= 2^62
    ([(I64, 0), (I64, 0)], 1),                 # two sparse columns
])
def test_wide_key_plans(bg, keys, n_fields):
    """Key tuples wider than one 64-bit word plan path (b) with a two-word key."""
    p = bg.blu_gby_plan(keys, [I64], [(SUM, 0)], 1000, 10**6)
    d = p.info()
    assert d["path"] == bg.BLU_PATH_HASH_GLOBAL
    assert d["hot_front"] == 0 and d["partitions"] == 1
    assert d["n_states"] == n_fields
    assert p.record_bytes == 8 * (2 + n_fields)
    assert d["slot_bytes"] >= 16 + 8


@pytest.mark.parametrize("name", ["C1", "C2", "C3", "C4", "C5", "K3"])
def test_jit_probe_compiles_plan_kernels(bg, name):
    """The NVRTC programs execute would JIT for each config compile with the NVRTC the library loads
    (no GPU needed); a failure here would silently fall back to the generic kernels on the GPU."""
    import blugen
    w = blugen.workload(name)
    plan = bg.plan_for(w.schema, w.est_groups, w.n_rows)
    st, n, log = bg.blu_gby_jit_probe(plan)
    assert st == bg.BLU_OK, log
    info = plan.info()
    assert n >= (1 if info["partitions"] == 1 else 3)


def test_jit_probe_wide_keys_unsupported(bg):
    plan = bg.blu_gby_plan([(I64, 0), (I64, 0)], [I64], [(SUM, 0)], 100, 1000)
    st, n, _ = bg.blu_gby_jit_probe(plan)
    assert st == bg.BLU_E_UNSUPPORTED and n == 0


def test_i128_plan_and_mask(bg):
    """128-bit payloads: path (b) in one pass (no front, no partitions, no kernel 3); the
    states are 16-byte fields at 16-byte offsets whose mask values are SUM 0, MIN INT128_MAX,
    MAX INT128_MIN (the Table 1 rule for a 128-bit type: "for MAX ... the minimum value")."""
    I128 = blugen.I128
    p = bg.blu_gby_plan([(I64, 0)], [I128, I64], [(COUNT, -1), (SUM, 0), (MIN, 0), (MAX, 0), (AVG, 0)], 10**7, 10**9)
    info = p.info()
    assert info["path"] == bg.BLU_PATH_HASH_GLOBAL and info["partitions"] == 1 and info["hot_front"] == 0
    assert sorted(info["state_dtypes"]) == [I64, I128, I128, I128]  # COUNT, SUM, MIN, MAX
    t = p.slot_template()
    assert struct.unpack_from("<q", t, 0)[0] == -1  # EMPTY key
    words = [struct.unpack_from("<QQ", t, o) for o in range(16, len(t) - 15, 16)]
    assert (0, 0) in words
    assert ((1 << 64) - 1, (1 << 63) - 1) in words   # INT128_MAX (MIN's identity)
    assert (0, 1 << 63) in words                     # INT128_MIN (MAX's identity)
    st, n, _ = bg.blu_gby_jit_probe(p)
    assert st == bg.BLU_E_UNSUPPORTED and n == 0     # generic k_agg_q only
    with pytest.raises(bg.BluError) as e:            # 128-bit payloads with two-word keys
        bg.blu_gby_plan([(I64, 0), (I64, 0)], [I128], [(SUM, 0)], 100, 1000)
    assert e.value.status == bg.BLU_E_UNSUPPORTED


def test_planner_no_u64_wrap_near_2_pow_62(bg):
    """two i32 keys of dict_size 2^31 give D = 2^62; D * entry bytes wrapped u64 to 0
    and the planner chose the shared-memory path with 0 bytes. The one-word packing now requires
    D < 2^62 strictly, so this tuple takes two key words (hash path); D just below 2^62 stays one word
    on the hash/direct path, never path (a)."""
    d = bg.blu_gby_plan([(I32, 2**31), (I32, 2**31)], [], [(COUNT, -1)], 1000, 10**6).info()
    assert d["path"] == bg.BLU_PATH_HASH_GLOBAL and d["slot_bytes"] >= 24  # two-word key
    d = bg.blu_gby_plan([(I32, 2**31), (I32, 2**31 - 1)], [], [(COUNT, -1)], 1000, 10**6).info()
    assert d["path"] == bg.BLU_PATH_HASH_GLOBAL and d["slot_bytes"] == 16 and d["capacity"] >= 1024
    # the largest dense domain path (a) takes still fits its 96 KB shared-memory budget
    d = bg.blu_gby_plan([(I32, 4096)], [], [(COUNT, -1)], 1000, 10**6).info()
    assert d["path"] == bg.BLU_PATH_DENSE_SMEM and 0 < d["smem_bytes"] <= 96 * 1024


def test_planner_rejects_slots_over_256_bytes(bg):
    """16 SUMs over 16 i128 columns need a 320-byte slot, more than the init
    template holds; the planner reports BLU_E_UNSUPPORTED instead of overflowing it."""
    from blugen import I128
    with pytest.raises(bg.BluError) as e:
        bg.blu_gby_plan([(I64, 0)], [I128] * 16, [(SUM, c) for c in range(16)], 1000, 10**6)
    assert e.value.status == bg.BLU_E_UNSUPPORTED
    ok = bg.blu_gby_plan([(I64, 0)], [I128] * 15, [(SUM, c) for c in range(15)], 1000, 10**6).info()
    assert ok["slot_bytes"] == 256


def test_env_knobs_follow_the_environment_per_call(bg, monkeypatch):
    """BLU_* knobs come from a per-API-call snapshot of the environment (csrc/env.cpp): a change is
    seen by the next call, a removal too, and another thread sees its process environment as well."""
    import threading
    w = blugen.workload("C2")
    monkeypatch.delenv("BLU_GBY_FORCE_PATH", raising=False)
    assert _plan(bg, w).info()["path"] == bg.BLU_PATH_DENSE_SMEM
    monkeypatch.setenv("BLU_GBY_FORCE_PATH", "b")
    assert _plan(bg, w).info()["path"] == bg.BLU_PATH_HASH_GLOBAL
    monkeypatch.setenv("BLU_GBY_FORCE_PATH", "d")
    assert _plan(bg, w).info()["path"] == bg.BLU_PATH_DIRECT_GLOBAL
    out = {}
    t = threading.Thread(target=lambda: out.setdefault("path", _plan(bg, w).info()["path"]))
    t.start()
    t.join()
    assert out["path"] == bg.BLU_PATH_DIRECT_GLOBAL
    monkeypatch.setenv("BLU_GBY_FORCE_PATH", "b")
    assert _plan(bg, w).info()["path"] == bg.BLU_PATH_HASH_GLOBAL
    monkeypatch.delenv("BLU_GBY_FORCE_PATH")
    assert _plan(bg, w).info()["path"] == bg.BLU_PATH_DENSE_SMEM


def test_planner_clamps_forced_l2_partitions(bg, monkeypatch):
    """The L2-slice pass 2 indexes at most kMaxSegs = 1024 buckets (its per-CTA prefix of the buckets'
    warp tiles): a forced BLU_GBY_PARTS above that is clamped (2048 forced buckets once overran the
    shared array: an illegal address on the GPU)."""
    monkeypatch.setenv("BLU_GBY_PART_SMEM", "0")
    monkeypatch.setenv("BLU_GBY_PARTS", "2048")
    info = _plan(bg, blugen.workload("C3")).info()
    assert info["part_smem"] == 0 and info["partitions"] == 1024
    monkeypatch.setenv("BLU_GBY_PART_SMEM", "1")
    info = _plan(bg, blugen.workload("C3")).info()
    assert info["part_smem"] == 1 and info["partitions"] == 2048
