"""Full-size parity (BASELINE.json configs at their real sizes, in the launch configuration bench.py
times): sampled groups checked exactly against the oracle, plus whole-result properties that hold at
any size (SURVEY.md §8(c) "Invariants").

The oracle runs over disjoint row ranges in a process pool (one plain single-threaded std::map per
range) restricted to the sampled key tuples; the ranges are combined by the definition's additivity
(COUNT and SUM add, MIN/MAX of the parts) with Python big ints. Column-wide sums for the invariants
come from torch reductions (library routines independent of libblugby and of the oracle)."""
import math
import os
from concurrent.futures import ProcessPoolExecutor

import numpy as np
import pytest

import blugen
from blugen import AVG, COUNT, F64, MAX, MIN, SUM

pytestmark = [pytest.mark.gpu, pytest.mark.slow]

torch = pytest.importorskip("torch")


def wrap64(x):
    return ((x + (1 << 63)) % (1 << 64)) - (1 << 63)


def _sum_schema(schema):
    """Same aggregates with AVG(v) replaced by SUM(v): parts must be combined on exact sums."""
    return blugen.Schema(schema.keys, schema.vals, [(SUM if op == AVG else op, col) for op, col in schema.aggs])


def _oracle_part(args):
    name, kw, row0, n, keys = args
    import oracle as orc
    w = blugen.workload(name, **kw)
    w.schema = _sum_schema(w.schema)
    o = orc.groupby_generated(w, row0=row0, n=n, filter_keys=keys)
    return o.keys, o.count, o.aggs


def sampled_oracle(name, kw, keys, n_rows):
    """Per sampled key tuple: (count, [per-agg parts]) combined over row ranges."""
    procs = max(1, min(32, os.cpu_count() or 1))
    cuts = np.linspace(0, n_rows, procs + 1).astype(np.int64)
    jobs = [(name, kw, int(a), int(b - a), keys) for a, b in zip(cuts[:-1], cuts[1:])]
    with ProcessPoolExecutor(procs) as ex:
        parts = list(ex.map(_oracle_part, jobs))
    return parts


def combine(parts, schema):
    acc = {}
    for keys, count, aggs in parts:
        for g in range(len(count)):
            k = tuple(int(x) for x in keys[g])
            c = int(count[g])
            if k not in acc:
                acc[k] = [0, [None] * len(schema.aggs)]
            e = acc[k]
            e[0] += c
            for a, (op, col) in enumerate(schema.aggs):
                v = aggs[a][g]  # AVG positions hold this part's SUM (see _sum_schema)
                isf = op != COUNT and schema.vals[col] == F64
                cur = e[1][a]
                if op in (SUM, AVG, COUNT):
                    val = (math.fsum([cur or 0.0, float(v)]) if isf else (cur or 0) + int(v))
                elif op == MIN:
                    val = v if cur is None else min(cur, v)
                else:
                    val = v if cur is None else max(cur, v)
                e[1][a] = val
    return acc


def check_sampled(res, schema, acc):
    gk = np.stack([k.cpu().numpy().astype(np.int64) for k in res.keys], axis=1)
    want = np.array(sorted(acc.keys()), dtype=np.int64)
    # locate the sampled tuples in the GPU result
    pos = {}
    for kk in want:
        m = np.nonzero(np.all(gk == kk[None, :], axis=1))[0]
        assert m.size == 1, (kk, m)
        pos[tuple(int(x) for x in kk)] = int(m[0])
    aggs = [a.cpu().numpy() for a in res.aggs]
    for k, (cnt, vals) in acc.items():
        i = pos[k]
        for a, (op, col) in enumerate(schema.aggs):
            g = aggs[a][i]
            if op == COUNT:
                assert int(g) == cnt
            elif op == AVG:
                s_ = float(vals[a]) if schema.vals[col] == F64 else float(wrap64(vals[a]))
                assert float(g) == s_ / float(cnt), (k, a)
            elif op == SUM and schema.vals[col] != F64:
                assert int(g) == wrap64(vals[a]), (k, a)
            elif op == SUM:
                assert float(g) == float(vals[a]), (k, a)
            else:
                assert g == vals[a], (k, a, g, vals[a])


def invariants(res, w, kc, vc):
    cnt_a = [a for a, (op, _) in enumerate(w.schema.aggs) if op == COUNT]
    if cnt_a:
        assert int(res.aggs[cnt_a[0]].sum().item()) == w.n_rows
    for a, (op, col) in enumerate(w.schema.aggs):
        if op != SUM:
            continue
        if w.schema.vals[col] == F64:
            assert float(res.aggs[a].sum().item()) == float(vc[col].sum().item())  # dyadic: exact
        else:
            assert int(res.aggs[a].sum().item()) == int(vc[col].long().sum().item())
    # MIN <= AVG <= MAX for columns carrying all three
    mins = {col: res.aggs[a] for a, (op, col) in enumerate(w.schema.aggs) if op == MIN}
    maxs = {col: res.aggs[a] for a, (op, col) in enumerate(w.schema.aggs) if op == MAX}
    for a, (op, col) in enumerate(w.schema.aggs):
        if op == AVG and col in mins and col in maxs:
            assert bool((mins[col].double() <= res.aggs[a]).all()) and bool((res.aggs[a] <= maxs[col].double()).all())
    # keys unique
    K = len(res.keys)
    packed = res.keys[0].long()
    for k in range(1, K):
        packed = packed * int(w.schema.keys[k - 1][1] or 1) + res.keys[k].long()
    assert torch.unique(packed).numel() == res.n_groups


@pytest.fixture(scope="module")
def bg():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sigmod_merajispcksygnk16_b200 import blugby
    return blugby


def run_full(bg, name, n_sample):
    w = blugen.workload(name)
    kc, vc = blugen.device_columns(w)
    torch.cuda.synchronize()
    plan = bg.plan_for(w.schema, w.est_groups, w.n_rows)
    res = bg.blu_gby_execute(plan, kc, vc)
    assert res.n_groups == w.expected_groups, (res.n_groups, w.expected_groups)
    invariants(res, w, kc, vc)
    # sample: the first rows' keys (for C4 this includes the hottest tuples) + strided groups
    idx = torch.from_numpy(np.linspace(0, res.n_groups - 1, n_sample // 2).astype(np.int64)).cuda()
    sk = torch.stack([k[idx].long() for k in res.keys], 1).cpu().numpy()
    hk = torch.stack([k[: n_sample // 2].long() for k in kc], 1).cpu().numpy()
    keys = np.unique(np.concatenate([sk, hk]), axis=0)
    del kc, vc
    torch.cuda.empty_cache()
    acc = combine(sampled_oracle(name, {}, keys, w.n_rows), w.schema)
    assert len(acc) == keys.shape[0]
    check_sampled(res, w.schema, acc)
    return res


def test_c2_full_all_groups(bg):
    run_full(bg, "C2", 2048)  # all 1024 groups are sampled


def test_c3_full_sampled(bg):
    run_full(bg, "C3", 48)


def test_c4_full_sampled(bg):
    run_full(bg, "C4", 48)


def test_c5_full_single_gpu_sampled(bg):
    bg.blu_gby_release_workspace()  # earlier full-size tests leave tens of GB of idle workspace cached
    torch.cuda.empty_cache()
    free, total = torch.cuda.mem_get_info()
    if free < 130 * 2**30:
        pytest.skip("C5 (4e9 rows, 96 GB of columns) needs ~130 GB free on one GPU")
    run_full(bg, "C5", 32)
