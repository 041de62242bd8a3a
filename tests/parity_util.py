"""Helpers for GPU-vs-oracle parity tests (test infrastructure; imports the oracle)."""
import numpy as np

import blugen
import oracle
from blugen import AVG, F64, I128, MAX, MIN, SUM


def _empty_aggs(schema):
    return [np.zeros((0, 2) if schema.agg_out_dtype(a) == I128 else 0) for a in range(len(schema.aggs))]


def gpu_sorted(res, schema):
    """(keys (G,K) int64 lexsorted, [agg arrays in the same order]) from a finalized Result."""
    K = len(schema.keys)
    if res.n_groups == 0:
        return np.zeros((0, K), np.int64), _empty_aggs(schema)
    keys = np.stack([k.cpu().numpy().astype(np.int64) for k in res.keys], axis=1)
    order = np.lexsort(keys.T[::-1])
    aggs = [a.cpu().numpy()[order] for a in res.aggs]
    return keys[order], aggs


def host_sorted(res, schema):
    K = len(schema.keys)
    if res.n_groups == 0:
        return np.zeros((0, K), np.int64), _empty_aggs(schema)
    keys = np.stack([k.astype(np.int64) for k in res.keys], axis=1)
    order = np.lexsort(keys.T[::-1])
    return keys[order], [a[order] for a in res.aggs]


def assert_parity(gkeys, gaggs, o: oracle.OracleResult, schema, f64_tol=None):
    """Bit-exact on keys, COUNT, MIN, MAX, integer SUM and (dyadic) f64; with f64_tol the f64
    SUM/AVG must be within f64_tol * sum|v| (per group; AVG divided by COUNT) — reading A13."""
    assert gkeys.shape == o.keys.shape, (gkeys.shape, o.keys.shape)
    assert np.array_equal(gkeys, o.keys)
    for a, (op, col) in enumerate(schema.aggs):
        g = gaggs[a]
        e = o.aggs[a]
        is_f = schema.agg_out_dtype(a) == F64
        if is_f and f64_tol is not None and op in (SUM, AVG) and o.sumabs[a] is not None:
            bound = f64_tol * o.sumabs[a]
            if op == AVG:
                bound = bound / o.count
            err = np.abs(g.astype(np.float64) - e)
            bad = np.nonzero(err > bound)[0]
            assert bad.size == 0, (a, bad[:5], g[bad[:5]], e[bad[:5]])
        elif is_f:
            ok = g.astype(np.float64).view(np.int64) == e.astype(np.float64).view(np.int64)
            bad = np.nonzero(~ok)[0]
            assert bad.size == 0, (a, op, bad[:5], g[bad[:5]], e[bad[:5]])
        else:
            bad = np.nonzero(g.astype(np.int64) != e.astype(np.int64))[0]
            assert bad.size == 0, (a, op, bad[:5], g[bad[:5]], e[bad[:5]])


def oracle_for(w: blugen.Workload, kc=None, vc=None):
    if kc is None:
        return oracle.groupby_generated(w)
    return oracle.groupby_arrays(w.schema, kc, vc)
