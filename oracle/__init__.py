"""ORACLE — test infrastructure only (see oracle/blu_oracle.cpp header).

ctypes wrapper around liboracle.so, the plain single-threaded C++ std::map GROUP BY. Only tests/,
__graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference leg may import this module.
It never imports the product package (paper_conf_sigmod_merajispcksygnk16_b200); it shares only the
input generator (blugen) with it.
"""
from __future__ import annotations

import ctypes
import dataclasses
import os
from typing import List, Optional, Sequence

import numpy as np

import blugen
from blugen import COUNT, SUM, MIN, MAX, AVG, I32, I64, F64, I128

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "liboracle.so")


class OracleSchema(ctypes.Structure):
    _fields_ = [
        ("n_keys", ctypes.c_int32),
        ("key_dtypes", ctypes.POINTER(ctypes.c_int32)),
        ("n_vals", ctypes.c_int32),
        ("val_dtypes", ctypes.POINTER(ctypes.c_int32)),
        ("n_aggs", ctypes.c_int32),
        ("agg_ops", ctypes.POINTER(ctypes.c_int32)),
        ("agg_cols", ctypes.POINTER(ctypes.c_int32)),
    ]


_lib = None


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} missing: run `make`")
        L = ctypes.CDLL(LIB_PATH)
        vp = ctypes.c_void_p
        L.oracle_groupby_arrays.argtypes = [ctypes.POINTER(OracleSchema), vp, vp, ctypes.c_uint64,
                                            ctypes.c_uint32, ctypes.c_uint32, vp, ctypes.c_uint64]
        L.oracle_groupby_arrays.restype = vp
        L.oracle_groupby_generated.argtypes = [ctypes.POINTER(OracleSchema), vp, vp, ctypes.c_uint64,
                                               ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint32, vp,
                                               ctypes.c_uint64]
        L.oracle_groupby_generated.restype = vp
        L.oracle_n_groups.argtypes = [vp]
        L.oracle_n_groups.restype = ctypes.c_uint64
        L.oracle_fetch.argtypes = [vp, vp, vp, vp, vp]
        L.oracle_fetch.restype = None
        L.oracle_free.argtypes = [vp]
        L.oracle_free.restype = None
        u64 = ctypes.c_uint64
        L.oracle_partial_keys.argtypes = [vp, u64, ctypes.c_uint32, ctypes.c_uint32, vp]
        L.oracle_partial_keys.restype = None
        L.oracle_sort_pairs.argtypes = [vp, vp, u64, vp, vp]
        L.oracle_sort_pairs.restype = None
        L.oracle_dup_ranges.argtypes = [vp, u64, vp, vp]
        L.oracle_dup_ranges.restype = u64
        L.oracle_sort_rows.argtypes = [vp, u64, ctypes.c_uint32, vp]
        L.oracle_sort_rows.restype = None
        L.oracle_kmv.argtypes = [vp, vp, vp, ctypes.c_int32, u64, ctypes.c_uint32, vp]
        L.oracle_kmv.restype = ctypes.c_double
        L.oracle_fmix64_export.argtypes = [u64]
        L.oracle_fmix64_export.restype = u64
        _lib = L
    return _lib


@dataclasses.dataclass
class OracleResult:
    """Groups in lexicographic key order. keys: (G, K) int64 (widened codes)."""
    keys: np.ndarray
    count: np.ndarray
    aggs: List[np.ndarray]     # per aggregate, dtype per Schema.agg_out_dtype (MIN/MAX int -> int64)
    sumabs: List[Optional[np.ndarray]]  # per aggregate: sum |v| for f64 SUM/AVG, else None

    @property
    def n_groups(self) -> int:
        return int(self.count.shape[0])


def _schema_struct(s: blugen.Schema):
    kd = (ctypes.c_int32 * max(1, len(s.keys)))(*[d for d, _ in s.keys])
    vd = (ctypes.c_int32 * max(1, len(s.vals)))(*s.vals)
    ops = (ctypes.c_int32 * max(1, len(s.aggs)))(*[o for o, _ in s.aggs])
    cols = (ctypes.c_int32 * max(1, len(s.aggs)))(*[c for _, c in s.aggs])
    st = OracleSchema(len(s.keys), kd, len(s.vals), vd, len(s.aggs), ops, cols)
    return st, (kd, vd, ops, cols)


def _fetch(h, s: blugen.Schema) -> OracleResult:
    L = lib()
    G = int(L.oracle_n_groups(h))
    K = len(s.keys)
    keys = np.zeros((G, K), np.int64)
    count = np.zeros(G, np.int64)
    aggs, sumabs = [], []
    for a, (op, col) in enumerate(s.aggs):
        od = s.agg_out_dtype(a)
        aggs.append(np.zeros((G, 2) if od == I128 else G, np.float64 if od == F64 else np.int64))
        f64_in = op in (SUM, AVG) and s.vals[col] == F64
        sumabs.append(np.zeros(G, np.float64) if f64_in else None)
    agg_ptrs = (ctypes.c_void_p * max(1, len(aggs)))(*[x.ctypes.data for x in aggs])
    sa_ptrs = (ctypes.c_void_p * max(1, len(aggs)))(*[(x.ctypes.data if x is not None else None) for x in sumabs])
    L.oracle_fetch(h, keys.ctypes.data, count.ctypes.data, agg_ptrs, sa_ptrs)
    L.oracle_free(h)
    return OracleResult(keys, count, aggs, sumabs)


def _filter_arg(filter_keys, K):
    if filter_keys is None:
        return None, 0, None
    fk = np.ascontiguousarray(np.asarray(filter_keys, np.int64).reshape(-1, K))
    return fk.ctypes.data, fk.shape[0], fk


def groupby_arrays(schema: blugen.Schema, key_cols: Sequence[np.ndarray], val_cols: Sequence[np.ndarray],
                   slice_p: int = 0, slice_P: int = 1, filter_keys=None) -> OracleResult:
    n = len(key_cols[0]) if key_cols else 0
    kc = [np.ascontiguousarray(k, blugen.NP_DTYPE[d]) for k, (d, _) in zip(key_cols, schema.keys)]
    vc = [np.ascontiguousarray(v, blugen.NP_DTYPE[d]) for v, d in zip(val_cols, schema.vals)]
    kp = (ctypes.c_void_p * max(1, len(kc)))(*[k.ctypes.data for k in kc])
    vp = (ctypes.c_void_p * max(1, len(vc)))(*[v.ctypes.data for v in vc])
    st, keep = _schema_struct(schema)
    fp, nf, fkeep = _filter_arg(filter_keys, len(schema.keys))
    h = lib().oracle_groupby_arrays(ctypes.byref(st), kp, vp, n, slice_p, slice_P, fp, nf)
    return _fetch(h, schema)


def groupby_generated(w: blugen.Workload, row0: int = 0, n: Optional[int] = None, slice_p: int = 0,
                      slice_P: int = 1, filter_keys=None) -> OracleResult:
    n = w.n_rows - row0 if n is None else n
    ks, vs, keep = blugen.host_specs(w)
    st, skeep = _schema_struct(w.schema)
    fp, nf, fkeep = _filter_arg(filter_keys, len(w.schema.keys))
    h = lib().oracle_groupby_generated(ctypes.byref(st), ks, vs, row0, n, slice_p, slice_P, fp, nf)
    return _fetch(h, w.schema)


def concat(results: Sequence[OracleResult]) -> OracleResult:
    """Union of key-disjoint slices, re-sorted lexicographically by key tuple."""
    keys = np.concatenate([r.keys for r in results])
    order = np.lexsort(keys.T[::-1]) if keys.shape[0] else np.arange(0)
    aggs = [np.concatenate([r.aggs[a] for r in results])[order] for a in range(len(results[0].aggs))]
    sumabs = []
    for a in range(len(results[0].aggs)):
        if results[0].sumabs[a] is None:
            sumabs.append(None)
        else:
            sumabs.append(np.concatenate([r.sumabs[a] for r in results])[order])
    return OracleResult(keys[order], np.concatenate([r.count for r in results])[order], aggs, sumabs)


# ---- sort offload (§3; oracle/sort_oracle.cpp) -----------------------------------
def partial_keys(rows: np.ndarray, word: int) -> np.ndarray:
    """4-byte binary-sortable partial keys of word `word` of (n, W) uint8 rows."""
    rows = np.ascontiguousarray(rows, np.uint8)
    n, W = rows.shape
    out = np.zeros(n, np.uint32)
    lib().oracle_partial_keys(rows.ctypes.data, n, W, word, out.ctypes.data)
    return out


def sort_pairs(keys: np.ndarray, payload: np.ndarray):
    """Stable sort of the partial key buffer by its 4-byte key."""
    k = np.ascontiguousarray(keys, np.uint32)
    p = np.ascontiguousarray(payload, np.uint32)
    ko, po = np.zeros_like(k), np.zeros_like(p)
    lib().oracle_sort_pairs(k.ctypes.data, p.ctypes.data, len(k), ko.ctypes.data, po.ctypes.data)
    return ko, po


def dup_ranges(sorted_keys: np.ndarray):
    """(starts, lens) of the duplicate ranges of a sorted buffer."""
    k = np.ascontiguousarray(sorted_keys, np.uint32)
    m = max(1, len(k) // 2)
    st, ln = np.zeros(m, np.uint64), np.zeros(m, np.uint64)
    r = lib().oracle_dup_ranges(k.ctypes.data, len(k), st.ctypes.data, ln.ctypes.data)
    return st[:r].astype(np.int64), ln[:r].astype(np.int64)


def sort_rows(rows: np.ndarray) -> np.ndarray:
    """The completed sort: stable lexicographic order of (n, W) uint8 rows, as row indices."""
    rows = np.ascontiguousarray(rows, np.uint8)
    n, W = rows.shape
    out = np.zeros(n, np.uint32)
    lib().oracle_sort_rows(rows.ctypes.data, n, W, out.ctypes.data)
    return out


# ---- KMV group-count estimate (oracle/kmv_oracle.cpp) --------------------------------
def kmv(key_cols: Sequence[np.ndarray], dict_sizes: Sequence[int], k: int):
    """(estimate, exact) of the number of distinct key tuples: the k-th smallest distinct
    fmix64(concatenated key ^ salt), est = (k - 1) * 2^64 / U_(k); exact count below k."""
    cols = [np.ascontiguousarray(c) for c in key_cols]
    for c in cols:
        assert c.dtype in (np.int32, np.int64), c.dtype
    n = len(cols[0]) if cols else 0
    kp = (ctypes.c_void_p * max(1, len(cols)))(*[c.ctypes.data for c in cols])
    is64 = (ctypes.c_int32 * max(1, len(cols)))(*[1 if c.dtype == np.int64 else 0 for c in cols])
    ds = (ctypes.c_uint64 * max(1, len(cols)))(*[int(d) for d in dict_sizes])
    ex = ctypes.c_int32(0)
    est = lib().oracle_kmv(kp, is64, ds, len(cols), n, k, ctypes.byref(ex))
    return float(est), bool(ex.value)


def fmix64(x: int) -> int:
    """The oracle's Murmur3 finalizer (for its bijectivity pin)."""
    return int(lib().oracle_fmix64_export(x))
