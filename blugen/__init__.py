"""blugen — seeded synthetic columnar inputs and the workload definitions (C1..C5).

Input infrastructure shared by the oracle (oracle/) and the CUDA path's tests/bench. It holds
NONE of the GROUP BY arithmetic: it only describes and generates columns. Every column is a pure
function of (spec, global row index), evaluated by include/blu_gen.h on the host (numpy arrays)
or on the device (libblugen.so kernel writing into a torch tensor).

Workloads follow SURVEY.md §8(d) / BASELINE.json "configs": a star-schema fact table shaped like
the paper's TPC-DS store_sales workload (Fig. 4), dictionary-encoded grouping
codes and quantity / money payload columns.
"""
from __future__ import annotations

import ctypes
import dataclasses
import os
from typing import List, Optional, Sequence, Tuple

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libblugen.so")

# dtype / op numbering — identical to include/blu_gby.h (by convention; no shared code).
I32, I64, F64, I128 = 0, 1, 2, 3  # I128 columns: int64 arrays of shape (n, 2) = (lo, hi) words
COUNT, SUM, MIN, MAX, AVG = 0, 1, 2, 3, 4
DTYPE_NAMES = {I32: "i32", I64: "i64", F64: "f64", I128: "i128"}
OP_NAMES = {COUNT: "COUNT", SUM: "SUM", MIN: "MIN", MAX: "MAX", AVG: "AVG"}
NP_DTYPE = {I32: np.int32, I64: np.int64, F64: np.float64, I128: np.int64}

# generator kinds (blu_gen_kind_t)
UNIFORM, DYADIC, SPARSE_KEY, ZIPF_DIGIT, CYCLIC_DIGIT, LINEAR, REAL, UNIFORM_DIGIT = range(8)


class GenSpec(ctypes.Structure):
    _fields_ = [
        ("kind", ctypes.c_int32),
        ("dtype", ctypes.c_int32),
        ("seed", ctypes.c_uint64),
        ("stream", ctypes.c_uint64),
        ("lo", ctypes.c_int64),
        ("hi", ctypes.c_int64),
        ("n_groups", ctypes.c_uint64),
        ("stride", ctypes.c_uint64),
        ("radix", ctypes.c_uint64),
        ("zipf_cdf", ctypes.c_void_p),
        ("perm", ctypes.c_void_p),
        ("table_n", ctypes.c_uint64),
    ]


@dataclasses.dataclass
class Col:
    """One synthetic column: dtype + generator recipe."""
    dtype: int
    kind: int
    stream: int
    lo: int = 0
    hi: int = 0
    n_groups: int = 0
    stride: int = 1
    radix: int = 1
    zipf_n: int = 0      # ZIPF_DIGIT: number of ranks
    zipf_s: float = 0.0  # ZIPF_DIGIT: exponent


@dataclasses.dataclass
class Schema:
    """keys: [(dtype, dict_size)] (dict_size 0 = sparse code); vals: [dtype]; aggs: [(op, col)]."""
    keys: List[Tuple[int, int]]
    vals: List[int]
    aggs: List[Tuple[int, int]]

    def agg_out_dtype(self, a: int) -> int:
        op, col = self.aggs[a]
        if op == COUNT:
            return I64
        if op == AVG:
            return F64
        vd = self.vals[col]
        if op == SUM:
            return vd if vd in (F64, I128) else I64
        return vd  # MIN / MAX keep the input dtype


@dataclasses.dataclass
class Workload:
    name: str
    n_rows: int
    seed: int
    key_cols: List[Col]
    val_cols: List[Col]
    schema: Schema
    est_groups: int
    expected_groups: int
    note: str = ""

    @property
    def bytes_per_row(self) -> int:
        return sum(4 if c.dtype == I32 else 8 for c in self.key_cols + self.val_cols)


_lib = None


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} missing: run `make` (or __graft_entry__.build())")
        L = ctypes.CDLL(LIB_PATH)
        L.blu_gen_fill_host.argtypes = [ctypes.POINTER(GenSpec), ctypes.c_uint64, ctypes.c_uint64, ctypes.c_void_p]
        L.blu_gen_fill_host.restype = ctypes.c_int
        L.blu_gen_fill_device.argtypes = [ctypes.POINTER(GenSpec), ctypes.c_uint64, ctypes.c_uint64,
                                          ctypes.c_void_p, ctypes.c_void_p]
        L.blu_gen_fill_device.restype = ctypes.c_int
        L.blu_gen_zipf_table.argtypes = [ctypes.c_uint64, ctypes.c_double, ctypes.c_void_p]
        L.blu_gen_zipf_table.restype = None
        L.blu_gen_permutation.argtypes = [ctypes.c_uint64, ctypes.c_uint64, ctypes.c_void_p]
        L.blu_gen_permutation.restype = None
        _lib = L
    return _lib


_table_cache = {}


def zipf_tables(n: int, s: float, seed: int):
    """(cdf u64[n], perm u32[n]) host tables for a ZIPF_DIGIT column; cached."""
    k = (n, s, seed)
    if k not in _table_cache:
        cdf = np.empty(n, np.uint64)
        perm = np.empty(n, np.uint32)
        lib().blu_gen_zipf_table(n, s, cdf.ctypes.data)
        lib().blu_gen_permutation(n, seed ^ 0x7E57, perm.ctypes.data)
        _table_cache[k] = (cdf, perm)
    return _table_cache[k]


def make_spec(col: Col, seed: int, cdf_ptr: int = 0, perm_ptr: int = 0) -> GenSpec:
    return GenSpec(col.kind, col.dtype, seed, col.stream, col.lo, col.hi, col.n_groups, col.stride,
                   col.radix, cdf_ptr, perm_ptr, col.zipf_n)


def host_spec(col: Col, seed: int) -> Tuple[GenSpec, tuple]:
    """Spec with host table pointers (keep the returned tables alive while using the spec)."""
    if col.kind == ZIPF_DIGIT:
        cdf, perm = zipf_tables(col.zipf_n, col.zipf_s, seed)
        return make_spec(col, seed, cdf.ctypes.data, perm.ctypes.data), (cdf, perm)
    return make_spec(col, seed), ()


def gen_host(col: Col, seed: int, row0: int, n: int) -> np.ndarray:
    out = np.empty(n, NP_DTYPE[col.dtype])
    spec, keep = host_spec(col, seed)
    if n:
        rc = lib().blu_gen_fill_host(ctypes.byref(spec), row0, n, out.ctypes.data)
        assert rc == 0
    del keep
    return out


_dev_tables = {}


def gen_device(col: Col, seed: int, row0: int, n: int, device="cuda", out=None, stream=None):
    """Generate rows row0..row0+n-1 of `col` directly in HBM (torch tensor)."""
    import torch
    tdt = {I32: torch.int32, I64: torch.int64, F64: torch.float64}[col.dtype]
    if out is None:
        out = torch.empty(n, dtype=tdt, device=device)
    cdf_p = perm_p = 0
    if col.kind == ZIPF_DIGIT:
        key = (col.zipf_n, col.zipf_s, seed, str(out.device))
        if key not in _dev_tables:
            cdf, perm = zipf_tables(col.zipf_n, col.zipf_s, seed)
            _dev_tables[key] = (torch.from_numpy(cdf.view(np.int64)).to(out.device),
                                torch.from_numpy(perm.view(np.int32)).to(out.device))
        cdf_p, perm_p = _dev_tables[key][0].data_ptr(), _dev_tables[key][1].data_ptr()
    spec = make_spec(col, seed, cdf_p, perm_p)
    if stream is None:
        stream = torch.cuda.current_stream(out.device).cuda_stream
    if n:
        rc = lib().blu_gen_fill_device(ctypes.byref(spec), row0, n, out.data_ptr(), stream)
        assert rc == 0, rc
    return out


# ----------------------------------------------------------------------------------------------
# Workloads (BASELINE.json "configs"). Seed = 0x5EED0000 + config.
# ----------------------------------------------------------------------------------------------

def _c1(n_rows=1_000_000) -> Workload:
    seed = 0x5EED0001
    keys = [Col(I32, UNIFORM, 0, 0, 16)]
    vals = [Col(I64, UNIFORM, 1, -(2**31), 2**31)]
    sch = Schema([(I32, 16)], [I64], [(COUNT, -1), (SUM, 0)])
    return Workload("C1", n_rows, seed, keys, vals, sch, 16, 16,
                    "1 i32 dict-16 key, 1 i64 value; COUNT, SUM")


def _c2(n_rows=100_000_000) -> Workload:
    seed = 0x5EED0002
    keys = [Col(I32, UNIFORM, 0, 0, 32), Col(I32, UNIFORM, 1, 0, 32)]
    vals = [Col(I32, UNIFORM, 2, 1, 101), Col(I64, UNIFORM, 3, 0, 10**7),
            Col(I64, UNIFORM, 4, -(10**7), 10**7), Col(F64, DYADIC, 5)]
    sch = Schema([(I32, 32), (I32, 32)], [I32, I64, I64, F64],
                 [(COUNT, -1), (SUM, 0), (MIN, 1), (MAX, 2), (AVG, 3)])
    return Workload("C2", n_rows, seed, keys, vals, sch, 1024, 1024,
                    "2 i32 keys 32x32, 4 values; COUNT, SUM, MIN, MAX, AVG")


def _c3(n_rows=1_000_000_000, n_groups=10_000_000) -> Workload:
    seed = 0x5EED0003
    keys = [Col(I64, SPARSE_KEY, 0, n_groups=n_groups)]
    vals = [Col(I64, UNIFORM, 1, -(2**31), 2**31), Col(F64, DYADIC, 2)]
    sch = Schema([(I64, 0)], [I64, F64], [(COUNT, -1), (SUM, 0), (AVG, 1)])
    return Workload("C3", n_rows, seed, keys, vals, sch, n_groups, n_groups,
                    "1 sparse i64 key, uniform over G codes; COUNT, SUM, AVG")


def _c4(n_rows=1_000_000_000) -> Workload:
    seed = 0x5EED0004
    D = 100 * 50 * 20
    z = dict(zipf_n=D, zipf_s=1.1)
    keys = [Col(I32, ZIPF_DIGIT, 0, stride=1, radix=100, **z),
            Col(I32, ZIPF_DIGIT, 0, stride=100, radix=50, **z),
            Col(I32, ZIPF_DIGIT, 0, stride=5000, radix=20, **z)]
    vals = [Col(I32, UNIFORM, 1, 1, 101), Col(I64, UNIFORM, 2, 0, 10**7),
            Col(I64, UNIFORM, 3, -(10**7), 10**7)]
    sch = Schema([(I32, 100), (I32, 50), (I32, 20)], [I32, I64, I64],
                 [(COUNT, -1), (SUM, 0), (SUM, 1), (AVG, 1), (SUM, 2), (MIN, 2), (MAX, 2)])
    return Workload("C4", n_rows, seed, keys, vals, sch, D, D,
                    "3 i32 keys 100x50x20, Zipf(1.1) composite rank; 7 aggregates")


def _c5(n_rows=4_000_000_000, n_groups=50_000_000) -> Workload:
    seed = 0x5EED0005
    keys = [Col(I64, SPARSE_KEY, 0, n_groups=n_groups)]
    vals = [Col(I64, UNIFORM, 1, -(10**9), 10**9), Col(F64, DYADIC, 2)]
    sch = Schema([(I64, 0)], [I64, F64], [(COUNT, -1), (SUM, 0), (AVG, 1)])
    return Workload("C5", n_rows, seed, keys, vals, sch, n_groups, n_groups,
                    "1 sparse i64 key, 50M groups; COUNT, SUM, AVG; sharded over GPUs")


def _k3(n_rows=100_000_000, n_groups=50_000_000) -> Workload:
    """Kernel-3 study: many aggregates (8 state fields) and a low
    rows/groups ratio (2 rows per group) — where the paper prefers one row lock over per-field atomics."""
    seed = 0x5EED0013
    keys = [Col(I64, SPARSE_KEY, 0, n_groups=n_groups)]
    vals = [Col(I32, UNIFORM, 1, 1, 101), Col(I64, UNIFORM, 2, 0, 10**7), Col(F64, DYADIC, 3),
            Col(I64, UNIFORM, 4, -(10**9), 10**9)]
    sch = Schema([(I64, 0)], [I32, I64, F64, I64],
                 [(COUNT, -1), (SUM, 0), (MIN, 0), (MAX, 0), (SUM, 1), (AVG, 2), (MIN, 3), (MAX, 3)])
    return Workload("K3", n_rows, seed, keys, vals, sch, n_groups, n_groups,
                    "kernel-3 study: sparse i64 key, 2 rows/group, 8 aggregates")


WORKLOADS = {"C1": _c1, "C2": _c2, "C3": _c3, "C4": _c4, "C5": _c5, "K3": _k3}


def workload(name: str, n_rows: Optional[int] = None, n_groups: Optional[int] = None) -> Workload:
    f = WORKLOADS[name]
    kw = {}
    if n_rows is not None:
        kw["n_rows"] = n_rows
    if n_groups is not None:
        kw["n_groups"] = n_groups
    return f(**kw)


def host_columns(w: Workload, row0: int = 0, n: Optional[int] = None):
    n = w.n_rows - row0 if n is None else n
    return ([gen_host(c, w.seed, row0, n) for c in w.key_cols],
            [gen_host(c, w.seed, row0, n) for c in w.val_cols])


def device_columns(w: Workload, row0: int = 0, n: Optional[int] = None, device="cuda"):
    n = w.n_rows - row0 if n is None else n
    return ([gen_device(c, w.seed, row0, n, device) for c in w.key_cols],
            [gen_device(c, w.seed, row0, n, device) for c in w.val_cols])


def host_specs(w: Workload):
    """(key GenSpec array, val GenSpec array, keepalive) with host table pointers."""
    keep = []
    ks = (GenSpec * max(1, len(w.key_cols)))()
    vs = (GenSpec * max(1, len(w.val_cols)))()
    for i, c in enumerate(w.key_cols):
        ks[i], k = host_spec(c, w.seed)
        keep.append(k)
    for i, c in enumerate(w.val_cols):
        vs[i], k = host_spec(c, w.seed)
        keep.append(k)
    return ks, vs, keep


# ---- sort offload workload (§3) ---------------------------------
SORT_SEED = 0x5EED0050


def sort_rows(n: int, W: int = 16, seed: int = SORT_SEED, cards=(1823, 502)) -> np.ndarray:
    """(n, W) uint8 binary-sortable keys (W a multiple of 4) shaped like an ORDER BY over TPC-DS
    store_sales: 4-byte word 0 a sold-date code (1823 distinct), word 1 a store code (502
    distinct), the remaining words uniform random bytes (item / ticket). Each word is stored most
    significant byte first, so lexicographic byte order is numeric order per word. Seeded numpy
    generator; no sort arithmetic here."""
    assert W % 4 == 0 and W >= 4
    rng = np.random.default_rng(seed)
    words = []
    for w in range(W // 4):
        if w < len(cards) and cards[w]:
            words.append(rng.integers(0, cards[w], n, dtype=np.uint32))
        else:
            words.append(rng.integers(0, 2**32, n, dtype=np.uint32))
    be = np.stack(words, axis=1).astype(">u4")
    return np.ascontiguousarray(be.view(np.uint8).reshape(n, W))
