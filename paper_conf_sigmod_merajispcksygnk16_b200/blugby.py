"""Thin ctypes binding of libblugby (include/blu_gby.h). Argument marshalling only.

Every step of the GROUP BY runs in libblugby's sm_100a kernels; this module converts torch tensors
/ numpy arrays to pointers, calls the C ABI with the same names, and wraps the library-owned result
arrays as zero-copy torch tensors. There is no fallback: if libblugby.so is missing the import of
this module raises.
"""
from __future__ import annotations

import ctypes
import os
from typing import List, Optional, Sequence, Tuple

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libblugby.so")

# enums (include/blu_gby.h)
BLU_OK, BLU_E_INVALID, BLU_E_UNSUPPORTED, BLU_E_KEY_RANGE, BLU_E_OOM, BLU_E_CUDA = range(6)
BLU_I32, BLU_I64, BLU_F64, BLU_I128 = 0, 1, 2, 3  # I128: int64 tensors of shape (n, 2) = (lo, hi)
BLU_COUNT, BLU_SUM, BLU_MIN, BLU_MAX, BLU_AVG = range(5)
BLU_PATH_DENSE_SMEM, BLU_PATH_HASH_GLOBAL, BLU_PATH_DIRECT_GLOBAL = range(3)
PATH_NAMES = {0: "a:dense_smem", 1: "b:hash_global", 2: "b':direct_global"}
STATUS_NAMES = {0: "BLU_OK", 1: "BLU_E_INVALID", 2: "BLU_E_UNSUPPORTED", 3: "BLU_E_KEY_RANGE",
                4: "BLU_E_OOM", 5: "BLU_E_CUDA"}


class BluError(RuntimeError):
    def __init__(self, status: int, detail: str):
        super().__init__(f"{STATUS_NAMES.get(status, status)}: {detail}")
        self.status = status


class KeyDesc(ctypes.Structure):
    _fields_ = [("dtype", ctypes.c_int32), ("dict_size", ctypes.c_uint64)]


class AggDesc(ctypes.Structure):
    _fields_ = [("op", ctypes.c_int32), ("val_col", ctypes.c_int32)]


class SchemaC(ctypes.Structure):
    _fields_ = [("n_keys", ctypes.c_int32), ("keys", ctypes.POINTER(KeyDesc)),
                ("n_vals", ctypes.c_int32), ("vals", ctypes.POINTER(ctypes.c_int32)),
                ("n_aggs", ctypes.c_int32), ("aggs", ctypes.POINTER(AggDesc))]


class ResultC(ctypes.Structure):
    _fields_ = [("n_groups", ctypes.c_uint64), ("n_keys", ctypes.c_int32), ("n_aggs", ctypes.c_int32),
                ("n_states", ctypes.c_int32), ("is_partial", ctypes.c_int32), ("is_host", ctypes.c_int32),
                ("key_cols", ctypes.POINTER(ctypes.c_void_p)), ("agg_cols", ctypes.POINTER(ctypes.c_void_p)),
                ("state_cols", ctypes.POINTER(ctypes.c_void_p)), ("_owner", ctypes.c_void_p)]


class PlanDescC(ctypes.Structure):
    _fields_ = [("path", ctypes.c_int32), ("capacity", ctypes.c_uint64), ("est_groups", ctypes.c_uint64),
                ("slot_bytes", ctypes.c_uint32), ("smem_bytes", ctypes.c_uint32), ("hot_front", ctypes.c_int32),
                ("front_slots", ctypes.c_uint32), ("partitions", ctypes.c_uint32), ("n_states", ctypes.c_int32),
                ("state_dtypes", ctypes.c_int32 * 32), ("grid", ctypes.c_uint32), ("block", ctypes.c_uint32),
                ("retries_last", ctypes.c_uint32), ("row_lock", ctypes.c_int32), ("part_smem", ctypes.c_int32),
                ("bucket_entries", ctypes.c_uint32)]


class TimingC(ctypes.Structure):
    _fields_ = [("init_ms", ctypes.c_float), ("aggregate_ms", ctypes.c_float), ("compact_ms", ctypes.c_float),
                ("h2d_ms", ctypes.c_float), ("total_ms", ctypes.c_float),
                ("aggregate_launches", ctypes.c_uint32), ("retries", ctypes.c_uint32), ("kernel", ctypes.c_char * 64),
                ("scatter_ms", ctypes.c_float), ("pass2_ms", ctypes.c_float), ("part_chunks", ctypes.c_uint32),
                ("part_fallbacks", ctypes.c_uint32)]


class SortStatsC(ctypes.Structure):
    _fields_ = [("levels", ctypes.c_uint32), ("ranges", ctypes.c_uint64 * 256), ("active", ctypes.c_uint64 * 256),
                ("ms", ctypes.c_float * 256), ("downsweep_ms", ctypes.c_float), ("downsweep_launches", ctypes.c_uint32),
                ("downsweep_bytes", ctypes.c_uint64)]


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"libblugby.so not built ({LIB_PATH}); run `make` or __graft_entry__.build()")
    L = ctypes.CDLL(LIB_PATH)
    vp, u64, i32, u32 = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int32, ctypes.c_uint32
    P = ctypes.POINTER
    sigs = {
        "blu_gby_plan": ([P(SchemaC), u64, u64, P(vp)], i32),
        "blu_gby_plan_info": ([vp, P(i32), P(u64), P(u32), P(u32)], i32),
        "blu_gby_plan_describe": ([vp, P(PlanDescC)], i32),
        "blu_gby_execute": ([vp, P(vp), P(vp), u64, vp, P(ResultC)], i32),
        "blu_gby_execute_host": ([vp, P(vp), P(vp), u64, vp, P(ResultC)], i32),
        "blu_gby_execute_partial": ([vp, P(vp), P(vp), u64, vp, P(ResultC)], i32),
        "blu_gby_merge": ([vp, P(ResultC), i32, vp, P(ResultC)], i32),
        "blu_gby_merge_partial": ([vp, P(ResultC), i32, vp, P(ResultC)], i32),
        "blu_gby_dense_state_shape": ([vp, P(i32), P(i32), P(i32), P(i32), P(u64)], i32),
        "blu_gby_execute_dense_state": ([vp, P(vp), P(vp), u64, vp, P(vp), i32], i32),
        "blu_gby_finalize_dense_state": ([vp, P(vp), vp, P(ResultC)], i32),
        "blu_gby_partition": ([vp, P(ResultC), i32, vp, vp, P(u64)], i32),
        "blu_gby_merge_records": ([vp, vp, u64, vp, i32, P(ResultC)], i32),
        "blu_gby_record_bytes": ([vp], u32),
        "blu_gby_row_record_bytes": ([vp], u32),
        "blu_gby_partition_rows": ([vp, P(vp), P(vp), u64, i32, vp, vp, P(u64)], i32),
        "blu_gby_execute_records": ([vp, vp, u64, vp, i32, P(ResultC)], i32),
        "blu_gby_estimate_groups": ([P(KeyDesc), i32, P(vp), u64, u32, vp, P(ctypes.c_double), P(i32)], i32),
        "blu_gby_slot_template": ([vp, vp, u32, P(u32)], i32),
        "blu_gby_init_table": ([vp, vp, u64, vp], i32),
        "blu_gby_set_timing": ([i32], None),
        "blu_sort_partial_keys": ([vp, u64, ctypes.c_uint32, ctypes.c_uint32, vp, vp], i32),
        "blu_sort_pairs": ([vp, vp, u64, vp, vp, vp], i32),
        "blu_sort_dup_ranges": ([vp, u64, vp, vp, u64, P(u64), vp], i32),
        "blu_sort_rows": ([vp, u64, ctypes.c_uint32, vp, vp, P(SortStatsC)], i32),
        "blu_gby_last_timing": ([P(TimingC)], i32),
        "blu_gby_launch_count": ([], u64),
        "blu_gby_read_roofline": ([P(vp), P(u64), i32, vp, vp], i32),
        "blu_gby_jit_probe": ([vp, ctypes.c_char_p, u32, P(i32)], i32),
        "blu_gby_bind_device": ([i32], i32),
        "blu_gby_release_workspace": ([P(u64)], i32),
        "blu_gby_result_free": ([P(ResultC), vp], None),
        "blu_gby_plan_destroy": ([vp], None),
        "blu_gby_status_str": ([i32], ctypes.c_char_p),
        "blu_gby_last_error": ([], ctypes.c_char_p),
    }
    for name, (args, res) in sigs.items():
        f = getattr(L, name)
        f.argtypes = args
        f.restype = res
    return L


lib = _load()


def _check(status: int):
    if status != BLU_OK:
        raise BluError(status, lib.blu_gby_last_error().decode(errors="replace"))


def _ptrs(cols) -> ctypes.Array:
    arr = (ctypes.c_void_p * max(1, len(cols)))()
    for i, c in enumerate(cols):
        arr[i] = _ptr(c)
    return arr


def _ptr(c) -> int:
    if c is None:
        return 0
    if hasattr(c, "data_ptr"):
        return c.data_ptr()
    if hasattr(c, "ctypes"):
        return c.ctypes.data
    return int(c)


def _stream_handle(stream) -> int:
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    if hasattr(stream, "cuda_stream"):
        return stream.cuda_stream
    return int(stream)


# ---------------------------------------------------------------------------------------------
# plan
# ---------------------------------------------------------------------------------------------
class Plan:
    """An immutable blu_gby_plan_t (freed on garbage collection)."""

    def __init__(self, handle: int, keys, vals, aggs):
        self.handle = handle
        self.keys = list(keys)
        self.vals = list(vals)
        self.aggs = list(aggs)

    def __del__(self):
        h, self.handle = getattr(self, "handle", None), None
        if h:
            try:
                lib.blu_gby_plan_destroy(h)
            except Exception:
                pass

    def info(self) -> dict:
        d = PlanDescC()
        _check(lib.blu_gby_plan_describe(self.handle, ctypes.byref(d)))
        out = {k: getattr(d, k) for k, _ in PlanDescC._fields_ if k != "state_dtypes"}
        out["state_dtypes"] = [d.state_dtypes[i] for i in range(d.n_states)]
        out["path_name"] = PATH_NAMES[d.path]
        return out

    def dense_state_shape(self) -> Tuple[int, int, int, int, int]:
        a, b, c, d, D = ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int32(), ctypes.c_uint64()
        _check(lib.blu_gby_dense_state_shape(self.handle, ctypes.byref(a), ctypes.byref(b), ctypes.byref(c),
                                             ctypes.byref(d), ctypes.byref(D)))
        return a.value, b.value, c.value, d.value, D.value

    def slot_template(self) -> bytes:
        sb = ctypes.c_uint32()
        _check(lib.blu_gby_slot_template(self.handle, None, 0, ctypes.byref(sb)))
        buf = (ctypes.c_uint8 * sb.value)()
        _check(lib.blu_gby_slot_template(self.handle, buf, sb.value, ctypes.byref(sb)))
        return bytes(buf)

    @property
    def record_bytes(self) -> int:
        return int(lib.blu_gby_record_bytes(self.handle))

    @property
    def row_record_bytes(self) -> int:
        return int(lib.blu_gby_row_record_bytes(self.handle))


def blu_gby_plan(keys: Sequence[Tuple[int, int]], vals: Sequence[int], aggs: Sequence[Tuple[int, int]],
                 est_groups: int, n_rows: int) -> Plan:
    """keys: [(dtype, dict_size)], vals: [dtype], aggs: [(op, val_col)] (COUNT: val_col -1)."""
    kd = (KeyDesc * max(1, len(keys)))(*[KeyDesc(int(d), int(s)) for d, s in keys])
    vd = (ctypes.c_int32 * max(1, len(vals)))(*[int(v) for v in vals])
    ad = (AggDesc * max(1, len(aggs)))(*[AggDesc(int(o), int(c)) for o, c in aggs])
    sc = SchemaC(len(keys), kd, len(vals), vd, len(aggs), ad)
    h = ctypes.c_void_p()
    _check(lib.blu_gby_plan(ctypes.byref(sc), int(est_groups), int(n_rows), ctypes.byref(h)))
    return Plan(h.value, keys, vals, aggs)


def plan_for(schema, est_groups: int, n_rows: int) -> Plan:
    """Plan from any object with .keys / .vals / .aggs (e.g. blugen.Schema)."""
    return blu_gby_plan(schema.keys, schema.vals, schema.aggs, est_groups, n_rows)


def plan_estimated(schema, key_cols, n_rows: Optional[int] = None, k: int = 2048, stream=None) -> Plan:
    """The paper's pipeline: KMV-estimate the group count on the device, then plan."""
    est, _ = blu_gby_estimate_groups(schema.keys, key_cols, k=k, n_rows=n_rows, stream=stream)
    n = int(len(key_cols[0]) if n_rows is None else n_rows)
    return blu_gby_plan(schema.keys, schema.vals, schema.aggs, max(1, int(round(est))), n)


# ---------------------------------------------------------------------------------------------
# results
# ---------------------------------------------------------------------------------------------
_TORCH_DT = None


def _torch_dtype(dt):
    global _TORCH_DT
    import torch
    if _TORCH_DT is None:
        _TORCH_DT = {BLU_I32: torch.int32, BLU_I64: torch.int64, BLU_F64: torch.float64, BLU_I128: torch.int64}
    return _TORCH_DT[dt]


class _Owner:
    """Owns one library result (blu_gby_result_t) and frees it when the last reference goes away.
    Result objects and every zero-copy tensor view reference the owner — never the other way round —
    so no reference cycle delays the free until a garbage-collection pass."""

    def __init__(self, rc: ResultC, stream: int):
        self.rc = rc
        self.stream = stream

    def free(self):
        rc, self.rc = self.rc, None
        if rc is not None and rc._owner:
            try:
                lib.blu_gby_result_free(ctypes.byref(rc), self.stream)
            except Exception:
                pass

    def __del__(self):
        self.free()


class _DevArray:
    """__cuda_array_interface__ provider that keeps the result's owner alive while a tensor views it."""

    def __init__(self, owner: _Owner, ptr: int, n: int, dt: int):
        typestr = {BLU_I32: "<i4", BLU_I64: "<i8", BLU_F64: "<f8", BLU_I128: "<i8"}[dt]
        self._owner = owner
        shape = (n, 2) if dt == BLU_I128 else (n,)
        self.__cuda_array_interface__ = {"shape": shape, "typestr": typestr, "data": (ptr if n else 0, False),
                                         "version": 3, "strides": None}


class _HostArray:
    """__array_interface__ provider for a host result column: numpy views it without a copy and keeps
    the result's owner (which frees the library's host memory) alive while any view exists."""

    def __init__(self, owner: _Owner, ptr: int, n: int, dt: int):
        typestr = {BLU_I32: "<i4", BLU_I64: "<i8", BLU_F64: "<f8", BLU_I128: "<i8"}[dt]
        self._owner = owner
        shape = (n, 2) if dt == BLU_I128 else (n,)
        self.__array_interface__ = {"shape": shape, "typestr": typestr, "data": (ptr, False), "version": 3}


class Result:
    """A blu_gby_result_t. keys / aggs / states are torch tensors (device, zero-copy) or numpy
    arrays (host results). Library memory is released when this object and every view are gone."""

    def __init__(self, rc: ResultC, key_dtypes: List[int], out_dtypes: List[int], stream: int, device=None):
        self._owner = _Owner(rc, stream)
        self.n_groups = int(rc.n_groups)
        self.is_partial = bool(rc.is_partial)
        self.is_host = bool(rc.is_host)
        self._spec = (key_dtypes, out_dtypes, device)
        self._cols = None  # the column views are built on first access (a caller that only needs
                           # n_groups pays no view construction)

    def _views(self):
        if self._cols is None:
            key_dtypes, out_dtypes, device = self._spec
            rc, n = self._owner.rc, self.n_groups
            if rc is None:
                raise BluError(BLU_E_INVALID, "result already freed")
            cols = rc.state_cols if self.is_partial else rc.agg_cols
            n_out = rc.n_states if self.is_partial else rc.n_aggs
            keys = [self._wrap(rc.key_cols[k], n, key_dtypes[k], device) for k in range(rc.n_keys)]
            vals = [self._wrap(cols[o], n, out_dtypes[o], device) for o in range(n_out)]
            self._cols = (keys, vals)
        return self._cols

    @property
    def keys(self):
        return self._views()[0]

    @property
    def aggs(self):
        return None if self.is_partial else self._views()[1]

    @property
    def states(self):
        return self._views()[1] if self.is_partial else None

    def _wrap(self, ptr, n, dt, device):
        if self.is_host:
            import numpy as np
            npdt = {BLU_I32: np.int32, BLU_I64: np.int64, BLU_F64: np.float64, BLU_I128: np.int64}[dt]
            w = 2 if dt == BLU_I128 else 1
            if n == 0:
                return np.zeros((0, 2) if w == 2 else 0, npdt)
            return np.asarray(_HostArray(self._owner, ptr, n, dt))  # zero-copy view of the library's host memory
        import torch
        if n == 0:
            return torch.zeros((0, 2) if dt == BLU_I128 else 0, dtype=_torch_dtype(dt), device=device or "cuda")
        return torch.as_tensor(_DevArray(self._owner, ptr, n, dt), device=device or "cuda")

    @property
    def c(self) -> ResultC:
        return self._owner.rc

    def free(self):
        """Release the library memory now (views become invalid)."""
        self._owner.free()


def _out_dtypes(plan: Plan, partial: bool) -> List[int]:
    if partial:
        return plan.info()["state_dtypes"]
    out = []
    for op, col in plan.aggs:
        if op == BLU_COUNT:
            out.append(BLU_I64)
        elif op == BLU_AVG:
            out.append(BLU_F64)
        elif op == BLU_SUM:
            out.append(plan.vals[col] if plan.vals[col] in (BLU_F64, BLU_I128) else BLU_I64)
        else:
            out.append(plan.vals[col])
    return out


def _key_dtypes(plan: Plan) -> List[int]:
    return [d for d, _ in plan.keys]


def _device_of(cols):
    for c in cols:
        if hasattr(c, "device"):
            return c.device
    return None


def blu_gby_execute(plan: Plan, key_cols, val_cols, n_rows: Optional[int] = None, stream=None) -> Result:
    n = int(len(key_cols[0]) if n_rows is None else n_rows)
    s = _stream_handle(stream)
    rc = ResultC()
    _check(lib.blu_gby_execute(plan.handle, _ptrs(key_cols), _ptrs(val_cols), n, s, ctypes.byref(rc)))
    r = Result(rc, _key_dtypes(plan), _out_dtypes(plan, False), s, _device_of(key_cols))
    if r.is_host:
        r.free()
    return r


def blu_gby_execute_partial(plan: Plan, key_cols, val_cols, n_rows: Optional[int] = None, stream=None) -> Result:
    n = int(len(key_cols[0]) if n_rows is None else n_rows)
    s = _stream_handle(stream)
    rc = ResultC()
    _check(lib.blu_gby_execute_partial(plan.handle, _ptrs(key_cols), _ptrs(val_cols), n, s, ctypes.byref(rc)))
    return Result(rc, _key_dtypes(plan), _out_dtypes(plan, True), s, _device_of(key_cols))


def blu_gby_execute_host(plan: Plan, key_cols, val_cols, n_rows: Optional[int] = None, stream=None) -> Result:
    """Host (numpy / pinned torch CPU) columns in, host (numpy) result out."""
    n = int(len(key_cols[0]) if n_rows is None else n_rows)
    s = _stream_handle(stream)
    rc = ResultC()
    _check(lib.blu_gby_execute_host(plan.handle, _ptrs(key_cols), _ptrs(val_cols), n, s, ctypes.byref(rc)))
    return Result(rc, _key_dtypes(plan), _out_dtypes(plan, False), s)


def _results_array(partials: Sequence[Result]):
    arr = (ResultC * max(1, len(partials)))()
    for i, p in enumerate(partials):
        arr[i] = p.c
    return arr


def blu_gby_merge(plan: Plan, partials: Sequence[Result], stream=None, partial_out: bool = False) -> Result:
    s = _stream_handle(stream)
    rc = ResultC()
    fn = lib.blu_gby_merge_partial if partial_out else lib.blu_gby_merge
    _check(fn(plan.handle, _results_array(partials), len(partials), s, ctypes.byref(rc)))
    dev = partials[0].keys[0].device if partials and partials[0].keys else None
    return Result(rc, _key_dtypes(plan), _out_dtypes(plan, partial_out), s, dev)


def blu_gby_merge_partial(plan: Plan, partials: Sequence[Result], stream=None) -> Result:
    return blu_gby_merge(plan, partials, stream, partial_out=True)


def blu_gby_merge_records(plan: Plan, records, n_records: int, stream=None, partial_out: bool = False) -> Result:
    s = _stream_handle(stream)
    rc = ResultC()
    _check(lib.blu_gby_merge_records(plan.handle, _ptr(records), int(n_records), s, int(partial_out),
                                     ctypes.byref(rc)))
    return Result(rc, _key_dtypes(plan), _out_dtypes(plan, partial_out), s, getattr(records, "device", None))


def blu_gby_partition(plan: Plan, partial: Result, n_parts: int, send_buf, stream=None) -> List[int]:
    s = _stream_handle(stream)
    counts = (ctypes.c_uint64 * n_parts)()
    _check(lib.blu_gby_partition(plan.handle, ctypes.byref(partial.c), n_parts, s, _ptr(send_buf), counts))
    return [int(c) for c in counts]


def blu_gby_partition_rows(plan: Plan, key_cols, val_cols, n_parts: int, send_buf, n_rows: Optional[int] = None,
                           stream=None) -> List[int]:
    """Rows mode of the exchange: raw rows bucketed by owner rank into send_buf (row records)."""
    n = int(len(key_cols[0]) if n_rows is None else n_rows)
    s = _stream_handle(stream)
    counts = (ctypes.c_uint64 * n_parts)()
    _check(lib.blu_gby_partition_rows(plan.handle, _ptrs(key_cols), _ptrs(val_cols), n, n_parts, s, _ptr(send_buf),
                                      counts))
    return [int(c) for c in counts]


def blu_gby_execute_records(plan: Plan, records, n_records: int, stream=None, partial_out: bool = False) -> Result:
    """S4-S8 over row records (the rows this rank owns after a rows-mode exchange)."""
    s = _stream_handle(stream)
    rc = ResultC()
    _check(lib.blu_gby_execute_records(plan.handle, _ptr(records), int(n_records), s, int(partial_out),
                                       ctypes.byref(rc)))
    return Result(rc, _key_dtypes(plan), _out_dtypes(plan, partial_out), s, getattr(records, "device", None))


def dense_state_arrays(plan: Plan, device="cuda"):
    """Allocate the 4 dense-state group arrays (int64 / f64 / int64 / int64) for this plan."""
    import torch
    ni, nf, nmin, nmax, D = plan.dense_state_shape()
    return [torch.empty(ni * D, dtype=torch.int64, device=device),
            torch.empty(nf * D, dtype=torch.float64, device=device),
            torch.empty(nmin * D, dtype=torch.int64, device=device),
            torch.empty(nmax * D, dtype=torch.int64, device=device)]


def blu_gby_execute_dense_state(plan: Plan, key_cols, val_cols, state_arrays, init: bool = True,
                                n_rows: Optional[int] = None, stream=None):
    n = int(len(key_cols[0]) if n_rows is None else n_rows)
    s = _stream_handle(stream)
    _check(lib.blu_gby_execute_dense_state(plan.handle, _ptrs(key_cols), _ptrs(val_cols), n, s,
                                           _ptrs(state_arrays), int(init)))


def blu_gby_finalize_dense_state(plan: Plan, state_arrays, stream=None) -> Result:
    s = _stream_handle(stream)
    rc = ResultC()
    _check(lib.blu_gby_finalize_dense_state(plan.handle, _ptrs(state_arrays), s, ctypes.byref(rc)))
    return Result(rc, _key_dtypes(plan), _out_dtypes(plan, False), s, _device_of(state_arrays))


def blu_gby_estimate_groups(keys: Sequence[Tuple[int, int]], key_cols, k: int = 2048, n_rows: Optional[int] = None,
                            stream=None) -> Tuple[float, bool]:
    """KMV estimate of the number of distinct key tuples: (estimate, exact)."""
    kd = (KeyDesc * max(1, len(keys)))(*[KeyDesc(int(d), int(s)) for d, s in keys])
    n = int(len(key_cols[0]) if n_rows is None else n_rows)
    est, exact = ctypes.c_double(), ctypes.c_int32()
    _check(lib.blu_gby_estimate_groups(kd, len(keys), _ptrs(key_cols), n, int(k), _stream_handle(stream),
                                       ctypes.byref(est), ctypes.byref(exact)))
    return est.value, bool(exact.value)


def blu_gby_init_table(plan: Plan, dev_table, n_slots: int, stream=None):
    _check(lib.blu_gby_init_table(plan.handle, _ptr(dev_table), int(n_slots), _stream_handle(stream)))


_timing_on = False


def blu_gby_set_timing(enable: bool):
    global _timing_on
    _timing_on = bool(enable)
    lib.blu_gby_set_timing(1 if enable else 0)


def timing_enabled() -> bool:
    """Whether blu_gby_set_timing(True) is in effect in this process (per-phase events in dist.py)."""
    return _timing_on


def blu_gby_last_timing() -> dict:
    t = TimingC()
    _check(lib.blu_gby_last_timing(ctypes.byref(t)))
    d = {k: getattr(t, k) for k, _ in TimingC._fields_}
    d["kernel"] = t.kernel.decode(errors="replace")
    return d


def blu_gby_launch_count() -> int:
    return int(lib.blu_gby_launch_count())


def blu_gby_jit_probe(plan: Plan) -> Tuple[int, int, str]:
    """Compile (no GPU needed) the plan-specialised kernels execute would JIT: (status, programs, log)."""
    buf = ctypes.create_string_buffer(1 << 16)
    n = ctypes.c_int32()
    st = int(lib.blu_gby_jit_probe(plan.handle, buf, len(buf), ctypes.byref(n)))
    return st, n.value, buf.value.decode(errors="replace")


def blu_gby_read_roofline(cols, out, stream=None):
    """Measurement helper: stream every byte of `cols` (device tensors) once with the aggregation
    kernels' load instructions; XOR-fold into `out` (device int64 tensor of 1 element)."""
    n = len(cols)
    by = (ctypes.c_uint64 * n)(*[c.numel() * c.element_size() for c in cols])
    _check(lib.blu_gby_read_roofline(_ptrs(cols), by, n, _stream_handle(stream), ctypes.c_void_p(out.data_ptr())))


def blu_gby_bind_device(device: int):
    _check(lib.blu_gby_bind_device(int(device)))


def blu_gby_release_workspace() -> int:
    """Free the library's idle cached workspace blocks on the current device; returns bytes freed."""
    freed = ctypes.c_uint64()
    _check(lib.blu_gby_release_workspace(ctypes.byref(freed)))
    return int(freed.value)


# ---- sort offload (include/blu_sort.h; §3) ----------------------------------------
# u32 partial keys / payloads / permutations travel as torch.int32 tensors holding the same bits.
def blu_sort_partial_keys(rows, word: int, stream=None):
    """big-endian 4-byte partial keys of word `word` of (n, W) uint8 device rows."""
    import torch
    n, W = rows.shape
    out = torch.empty(n, dtype=torch.int32, device=rows.device)
    _check(lib.blu_sort_partial_keys(_ptr(rows), n, W, word, _ptr(out), _stream_handle(stream)))
    return out


def blu_sort_pairs(keys, payload, stream=None):
    """stable sort of the partial key buffer by its unsigned 4-byte key."""
    import torch
    ko, po = torch.empty_like(keys), torch.empty_like(payload)
    _check(lib.blu_sort_pairs(_ptr(keys), _ptr(payload), keys.numel(), _ptr(ko), _ptr(po), _stream_handle(stream)))
    return ko, po


def blu_sort_dup_ranges(sorted_keys, stream=None):
    """(starts, lens) int64 device tensors of the duplicate ranges of a sorted buffer."""
    import torch
    n = sorted_keys.numel()
    cap = max(1, n // 2)
    st = torch.empty(cap, dtype=torch.int64, device=sorted_keys.device)
    ln = torch.empty(cap, dtype=torch.int64, device=sorted_keys.device)
    r = ctypes.c_uint64()
    _check(lib.blu_sort_dup_ranges(_ptr(sorted_keys), n, _ptr(st), _ptr(ln), cap, ctypes.byref(r), _stream_handle(stream)))
    return st[: r.value], ln[: r.value]


def blu_sort_rows(rows, stream=None):
    """(perm, stats): perm[p] = row at position p of the stable lexicographic order of the
    (n, W) uint8 device rows; stats = levels, ranges / active rows / ms per level."""
    import torch
    n, W = rows.shape
    perm = torch.empty(n, dtype=torch.int32, device=rows.device)
    st = SortStatsC()
    _check(lib.blu_sort_rows(_ptr(rows), n, W, _ptr(perm), _stream_handle(stream), ctypes.byref(st)))
    L = st.levels
    stats = {"levels": L, "ranges": list(st.ranges[:L]), "active": list(st.active[:L]), "ms": list(st.ms[:L]),
             "downsweep_ms": st.downsweep_ms, "downsweep_launches": st.downsweep_launches,
             "downsweep_bytes": st.downsweep_bytes}
    return perm, stats
