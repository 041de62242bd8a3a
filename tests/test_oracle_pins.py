"""Pins for the CPU oracle (oracle/blu_oracle.cpp) against things other than itself.

Each pin is chosen so that a plausible oracle mistake (a dropped term, a wrong index, a transposed
operand, wrong first-value handling for MIN/MAX, missing wrap) fails at least one test:

  * brute force: O(N^2) nested loops in pure Python on tiny inputs (SURVEY.md §8(c) "Brute force");
  * closed form: k(i) = decode(i mod G), v(i) = a*i + b, exact with Python big ints (§8(c));
  * invariants: sum COUNT = N, sum SUM = column sum (wrap / exact dyadic), MIN <= AVG <= MAX,
    row-permutation invariance (north_star "checked ... against invariants");
  * special cases reducing to library routines: one group -> numpy column reductions; all
    distinct -> each group is its row; N = 0 -> no groups;
  * A11 two's-complement wrap of int64 SUM; A12 AVG rounding.

The definition pinned is SQL GROUP BY with COUNT/SUM/MIN/MAX/AVG (PAPER.md P:151, P:153, P:162,
P:176; BASELINE.json north_star). No GPU needed.
"""
import math

import numpy as np
import pytest

import blugen
import oracle
from blugen import AVG, COUNT, F64, I32, I64, MAX, MIN, SUM

pytestmark = pytest.mark.filterwarnings("ignore::RuntimeWarning")


def wrap64(x: int) -> int:
    return ((x + (1 << 63)) % (1 << 64)) - (1 << 63)


def brute_force(schema, key_cols, val_cols):
    """O(N^2): for each first occurrence of a key tuple, scan every row. Pure Python."""
    n = len(key_cols[0]) if key_cols else 0
    K = len(schema.keys)
    rk = [tuple(int(key_cols[k][i]) for k in range(K)) for i in range(n)]
    pyvals = [[(float(v[i]) if d == F64 else int(v[i])) for i in range(n)] for v, d in zip(val_cols, schema.vals)]
    out = []
    for i in range(n):
        g = rk[i]
        first = True
        for j in range(i):
            if rk[j] == g:
                first = False
                break
        if not first:
            continue
        members = [j for j in range(n) if rk[j] == g]
        res = []
        for op, col in schema.aggs:
            if op == COUNT:
                res.append(("i", len(members), None))
                continue
            vs = [pyvals[col][j] for j in members]
            isf = schema.vals[col] == F64
            if op in (SUM, AVG):
                if isf:
                    s = math.fsum(vs)
                    sa = math.fsum(abs(x) for x in vs)
                    res.append(("f", s if op == SUM else s / len(members), sa))
                else:
                    s = wrap64(sum(vs))
                    res.append(("i", s, None) if op == SUM else ("f", float(s) / float(len(members)), None))
            elif op == MIN:
                res.append(("f" if isf else "i", min(vs), None))
            else:
                res.append(("f" if isf else "i", max(vs), None))
        out.append((g, len(members), res))
    out.sort(key=lambda t: t[0])
    return out


def assert_matches_brute(schema, kc, vc, exact_f64=True):
    o = oracle.groupby_arrays(schema, kc, vc)
    b = brute_force(schema, kc, vc)
    assert o.n_groups == len(b)
    for gi, (key, cnt, res) in enumerate(b):
        assert tuple(int(x) for x in o.keys[gi]) == key
        assert int(o.count[gi]) == cnt
        for a, (kind, val, sa) in enumerate(res):
            got = o.aggs[a][gi]
            if sa is not None:
                # the oracle's sum|v| sets the A13 tolerance of every f64 SUM/AVG parity check: pin it
                # to the correctly rounded math.fsum of |v| (long double accumulation: <= n * 2^-64 rel.)
                osa = float(o.sumabs[a][gi])
                assert abs(osa - sa) <= 4e-16 * sa * max(1, cnt) + 0.0, (gi, a, osa, sa)
                if exact_f64:
                    assert osa == sa, (gi, a, osa, sa)
            else:
                assert o.sumabs[a] is None or schema.aggs[a][0] not in (SUM, AVG), (gi, a)
            if kind == "i":
                assert int(got) == val, (gi, a, got, val)
            elif exact_f64 or sa is None:
                assert float(got) == val, (gi, a, got, val)
            else:
                assert abs(float(got) - val) <= 1e-12 * max(sa, 1e-300) + 0.0, (gi, a, got, val, sa)


def _rand_cols(rng, n, key_spec, val_dtypes, dyadic=True):
    kc = []
    for d, dict_size in key_spec:
        hi = dict_size if dict_size else 7
        arr = rng.integers(0, hi, n)
        if not dict_size:  # sparse codes: large, spread values with collisions
            arr = arr * 1_000_000_007 + 3
        kc.append(arr.astype(blugen.NP_DTYPE[d]))
    vc = []
    for d in val_dtypes:
        if d == I32:
            v = rng.integers(-(2**31), 2**31, n).astype(np.int32)
        elif d == I64:
            v = rng.integers(-(2**62), 2**62, n).astype(np.int64)
        else:
            if dyadic:
                v = (rng.integers(-(2**20), 2**20, n) / 64.0).astype(np.float64)
            else:
                v = (rng.random(n) - 0.5) * 1e6
        vc.append(v)
    return kc, vc


ALL_AGGS = lambda nv, vdt: [(COUNT, -1)] + [(op, c) for c in range(nv) for op in (SUM, MIN, MAX, AVG)]


@pytest.mark.parametrize("case", range(8))
def test_brute_force_small(case):
    rng = np.random.default_rng(1000 + case)
    K = 1 + case % 3
    key_spec = [([I32, I64][(case + j) % 2], [3, 5, 2, 0][(case + j) % 4]) for j in range(K)]
    vdt = [I32, I64, F64]
    n = [1, 2, 31, 33, 200, 500, 700, 300][case]
    kc, vc = _rand_cols(rng, n, key_spec, vdt)
    sch = blugen.Schema(key_spec, vdt, ALL_AGGS(3, vdt))
    assert_matches_brute(sch, kc, vc)


def test_brute_force_n2000():
    rng = np.random.default_rng(7)
    key_spec = [(I32, 9), (I64, 4)]
    vdt = [I64, F64, I32]
    kc, vc = _rand_cols(rng, 2000, key_spec, vdt)
    sch = blugen.Schema(key_spec, vdt, ALL_AGGS(3, vdt))
    assert_matches_brute(sch, kc, vc)


def test_brute_force_general_f64_tolerance():
    """Non-dyadic doubles: the oracle's long-double sum is within 1e-12 * sum|v| of fsum (A13)."""
    rng = np.random.default_rng(11)
    key_spec = [(I32, 6)]
    vdt = [F64]
    kc, vc = _rand_cols(rng, 1500, key_spec, vdt, dyadic=False)
    sch = blugen.Schema(key_spec, vdt, [(COUNT, -1), (SUM, 0), (AVG, 0), (MIN, 0), (MAX, 0)])
    assert_matches_brute(sch, kc, vc, exact_f64=False)


def test_int64_sum_wraps_twos_complement():
    """A11: int64 SUM wraps like the GPU's 64-bit adds; pinned by explicit big-int arithmetic."""
    sch = blugen.Schema([(I32, 2)], [I64], [(SUM, 0), (MIN, 0), (MAX, 0), (AVG, 0)])
    k = np.array([0, 0, 0, 1, 1], np.int32)
    v = np.array([2**62, 2**62, 2**62, -(2**63), -1], np.int64)
    o = oracle.groupby_arrays(sch, [k], [v])
    assert int(o.aggs[0][0]) == wrap64(3 * 2**62) == -(2**62)
    assert int(o.aggs[0][1]) == wrap64(-(2**63) - 1) == 2**63 - 1
    assert int(o.aggs[1][1]) == -(2**63) and int(o.aggs[2][1]) == -1
    assert float(o.aggs[3][0]) == float(-(2**62)) / 3.0


def test_minmax_first_value_not_sentinel():
    """MIN/MAX start from the first row (no sentinel can leak): all-negative MAX, all-positive MIN."""
    sch = blugen.Schema([(I64, 0)], [I32, F64], [(MAX, 0), (MIN, 0), (MAX, 1), (MIN, 1)])
    k = np.array([5, 5, 9], np.int64)
    v0 = np.array([-7, -3, 2**31 - 1], np.int32)
    v1 = np.array([-2.5, -0.5, 1e300], np.float64)
    o = oracle.groupby_arrays(sch, [k], [v0, v1])
    assert list(o.keys[:, 0]) == [5, 9]
    assert list(o.aggs[0]) == [-3, 2**31 - 1] and list(o.aggs[1]) == [-7, 2**31 - 1]
    assert list(o.aggs[2]) == [-0.5, 1e300] and list(o.aggs[3]) == [-2.5, 1e300]


@pytest.mark.parametrize("a,b,vd,G,N", [(3, -1000, I32, 1024, 100_003), (-7919, 123456789, I64, 16, 1_000_000),
                                       (5, 7, I64, 100_000, 250_001), (1, 0, I32, 1, 1000),
                                       (1, -5, I64, 1, 2_000_001)])
def test_closed_form(a, b, vd, G, N):
    """k(i) = decode(i mod G) (mixed radix), v(i) = a*i + b. With c_g = ceil((N-g)/G):
    COUNT_g = c_g; SUM_g = a(g c_g + G c_g (c_g-1)/2) + b c_g; MIN/MAX = a g + b and
    a(g + G(c_g-1)) + b (swapped if a < 0); AVG = SUM/COUNT."""
    # radices whose product is G (G = 1024 -> 32 x 32; 100000 -> 100 x 50 x 20; 16 -> 16; 1 -> 1)
    radix = {1024: [32, 32], 16: [16], 100_000: [100, 50, 20], 1: [1]}[G]
    strides = [int(np.prod(radix[:j])) for j in range(len(radix))]
    w = blugen.Workload(
        "closed", N, 0xC105ED,
        [blugen.Col(I32, blugen.CYCLIC_DIGIT, 0, n_groups=G, stride=s, radix=r) for s, r in zip(strides, radix)],
        [blugen.Col(vd, blugen.LINEAR, 1, lo=a, hi=b)],
        blugen.Schema([(I32, r) for r in radix], [vd], [(COUNT, -1), (SUM, 0), (MIN, 0), (MAX, 0), (AVG, 0)]),
        G, G)
    o = oracle.groupby_generated(w)
    assert o.n_groups == min(G, N)
    for gi in range(o.n_groups):
        g = sum(int(o.keys[gi][j]) * strides[j] for j in range(len(radix)))
        c = -(-(N - g) // G)
        s = a * (g * c + G * c * (c - 1) // 2) + b * c
        lo, hi = a * g + b, a * (g + G * (c - 1)) + b
        if a < 0:
            lo, hi = hi, lo
        assert int(o.count[gi]) == c
        assert int(o.aggs[0][gi]) == c
        assert int(o.aggs[1][gi]) == wrap64(s)
        assert int(o.aggs[2][gi]) == lo and int(o.aggs[3][gi]) == hi
        assert float(o.aggs[4][gi]) == float(s) / float(c)


def _invariants(sch, kc, vc, o):
    n = len(kc[0])
    assert int(o.count.sum()) == n
    for a, (op, col) in enumerate(sch.aggs):
        if op == SUM:
            if sch.vals[col] == F64:
                assert float(math.fsum(o.aggs[a])) == math.fsum(vc[col].tolist())  # dyadic: exact
            else:
                assert wrap64(sum(int(x) for x in o.aggs[a])) == wrap64(sum(int(x) for x in vc[col]))
    mins = {col: o.aggs[a] for a, (op, col) in enumerate(sch.aggs) if op == MIN}
    maxs = {col: o.aggs[a] for a, (op, col) in enumerate(sch.aggs) if op == MAX}
    for a, (op, col) in enumerate(sch.aggs):
        if op == AVG and col in mins and col in maxs:
            assert np.all(mins[col].astype(np.float64) <= o.aggs[a]) and np.all(o.aggs[a] <= maxs[col].astype(np.float64))


def test_invariants_and_permutation():
    rng = np.random.default_rng(3)
    key_spec = [(I32, 40), (I32, 25)]
    vdt = [I32, I64, F64]
    n = 60_000
    kc, vc = _rand_cols(rng, n, key_spec, vdt)
    vc[1] = rng.integers(-(10**12), 10**12, n)
    sch = blugen.Schema(key_spec, vdt, ALL_AGGS(3, vdt))
    o = oracle.groupby_arrays(sch, kc, vc)
    _invariants(sch, kc, vc, o)
    perm = rng.permutation(n)
    o2 = oracle.groupby_arrays(sch, [k[perm] for k in kc], [v[perm] for v in vc])
    assert np.array_equal(o.keys, o2.keys) and np.array_equal(o.count, o2.count)
    for x, y in zip(o.aggs, o2.aggs):
        assert np.array_equal(x, y)


def test_one_group_reduces_to_column_reductions():
    rng = np.random.default_rng(5)
    n = 10_000
    k = np.full(n, 3, np.int32)
    v0 = rng.integers(-(2**31), 2**31, n).astype(np.int32)
    v1 = rng.integers(-(2**40), 2**40, n).astype(np.int64)
    v2 = (rng.integers(-(2**20), 2**20, n) / 64.0)
    sch = blugen.Schema([(I32, 8)], [I32, I64, F64], ALL_AGGS(3, None))
    o = oracle.groupby_arrays(sch, [k], [v0, v1, v2])
    assert o.n_groups == 1 and int(o.keys[0, 0]) == 3 and int(o.count[0]) == n
    exp = []
    for v in (v0, v1, v2):
        s = float(np.sum(v)) if v.dtype == np.float64 else int(np.sum(v.astype(np.int64)))
        exp += [s, v.min(), v.max(), s / n if v.dtype == np.float64 else float(s) / n]
    got = [x[0] for x in o.aggs[1:]]
    for g, e in zip(got, exp):
        assert g == e


def test_all_distinct_each_group_is_its_row():
    rng = np.random.default_rng(6)
    n = 5000
    k = rng.permutation(10**6)[:n].astype(np.int64)
    v = rng.integers(-(2**62), 2**62, n)
    f = (rng.random(n) - 0.5) * 1e9
    sch = blugen.Schema([(I64, 0)], [I64, F64], ALL_AGGS(2, None))
    o = oracle.groupby_arrays(sch, [k], [v, f])
    order = np.argsort(k)
    assert np.array_equal(o.keys[:, 0], k[order]) and np.all(o.count == 1)
    for a, (op, col) in enumerate(sch.aggs[1:], start=1):
        src = [v, f][col][order]
        if op == AVG:
            assert np.array_equal(o.aggs[a], src.astype(np.float64))
        else:
            assert np.array_equal(o.aggs[a], src)


def test_empty_input():
    sch = blugen.Schema([(I32, 4)], [I64], [(COUNT, -1), (SUM, 0)])
    o = oracle.groupby_arrays(sch, [np.zeros(0, np.int32)], [np.zeros(0, np.int64)])
    assert o.n_groups == 0


def test_slices_partition_the_result():
    w = blugen.workload("C4", n_rows=200_000)
    full = oracle.groupby_generated(w)
    parts = [oracle.groupby_generated(w, slice_p=p, slice_P=5) for p in range(5)]
    for p, r in enumerate(parts):  # slice rule (k0 + 31 k1 + 961 k2) mod P == p
        k = r.keys.astype(np.int64)
        assert np.all((k[:, 0] + 31 * k[:, 1] + 961 * k[:, 2]) % 5 == p)
    u = oracle.concat(parts)
    assert np.array_equal(u.keys, full.keys) and np.array_equal(u.count, full.count)
    for x, y in zip(u.aggs, full.aggs):
        assert np.array_equal(x, y)


def test_filter_is_subset_and_generated_equals_arrays():
    w = blugen.workload("C2", n_rows=100_000)
    kc, vc = blugen.host_columns(w)
    full_a = oracle.groupby_arrays(w.schema, kc, vc)
    full_g = oracle.groupby_generated(w)
    assert np.array_equal(full_a.keys, full_g.keys)
    for x, y in zip(full_a.aggs, full_g.aggs):
        assert np.array_equal(x, y)
    pick = full_a.keys[::97]
    sub = oracle.groupby_generated(w, filter_keys=pick)
    idx = np.arange(0, full_a.n_groups, 97)
    assert np.array_equal(sub.keys, pick)
    for x, y in zip(sub.aggs, full_a.aggs):
        assert np.array_equal(x, y[idx])


# ---- 128-bit payloads (NEXT-2, reading A18) ------------------------------------------------------
def i128_cols(ints):
    """Python ints -> (n, 2) int64 (low word, high word), two's complement mod 2^128."""
    out = np.zeros((len(ints), 2), np.int64)
    for i, x in enumerate(ints):
        u = x % (1 << 128)
        out[i, 0] = np.int64(np.uint64(u & ((1 << 64) - 1)).view(np.int64))
        out[i, 1] = np.int64(np.uint64(u >> 64).view(np.int64))
    return out


def i128_value(row):
    u = (int(np.uint64(row[1]).view(np.uint64)) << 64) | int(np.int64(row[0]).view(np.uint64))
    return u - (1 << 128) if u >> 127 else u


def test_i128_brute_force():
    """SUM (mod 2^128), MIN, MAX, AVG, COUNT over 128-bit payloads vs Python integers."""
    rng = np.random.default_rng(128)
    n = 3000
    keys = rng.integers(0, 9, n)
    vals = [int(x) for x in rng.integers(-(2**62), 2**62, n)]
    vals = [v * (1 << 64) + int(rng.integers(0, 2**62)) if i % 3 else v for i, v in enumerate(vals)]  # full range
    sch = blugen.Schema([(I64, 9)], [blugen.I128], [(COUNT, -1), (SUM, 0), (MIN, 0), (MAX, 0), (AVG, 0)])
    o = oracle.groupby_arrays(sch, [keys.astype(np.int64)], [i128_cols(vals)])
    assert list(o.keys[:, 0]) == sorted(set(keys.tolist()))
    for gi, k in enumerate(o.keys[:, 0]):
        g = [v for kk, v in zip(keys, vals) if kk == k]
        s = sum(g) % (1 << 128)
        s = s - (1 << 128) if s >> 127 else s
        assert o.aggs[0][gi] == len(g)
        assert i128_value(o.aggs[1][gi]) == s
        assert i128_value(o.aggs[2][gi]) == min(g)
        assert i128_value(o.aggs[3][gi]) == max(g)
        assert o.aggs[4][gi] == float(s) / len(g)  # (double)sum correctly rounded, then IEEE division


def test_i128_sum_wraps_mod_2_128():
    """Closed form: 4 rows of 2^126 sum to 2^128 = 0; 5 rows of 2^126 to 2^126 (mod 2^128)."""
    sch = blugen.Schema([(I64, 2)], [blugen.I128], [(SUM, 0)])
    keys = np.array([0, 0, 0, 0, 1, 1, 1, 1, 1], np.int64)
    o = oracle.groupby_arrays(sch, [keys], [i128_cols([1 << 126] * 9)])
    assert i128_value(o.aggs[0][0]) == 0 and i128_value(o.aggs[0][1]) == 1 << 126


def test_i128_in_int64_range_equals_i64_column():
    """Special case: 128-bit payloads that fit 64 bits give the i64 results (sums far from wrapping)."""
    rng = np.random.default_rng(7)
    n = 5000
    keys = rng.integers(0, 13, n).astype(np.int64)
    v = rng.integers(-(2**40), 2**40, n)
    s64 = blugen.Schema([(I64, 13)], [I64], [(SUM, 0), (MIN, 0), (MAX, 0), (AVG, 0)])
    s128 = blugen.Schema([(I64, 13)], [blugen.I128], [(SUM, 0), (MIN, 0), (MAX, 0), (AVG, 0)])
    a = oracle.groupby_arrays(s64, [keys], [v])
    b = oracle.groupby_arrays(s128, [keys], [i128_cols([int(x) for x in v])])
    for j in range(3):
        assert np.array_equal(b.aggs[j][:, 0], a.aggs[j]) and np.array_equal(b.aggs[j][:, 1], a.aggs[j] >> 63)
    assert np.array_equal(b.aggs[3], a.aggs[3])


# ---- sort offload oracle (§3; oracle/sort_oracle.cpp) -----------------------------
def _rows(rng, n, W, alphabet=4):
    """Small-alphabet byte rows: many shared prefixes, so duplicate ranges occur at every word."""
    return rng.integers(0, alphabet, (n, W), dtype=np.uint8)


def test_partial_key_is_big_endian_and_order_isomorphic():
    """P:78 "partial binary sortable representation": the u32 of bytes [4w, 4w+4) read most
    significant first; comparing two partial keys = comparing those 4 bytes lexicographically."""
    rng = np.random.default_rng(11)
    rows = rng.integers(0, 256, (300, 12), dtype=np.uint8)
    for w in range(3):
        k = oracle.partial_keys(rows, w)
        for i in range(300):
            assert int(k[i]) == int.from_bytes(bytes(rows[i, 4 * w:4 * w + 4]), "big")
        for i in range(0, 299):
            a, b = bytes(rows[i, 4 * w:4 * w + 4]), bytes(rows[i + 1, 4 * w:4 * w + 4])
            assert (k[i] < k[i + 1]) == (a < b) and (k[i] == k[i + 1]) == (a == b)


@pytest.mark.parametrize("n,card", [(0, 3), (1, 3), (500, 3), (2000, 50), (2000, 2**32)])
def test_sort_pairs_is_stable_sort_by_key(n, card):
    """The sorted partial key buffer equals Python's (stable) sorted() by key, and numpy's
    stable argsort; payload order within equal keys is buffer order."""
    rng = np.random.default_rng(n + 5)
    keys = rng.integers(0, card, n, dtype=np.uint64).astype(np.uint32)
    pay = rng.permutation(n).astype(np.uint32)
    ko, po = oracle.sort_pairs(keys, pay)
    order = sorted(range(n), key=lambda i: int(keys[i]))
    assert [int(x) for x in po] == [int(pay[i]) for i in order]
    assert np.array_equal(ko, keys[order] if n else keys)
    assert np.array_equal(po, pay[np.argsort(keys, kind="stable")])


def test_dup_ranges_brute_force():
    """Duplicate ranges = maximal runs of >= 2 equal keys, by itertools.groupby."""
    import itertools
    rng = np.random.default_rng(3)
    for n, card in [(0, 2), (1, 2), (7, 1), (400, 5), (400, 1000)]:
        keys = np.sort(rng.integers(0, card, n)).astype(np.uint32)
        st, ln = oracle.dup_ranges(keys)
        exp, pos = [], 0
        for _, g in itertools.groupby(keys.tolist()):
            c = len(list(g))
            if c >= 2:
                exp.append((pos, c))
            pos += c
        assert list(zip(st.tolist(), ln.tolist())) == exp
        assert int(ln.sum()) == sum(c for _, c in exp)


@pytest.mark.parametrize("W", [4, 8, 12, 16])
def test_sort_rows_brute_force(W):
    """The completed sort = Python's stable sorted() of row indices by the key bytes."""
    rng = np.random.default_rng(W)
    for n in (0, 1, 2, 37, 700):
        rows = _rows(rng, n, W)
        perm = oracle.sort_rows(rows)
        exp = sorted(range(n), key=lambda i: bytes(rows[i]))
        assert [int(x) for x in perm] == exp


def test_sort_rows_special_cases_and_invariants():
    rng = np.random.default_rng(9)
    n, W = 1000, 8
    same = np.tile(rng.integers(0, 256, (1, W), dtype=np.uint8), (n, 1))
    assert np.array_equal(oracle.sort_rows(same), np.arange(n))           # all equal: row order
    distinct = np.stack([np.frombuffer(int(x).to_bytes(W, "big"), np.uint8) for x in range(n)])
    assert np.array_equal(oracle.sort_rows(distinct), np.arange(n))       # already sorted
    assert np.array_equal(oracle.sort_rows(distinct[::-1].copy()), np.arange(n)[::-1])  # reversed
    rows = _rows(rng, 5000, 12)
    perm = oracle.sort_rows(rows)
    assert np.array_equal(np.sort(perm), np.arange(5000))                 # a permutation
    s = rows[perm]
    for i in range(4999):                                                  # non-decreasing, stable
        a, b = bytes(s[i]), bytes(s[i + 1])
        assert a < b or (a == b and perm[i] < perm[i + 1])
    # the job queue of P:84-86 written out step by step reaches the same order: sort by word 0,
    # then every duplicate range by the next word, until no range is left
    order = np.arange(5000)
    ranges = [(0, 5000)]
    for w in range(3):
        nxt = []
        for a, b in ranges:
            seg = order[a:b]
            k = oracle.partial_keys(rows[seg], w)
            _, po = oracle.sort_pairs(k, np.arange(b - a, dtype=np.uint32))
            order[a:b] = seg[po.astype(np.int64)]
            ks = k[po.astype(np.int64)]
            st, ln = oracle.dup_ranges(ks)
            nxt += [(a + int(x), a + int(x) + int(y)) for x, y in zip(st, ln)]
        ranges = nxt
    assert np.array_equal(order, perm)


# ---- KMV group-count estimate (oracle/kmv_oracle.cpp; NEXT-3) --------------------------
def test_kmv_exact_below_k_equals_distinct_tuples():
    """Fewer than k distinct tuples: the estimate is exact and equals a Python set's size (fmix64 is a
    bijection and the mixed-radix concatenation is injective on in-dictionary codes)."""
    rng = np.random.default_rng(77)
    for dicts, n in (((7, 5, 3), 5000), ((16,), 100), ((1,), 50), ((300,), 4000)):
        cols = [rng.integers(0, d, n).astype(np.int32) for d in dicts]
        est, exact = oracle.kmv(cols, dicts, k=512)
        assert exact and est == len(set(zip(*[c.tolist() for c in cols])))
    sparse = rng.integers(0, 2**62, 200).astype(np.int64)[rng.integers(0, 200, 3000)]
    est, exact = oracle.kmv([sparse], [0], k=1024)
    assert exact and est == len(set(sparse.tolist()))
    est, exact = oracle.kmv([np.zeros(0, np.int64)], [0], k=16)
    assert exact and est == 0


def test_kmv_kth_value_matches_python_sort():
    """U_(k) is the k-th smallest DISTINCT hash (Python sorted() of a set, not std::set) and
    est = (k - 1) * 2^64 / U_(k) (the estimator of the paper's KMV reference [2])."""
    rng = np.random.default_rng(5)
    keys = rng.integers(0, 2**62, 300).astype(np.int64)
    rows = keys[rng.integers(0, 300, 2000)]
    salt = 0x6B6D765F73616C74  # "kmv_salt"
    hs = sorted({oracle.fmix64(int(x) ^ salt) for x in rows.tolist()} - {2**64 - 1})
    for k in (16, 64, 255):
        est, exact = oracle.kmv([rows], [0], k=k)
        assert not exact and est == (k - 1) * 18446744073709551616.0 / float(hs[k - 1])


def test_kmv_relative_error_bound_over_seeds():
    """KMV is unbiased with relative standard error ~ 1/sqrt(k - 2): over 30 independent key sets of
    G = 20000 groups every estimate is within 5 sd and the mean within 4 sd / sqrt(30)."""
    G, k = 20000, 256
    sd = 1.0 / math.sqrt(k - 2)
    ratios = []
    for seed in range(30):
        rng = np.random.default_rng(9000 + seed)
        keys = np.unique(rng.integers(0, 2**62, G + 64).astype(np.int64))[:G]
        rows = keys[rng.integers(0, G, 3 * G)]
        rows = np.concatenate([keys, rows])  # every key present
        est, exact = oracle.kmv([rows], [0], k=k)
        assert not exact
        ratios.append(est / G)
        assert abs(est / G - 1) <= 5 * sd, (seed, est)
    assert abs(float(np.mean(ratios)) - 1) <= 4 * sd / math.sqrt(30), np.mean(ratios)


def test_kmv_invariant_to_row_order_and_duplicates():
    rng = np.random.default_rng(11)
    cols = [rng.integers(0, 100, 50000).astype(np.int32), rng.integers(0, 50, 50000).astype(np.int32)]
    est, _ = oracle.kmv(cols, [100, 50], k=128)
    perm = rng.permutation(50000)
    est_p, _ = oracle.kmv([c[perm] for c in cols], [100, 50], k=128)
    est_d, _ = oracle.kmv([np.concatenate([c, c[:777]]) for c in cols], [100, 50], k=128)
    assert est == est_p == est_d


def test_kmv_hash_is_a_bijective_avalanching_mix():
    """fmix64 (Murmur3 finalizer): 0 -> 0, no collisions on 2^16 consecutive inputs, and one flipped
    input bit flips ~half of the output bits (a dropped xorshift or multiply fails one of these)."""
    assert oracle.fmix64(0) == 0
    outs = {oracle.fmix64(i) for i in range(1 << 16)}
    assert len(outs) == 1 << 16
    rng = np.random.default_rng(3)
    flips = []
    for _ in range(2000):
        x = int(rng.integers(0, 2**63))
        b = int(rng.integers(0, 64))
        flips.append(bin(oracle.fmix64(x) ^ oracle.fmix64(x ^ (1 << b))).count("1"))
    assert 31.0 <= float(np.mean(flips)) <= 33.0
