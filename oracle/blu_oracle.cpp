/*
 * ORACLE — TEST INFRASTRUCTURE ONLY. Not part of libblugby; the product path never loads it.
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference leg may
 * load or call this library.
 *
 * A plain, slow, single-threaded C++ std::map GROUP BY (BASELINE.json
 * north_star "a plain, slow single-threaded C++ std::map GROUP BY that shares no code with the
 * GPU path"). It shares NO code with paper_conf_sigmod_merajispcksygnk16_b200/csrc: its only
 * include from the repo is include/blu_gen.h, the seeded input generator, which holds none of
 * the method's arithmetic.
 *
 * What it computes is the plain definition of SQL GROUP BY with the paper's aggregates:
 *   - one output row per distinct key tuple ("Each entry in the input table has
 *     one grouping key"; "CCAT: Concatenate keys for queries that group by on more than
 *     one column");
 *   - aggregates applied "right after the insertion/finding of grouping key",
 *     Min, Max, Sum, Count and AVG (north_star);
 *   - COUNT_g = |{i : k(i) = g}|, SUM_g = sum of v over g, MIN/MAX over g, AVG = SUM / COUNT.
 * No packing, no hashing, no sentinels, no blocking: keys are the widened tuple itself.
 *
 * Readings of silent/ambiguous points:
 *   A11 integer SUM is int64 with two's-complement wrap (accumulated in uint64_t);
 *   A12 AVG is f64: (double)(int64)sum / (double)count, IEEE round-to-nearest;
 *   A13 f64 SUM accumulates in long double (x86 80-bit) plus sum |v| for the tolerance check;
 *   A14 MIN/MAX use < and > (inputs hold no NaN, no -0.0);
 *   A15 all columns NOT NULL, COUNT means COUNT(*);
 *   A18 128-bit integer payloads ("128bit Integer or Decimal data type", NEXT-2): SUM wraps
 *       mod 2^128 (accumulated in unsigned __int128), MIN/MAX compare as signed __int128, AVG is
 *       (double)(__int128)sum / (double)count (GCC's correctly rounded __int128 -> double).
 *
 * Parity pins for this file live in tests/test_oracle_pins.py (brute force, closed forms,
 * invariants, special cases).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#include <map>
#include <set>
#include <vector>

#include "blu_gen.h"

namespace {

enum { O_I32 = 0, O_I64 = 1, O_F64 = 2, O_I128 = 3 };
enum { O_COUNT = 0, O_SUM = 1, O_MIN = 2, O_MAX = 3, O_AVG = 4 };

struct Schema {
    int n_keys;
    std::vector<int> key_dtypes;
    int n_vals;
    std::vector<int> val_dtypes;
    int n_aggs;
    std::vector<int> agg_ops;
    std::vector<int> agg_cols;
};

struct AggState {
    uint64_t isum = 0;        // integer SUM / AVG numerator, wraps like int64
    long double fsum = 0.0L;  // f64 SUM / AVG numerator
    long double fabs_sum = 0.0L;
    int64_t imm = 0;          // integer MIN or MAX
    double fmm = 0.0;         // f64 MIN or MAX
    unsigned __int128 qsum = 0;  // 128-bit SUM / AVG numerator, wraps mod 2^128
    __int128 qmm = 0;            // 128-bit MIN or MAX
};

struct Group {
    int64_t count = 0;
    std::vector<AggState> a;
};

struct Result {
    Schema s;
    std::map<std::vector<int64_t>, Group> groups;
};

// One input value, widened: integers to int64, doubles kept as double.
struct Val {
    int64_t i;
    double d;
    __int128 q;  // 128-bit payloads only
};

Val widen(int dtype, uint64_t bits) {
    Val v{0, 0.0, 0};
    if (dtype == O_I32) v.i = (int64_t)(int32_t)(uint32_t)bits;
    else if (dtype == O_I64) v.i = (int64_t)bits;
    else memcpy(&v.d, &bits, sizeof(double));
    return v;
}

uint64_t read_bits(int dtype, const void* col, uint64_t i) {
    if (dtype == O_I32) return (uint64_t)(uint32_t)((const int32_t*)col)[i];
    return ((const uint64_t*)col)[i];
}

// A 128-bit payload: 16 bytes per row, low 64-bit word first (two's complement).
Val read_i128(const void* col, uint64_t i) {
    const uint64_t lo = ((const uint64_t*)col)[2 * i], hi = ((const uint64_t*)col)[2 * i + 1];
    Val v{0, 0.0, 0};
    v.q = (__int128)(((unsigned __int128)hi << 64) | lo);
    return v;
}

// The per-row step: find or insert the group, then apply every aggregate.
void add_row(Result& r, const std::vector<int64_t>& key, const std::vector<Val>& vals) {
    const Schema& s = r.s;
    auto it = r.groups.find(key);
    bool first = false;
    if (it == r.groups.end()) {
        Group g;
        g.a.resize(s.n_aggs);
        it = r.groups.emplace(key, g).first;
        first = true;
    }
    Group& g = it->second;
    g.count += 1;
    for (int a = 0; a < s.n_aggs; ++a) {
        int op = s.agg_ops[a];
        if (op == O_COUNT) continue;
        int c = s.agg_cols[a];
        int dt = s.val_dtypes[c];
        const Val& v = vals[c];
        AggState& st = g.a[a];
        if (dt == O_I128) {
            if (op == O_SUM || op == O_AVG) st.qsum += (unsigned __int128)v.q;
            else if (op == O_MIN) { if (first || v.q < st.qmm) st.qmm = v.q; }
            else if (op == O_MAX) { if (first || v.q > st.qmm) st.qmm = v.q; }
            continue;
        }
        if (op == O_SUM || op == O_AVG) {
            if (dt == O_F64) {
                st.fsum += (long double)v.d;
                st.fabs_sum += (long double)(v.d < 0 ? -v.d : v.d);
            } else {
                st.isum += (uint64_t)v.i;
            }
        } else if (op == O_MIN) {
            if (dt == O_F64) { if (first || v.d < st.fmm) st.fmm = v.d; }
            else { if (first || v.i < st.imm) st.imm = v.i; }
        } else if (op == O_MAX) {
            if (dt == O_F64) { if (first || v.d > st.fmm) st.fmm = v.d; }
            else { if (first || v.i > st.imm) st.imm = v.i; }
        }
    }
}

// Key-sliced mode: (k0 + 31 k1 + 961 k2) mod P, unsigned 64-bit.
bool in_slice(const std::vector<int64_t>& key, uint32_t p, uint32_t P) {
    if (P <= 1) return true;
    uint64_t k0 = (uint64_t)key[0];
    uint64_t k1 = key.size() > 1 ? (uint64_t)key[1] : 0;
    uint64_t k2 = key.size() > 2 ? (uint64_t)key[2] : 0;
    return (k0 + 31ull * k1 + 961ull * k2) % P == p;
}

Schema make_schema(int n_keys, const int32_t* kd, int n_vals, const int32_t* vd, int n_aggs,
                   const int32_t* ops, const int32_t* cols) {
    Schema s;
    s.n_keys = n_keys;
    s.key_dtypes.assign(kd, kd + n_keys);
    s.n_vals = n_vals;
    s.val_dtypes.assign(vd, vd + n_vals);
    s.n_aggs = n_aggs;
    s.agg_ops.assign(ops, ops + n_aggs);
    s.agg_cols.assign(cols, cols + n_aggs);
    return s;
}

std::set<std::vector<int64_t>> make_filter(int n_keys, const int64_t* fk, uint64_t nf) {
    std::set<std::vector<int64_t>> f;
    for (uint64_t g = 0; g < nf; ++g) f.insert(std::vector<int64_t>(fk + g * n_keys, fk + (g + 1) * n_keys));
    return f;
}

}  // namespace

extern "C" {

/* Plain schema struct of the oracle's own (same enum numbering as blu_gby.h by convention). */
typedef struct {
    int32_t n_keys;
    const int32_t* key_dtypes;
    int32_t n_vals;
    const int32_t* val_dtypes;
    int32_t n_aggs;
    const int32_t* agg_ops;
    const int32_t* agg_cols;
} oracle_schema_t;

/* GROUP BY over host column arrays. slice_P <= 1 disables slicing; filter_keys (n_filter x
 * n_keys, row-major, widened to int64) restricts the rows to those key tuples if non-NULL.
 * Returns an opaque handle (free with oracle_free). */
void* oracle_groupby_arrays(const oracle_schema_t* sc, const void* const* keys, const void* const* vals,
                            uint64_t n, uint32_t slice_p, uint32_t slice_P, const int64_t* filter_keys,
                            uint64_t n_filter) {
    Result* r = new Result;
    r->s = make_schema(sc->n_keys, sc->key_dtypes, sc->n_vals, sc->val_dtypes, sc->n_aggs, sc->agg_ops,
                       sc->agg_cols);
    std::set<std::vector<int64_t>> filter;
    if (filter_keys) filter = make_filter(sc->n_keys, filter_keys, n_filter);
    std::vector<int64_t> key(sc->n_keys);
    std::vector<Val> v(sc->n_vals);
    for (uint64_t i = 0; i < n; ++i) {
        for (int k = 0; k < sc->n_keys; ++k) key[k] = widen(sc->key_dtypes[k], read_bits(sc->key_dtypes[k], keys[k], i)).i;
        if (!in_slice(key, slice_p, slice_P)) continue;
        if (filter_keys && !filter.count(key)) continue;
        for (int c = 0; c < sc->n_vals; ++c)
            v[c] = sc->val_dtypes[c] == O_I128 ? read_i128(vals[c], i)
                                               : widen(sc->val_dtypes[c], read_bits(sc->val_dtypes[c], vals[c], i));
        add_row(*r, key, v);
    }
    return r;
}

/* GROUP BY over rows row0..row0+n-1 generated on the fly from include/blu_gen.h specs
 * (host pointers for zipf tables). Same slicing / filtering as above. */
void* oracle_groupby_generated(const oracle_schema_t* sc, const blu_gen_spec_t* key_specs,
                               const blu_gen_spec_t* val_specs, uint64_t row0, uint64_t n, uint32_t slice_p,
                               uint32_t slice_P, const int64_t* filter_keys, uint64_t n_filter) {
    Result* r = new Result;
    r->s = make_schema(sc->n_keys, sc->key_dtypes, sc->n_vals, sc->val_dtypes, sc->n_aggs, sc->agg_ops,
                       sc->agg_cols);
    std::set<std::vector<int64_t>> filter;
    if (filter_keys) filter = make_filter(sc->n_keys, filter_keys, n_filter);
    std::vector<int64_t> key(sc->n_keys);
    std::vector<Val> v(sc->n_vals);
    for (uint64_t i = row0; i < row0 + n; ++i) {
        for (int k = 0; k < sc->n_keys; ++k) {
            uint64_t b = blu_gen_bits(&key_specs[k], i);
            if (sc->key_dtypes[k] == O_I32) b = (uint64_t)(uint32_t)b;
            key[k] = widen(sc->key_dtypes[k], b).i;
        }
        if (!in_slice(key, slice_p, slice_P)) continue;
        if (filter_keys && !filter.count(key)) continue;
        for (int c = 0; c < sc->n_vals; ++c) {
            uint64_t b = blu_gen_bits(&val_specs[c], i);
            if (sc->val_dtypes[c] == O_I32) b = (uint64_t)(uint32_t)b;
            v[c] = widen(sc->val_dtypes[c], b);
        }
        add_row(*r, key, v);
    }
    return r;
}

uint64_t oracle_n_groups(void* h) { return ((Result*)h)->groups.size(); }

/* Emit in map order (lexicographic on the key tuple).
 *   keys_out:   n_groups x n_keys int64 (row-major)
 *   count_out:  n_groups int64
 *   agg_out[a]: n_groups elements: COUNT -> int64; SUM(int) -> int64; SUM(f64) -> double;
 *               MIN/MAX -> int64 (integer inputs, widened) or double; AVG -> double;
 *               SUM/MIN/MAX of a 128-bit column -> 2 x uint64 per group (low word first)
 *   sumabs_out[a] (optional, may be NULL or hold NULLs): sum |v| per group for f64 SUM/AVG. */
void oracle_fetch(void* h, int64_t* keys_out, int64_t* count_out, void* const* agg_out, double* const* sumabs_out) {
    Result* r = (Result*)h;
    const Schema& s = r->s;
    uint64_t g = 0;
    for (const auto& kv : r->groups) {
        const Group& G = kv.second;
        if (keys_out) for (int k = 0; k < s.n_keys; ++k) keys_out[g * s.n_keys + k] = kv.first[k];
        if (count_out) count_out[g] = G.count;
        for (int a = 0; a < s.n_aggs; ++a) {
            if (!agg_out || !agg_out[a]) continue;
            int op = s.agg_ops[a];
            int dt = op == O_COUNT ? O_I64 : s.val_dtypes[s.agg_cols[a]];
            const AggState& st = G.a[a];
            if (dt == O_I128 && op != O_COUNT) {
                if (op == O_AVG) {
                    ((double*)agg_out[a])[g] = (double)(__int128)st.qsum / (double)G.count;
                } else {
                    const unsigned __int128 x = op == O_SUM ? st.qsum : (unsigned __int128)st.qmm;
                    ((uint64_t*)agg_out[a])[2 * g] = (uint64_t)x;
                    ((uint64_t*)agg_out[a])[2 * g + 1] = (uint64_t)(x >> 64);
                }
                continue;
            }
            if (op == O_COUNT) {
                ((int64_t*)agg_out[a])[g] = G.count;
            } else if (op == O_SUM) {
                if (dt == O_F64) ((double*)agg_out[a])[g] = (double)st.fsum;
                else ((int64_t*)agg_out[a])[g] = (int64_t)st.isum;
            } else if (op == O_AVG) {
                if (dt == O_F64) ((double*)agg_out[a])[g] = (double)st.fsum / (double)G.count;
                else ((double*)agg_out[a])[g] = (double)(int64_t)st.isum / (double)G.count;
            } else {
                if (dt == O_F64) ((double*)agg_out[a])[g] = st.fmm;
                else ((int64_t*)agg_out[a])[g] = st.imm;
            }
            if (sumabs_out && sumabs_out[a]) sumabs_out[a][g] = (double)st.fabs_sum;
        }
        ++g;
    }
}

void oracle_free(void* h) { delete (Result*)h; }

}  // extern "C"
