/*
 * blu_gen.h — seeded synthetic columnar input generator (test/bench infrastructure).
 *
 * This module only MAKES INPUT COLUMNS. It holds none of the GROUP BY arithmetic: no key
 * packing, no hashing, no aggregation. It is the one piece of code shared by the oracle
 * (oracle/, plain C++) and the CUDA path (the bench/test generator kernels in
 * blugen/csrc/gen.cu), so both sides see identical bits.
 *
 * Shape of the data: a star-schema fact table in the spirit of the
 * paper's TPC-DS store_sales workload (Fig. 4): dictionary-encoded integer
 * grouping codes ("LCOG ... CCAT") plus quantity / money payload columns.
 *
 * Every value is a pure function of (spec, global row index i):
 *     u = splitmix64(seed ^ (stream * 0x9E3779B97F4A7C15) ^ i)
 * and integer-only formulas on u, so host and device produce identical bits.
 *
 * Header-only; usable from C, C++ (g++) and CUDA (nvcc, __host__ __device__).
 */
#ifndef BLU_GEN_H
#define BLU_GEN_H

#include <stdint.h>

#ifdef __CUDACC__
#define BLU_GEN_HD __host__ __device__ __forceinline__
#else
#define BLU_GEN_HD static inline
#endif

#ifdef __cplusplus
extern "C" {
#endif

/* Column kinds. */
typedef enum {
    BLU_GEN_UNIFORM = 0,       /* lo + mulhi(u, hi - lo): integer uniform in [lo, hi)              */
    BLU_GEN_DYADIC = 1,        /* f64 (mulhi(u, 2^21) - 2^20) / 64: every partial sum is exact     */
    BLU_GEN_SPARSE_KEY = 2,    /* bij62(mulhi(u, n_groups)): exactly n_groups distinct codes < 2^62 */
    BLU_GEN_ZIPF_DIGIT = 3,    /* digit of perm[zipf_rank(u)] in a mixed radix (composite key)     */
    BLU_GEN_CYCLIC_DIGIT = 4,  /* digit of (i mod n_groups) in a mixed radix (closed-form tests)   */
    BLU_GEN_LINEAR = 5,        /* a * i + b (two's-complement wrap), closed-form tests             */
    BLU_GEN_REAL = 6,          /* general f64: full 53-bit mantissa, (m * 2^-53 - 0.5) * a          */
    BLU_GEN_UNIFORM_DIGIT = 7  /* digit of mulhi(u, n_groups) in a mixed radix (uniform composite) */
} blu_gen_kind_t;

/* Output element type. Same numbering as blu_dtype_t in blu_gby.h (by convention only). */
typedef enum { BLU_GEN_I32 = 0, BLU_GEN_I64 = 1, BLU_GEN_F64 = 2 } blu_gen_dtype_t;

typedef struct {
    int32_t kind;              /* blu_gen_kind_t                                                   */
    int32_t dtype;             /* blu_gen_dtype_t                                                  */
    uint64_t seed;             /* per-config seed, e.g. 0x5EED0000 + config                         */
    uint64_t stream;           /* counter stream id (columns of one composite key share a stream)  */
    int64_t lo, hi;            /* UNIFORM: [lo, hi). LINEAR: a = lo, b = hi. REAL: scale = lo      */
    uint64_t n_groups;         /* SPARSE_KEY / CYCLIC_DIGIT / UNIFORM_DIGIT: domain size           */
    uint64_t stride;           /* *_DIGIT: digit = (t / stride) % radix                            */
    uint64_t radix;
    const uint64_t* zipf_cdf;  /* ZIPF_DIGIT: table_n thresholds (host or device pointer)          */
    const uint32_t* perm;      /* ZIPF_DIGIT: permutation of [0, table_n) (rank -> tuple index)    */
    uint64_t table_n;
} blu_gen_spec_t;

BLU_GEN_HD uint64_t blu_gen_splitmix64(uint64_t x) {
    x += 0x9E3779B97F4A7C15ull;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
    return x ^ (x >> 31);
}

BLU_GEN_HD uint64_t blu_gen_mulhi(uint64_t a, uint64_t b) {
#ifdef __CUDA_ARCH__
    return __umul64hi(a, b);
#else
    return (uint64_t)(((unsigned __int128)a * (unsigned __int128)b) >> 64);
#endif
}

BLU_GEN_HD uint64_t blu_gen_u(uint64_t seed, uint64_t stream, uint64_t i) {
    return blu_gen_splitmix64(seed ^ (stream * 0x9E3779B97F4A7C15ull) ^ i);
}

/* Bijection on [0, 2^62): odd multiply, xorshift, odd multiply (all mod 2^62). */
BLU_GEN_HD uint64_t blu_gen_bij62(uint64_t r) {
    const uint64_t M = (1ull << 62) - 1ull;
    r = (r * 0x9E3779B97F4A7C15ull) & M;
    r ^= r >> 31;
    r = (r * 0xD6E8FEB86659FD93ull) & M;
    return r;
}

/* Smallest k with u < cdf[k]; cdf is non-decreasing and cdf[n-1] == UINT64_MAX. */
BLU_GEN_HD uint64_t blu_gen_zipf_rank(const uint64_t* cdf, uint64_t n, uint64_t u) {
    uint64_t lo = 0, hi = n - 1;
    while (lo < hi) {
        uint64_t mid = (lo + hi) >> 1;
        if (u < cdf[mid]) hi = mid; else lo = mid + 1;
    }
    return lo;
}

/* Raw 64-bit pattern of element i (reinterpret as int32 (low word), int64 or double). */
BLU_GEN_HD uint64_t blu_gen_bits(const blu_gen_spec_t* s, uint64_t i) {
    uint64_t u = blu_gen_u(s->seed, s->stream, i);
    switch (s->kind) {
    case BLU_GEN_UNIFORM: {
        uint64_t span = (uint64_t)s->hi - (uint64_t)s->lo;
        return (uint64_t)s->lo + blu_gen_mulhi(u, span);
    }
    case BLU_GEN_DYADIC: {
        int64_t k = (int64_t)blu_gen_mulhi(u, 1ull << 21) - (1ll << 20);
        double d = (double)k / 64.0;
        union { double d; uint64_t b; } c; c.d = d; return c.b;
    }
    case BLU_GEN_SPARSE_KEY:
        return blu_gen_bij62(blu_gen_mulhi(u, s->n_groups));
    case BLU_GEN_ZIPF_DIGIT: {
        uint64_t r = blu_gen_zipf_rank(s->zipf_cdf, s->table_n, u);
        uint64_t t = s->perm[r];
        return (t / s->stride) % s->radix;
    }
    case BLU_GEN_CYCLIC_DIGIT:
        return ((i % s->n_groups) / s->stride) % s->radix;
    case BLU_GEN_LINEAR:
        return (uint64_t)s->lo * i + (uint64_t)s->hi;
    case BLU_GEN_REAL: {
        double m = (double)(u >> 11) * (1.0 / 9007199254740992.0); /* [0, 1), 53 bits */
        double d = (m - 0.5) * (double)s->lo;
        union { double d; uint64_t b; } c; c.d = d; return c.b;
    }
    case BLU_GEN_UNIFORM_DIGIT:
        return (blu_gen_mulhi(u, s->n_groups) / s->stride) % s->radix;
    default:
        return 0;
    }
}

#include <math.h>
/* Zipf(s) CDF thresholds over ranks 1..n as u64 fractions of 2^64 (host only).
 * Deterministic for a given libm; both sides receive the same table bytes. */
static inline void blu_gen_zipf_table_host(uint64_t n, double s, uint64_t* out) {
    long double h = 0.0L;
    for (uint64_t k = 1; k <= n; ++k) h += powl((long double)k, -(long double)s);
    long double c = 0.0L;
    for (uint64_t k = 1; k <= n; ++k) {
        c += powl((long double)k, -(long double)s);
        long double f = c / h;
        if (k == n || f >= 1.0L) { out[k - 1] = UINT64_MAX; continue; }
        out[k - 1] = (uint64_t)(f * 18446744073709551616.0L);
    }
    for (uint64_t k = 1; k < n; ++k) if (out[k] < out[k - 1]) out[k] = out[k - 1];
}

/* Fisher-Yates permutation of [0, n) driven by splitmix64 (host only). */
static inline void blu_gen_permutation_host(uint64_t n, uint64_t seed, uint32_t* out) {
    for (uint64_t i = 0; i < n; ++i) out[i] = (uint32_t)i;
    for (uint64_t i = n; i > 1; --i) {
        uint64_t j = blu_gen_mulhi(blu_gen_splitmix64(seed ^ (i * 0xA24BAED4963EE407ull)), i);
        uint32_t t = out[i - 1]; out[i - 1] = out[j]; out[j] = t;
    }
}

/* Fill out[0..n) with rows row0..row0+n-1 (host). */
static inline void blu_gen_fill_host_inline(const blu_gen_spec_t* s, uint64_t row0, uint64_t n,
                                            void* out) {
    if (s->dtype == BLU_GEN_I32) {
        int32_t* o = (int32_t*)out;
        for (uint64_t i = 0; i < n; ++i) o[i] = (int32_t)(uint32_t)blu_gen_bits(s, row0 + i);
    } else {
        uint64_t* o = (uint64_t*)out;
        for (uint64_t i = 0; i < n; ++i) o[i] = blu_gen_bits(s, row0 + i);
    }
}

/* Exported by libblugen.so (blugen/csrc/gen.cu). */
int blu_gen_fill_host(const blu_gen_spec_t* spec, uint64_t row0, uint64_t n, void* out);
/* spec->zipf_cdf / perm must be DEVICE pointers here. stream = cudaStream_t. 0 = ok. */
int blu_gen_fill_device(const blu_gen_spec_t* spec, uint64_t row0, uint64_t n, void* out,
                        void* stream);
void blu_gen_zipf_table(uint64_t n, double s, uint64_t* out);
void blu_gen_permutation(uint64_t n, uint64_t seed, uint32_t* out);

#ifdef __cplusplus
}
#endif
#endif /* BLU_GEN_H */
