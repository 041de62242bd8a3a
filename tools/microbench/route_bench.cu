// route_bench.cu — prototype of the partitioned path (b) pass 2 "route + aggregate" (design study).
//
// Level-1 buckets of (key i64, v0 i64, v1 f64) rows sit in HBM (as after the level-1 scatter). One
// persistent cooperative kernel, one CTA per SM: producer warps stream slices of the current bucket from
// HBM and route every row to its OWNER CTA (a sub-range of the bucket's slot range) through triple-
// buffered per-owner regions in L2; consumer warps aggregate their owner region into a shared-memory
// hash table holding that owner's groups and flush it into the global table at the end of each bucket.
// Producer step s waits for every consumer to finish step s-3; consumer step s waits for every producer
// to finish step s (two monotonic counters). Checked against a naive one-pass global-table kernel.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -lineinfo -o route_bench route_bench.cu
//   ./route_bench G N B1 capbits Tp S block np
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

#include <algorithm>
#include <vector>

#define CK(x)                                                                                  \
  do {                                                                                         \
    cudaError_t e_ = (x);                                                                      \
    if (e_ != cudaSuccess) {                                                                   \
      fprintf(stderr, "%s:%d %s: %s\n", __FILE__, __LINE__, #x, cudaGetErrorString(e_));       \
      exit(1);                                                                                 \
    }                                                                                          \
  } while (0)

constexpr uint64_t kEmpty = ~0ull;

__host__ __device__ __forceinline__ uint64_t fmix64(uint64_t h) {
  h ^= h >> 33;
  h *= 0xff51afd7ed558ccdull;
  h ^= h >> 33;
  h *= 0xc4ceb9fe1a85ec53ull;
  h ^= h >> 33;
  return h;
}
__host__ __device__ __forceinline__ uint64_t splitmix(uint64_t x) {
  x += 0x9E3779B97F4A7C15ull;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
  return x ^ (x >> 31);
}

struct Slot {  // 32-byte global slot (Table-1 style): key, count, sum0, sum1
  unsigned long long key, cnt, s0;
  double s1;
};

__device__ __forceinline__ uint64_t evict_first() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t ldn(const void* a, uint64_t pol) {
  uint64_t v;
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.u64 %0, [%1], %2;" : "=l"(v) : "l"(a), "l"(pol));
  return v;
}
__device__ __forceinline__ uint32_t ld_acq(const uint32_t* a) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(a) : "memory");
  return v;
}
__device__ __forceinline__ void bar_named(int id, int n) { asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory"); }

__device__ __forceinline__ bool g_locate(Slot* t, uint64_t mask, uint64_t key, uint64_t& out) {
  uint64_t idx = fmix64(key) & mask;
  for (int p = 0; p < 4096; ++p) {
    unsigned long long k = __ldcg(&t[idx].key);
    if (k == key) {
      out = idx;
      return true;
    }
    if (k == kEmpty) {
      unsigned long long old = atomicCAS(&t[idx].key, kEmpty, (unsigned long long)key);
      if (old == kEmpty || old == key) {
        out = idx;
        return true;
      }
      continue;  // lost the race to another key: re-read this slot
    }
    idx = (idx + 1) & mask;
  }
  return false;
}

__global__ void k_gen(uint64_t* key, int64_t* v0, double* v1, const uint64_t* gkeys, const uint64_t* goff,
                      const uint64_t* nrows, uint32_t B1, uint64_t seg_stride) {
  for (uint32_t b = blockIdx.y; b < B1; b += gridDim.y) {
    const uint64_t n = nrows[b], g0 = goff[b], ng = goff[b + 1] - goff[b];
    for (uint64_t r = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; r < n; r += (uint64_t)gridDim.x * blockDim.x) {
      const uint64_t u = splitmix(0x5EEDull ^ ((uint64_t)b << 40) ^ r);
      const uint64_t g = g0 + __umul64hi(u, ng);
      const uint64_t i = (uint64_t)b * seg_stride + r;
      key[i] = gkeys[g];
      const uint64_t w = splitmix(u);
      v0[i] = (int64_t)(w >> 33) - (1ll << 30);
      v1[i] = (double)((int64_t)(w & 0x1FFFFF) - (1 << 20)) / 64.0;
    }
  }
}

__global__ void k_init(Slot* t, uint64_t cap) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < cap; i += (uint64_t)gridDim.x * blockDim.x)
    t[i] = Slot{kEmpty, 0ull, 0ull, 0.0};
}

__global__ void k_naive(const uint64_t* key, const int64_t* v0, const double* v1, const uint64_t* nrows, uint32_t B1,
                        uint64_t seg_stride, Slot* t, uint64_t mask, uint32_t* flags) {
  for (uint32_t b = blockIdx.y; b < B1; b += gridDim.y)
    for (uint64_t r = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; r < nrows[b]; r += (uint64_t)gridDim.x * blockDim.x) {
      const uint64_t i = (uint64_t)b * seg_stride + r;
      uint64_t s;
      if (!g_locate(t, mask, key[i], s)) {
        atomicOr(flags, 1u);
        continue;
      }
      atomicAdd(&t[s].cnt, 1ull);
      atomicAdd(&t[s].s0, (unsigned long long)v0[i]);
      atomicAdd(&t[s].s1, v1[i]);
    }
}

__global__ void k_check(const Slot* a, const Slot* b, uint64_t cap, uint64_t mask, unsigned long long* out) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < cap; i += (uint64_t)gridDim.x * blockDim.x) {
    if (a[i].key != kEmpty) atomicAdd(&out[0], 1ull);
    if (b[i].key != kEmpty) atomicAdd(&out[1], 1ull);
    if (a[i].key == kEmpty) continue;
    uint64_t idx = fmix64(a[i].key) & mask;
    bool ok = false;
    for (int p = 0; p < 4096; ++p) {
      if (b[idx].key == a[i].key) {
        ok = a[i].cnt == b[idx].cnt && a[i].s0 == b[idx].s0 && a[i].s1 == b[idx].s1;
        break;
      }
      if (b[idx].key == kEmpty) break;
      idx = (idx + 1) & mask;
    }
    if (!ok) atomicAdd(&out[2], 1ull);
    atomicAdd(&out[3], a[i].cnt);
  }
}

// ------------------------------------------------------------------------------------------------
struct RP {
  const uint64_t* key;
  const int64_t* v0;
  const double* v1;
  const uint64_t* nrows;
  uint32_t B1;
  uint64_t seg_stride;
  Slot* table;
  uint64_t mask;
  uint32_t bshift;  // bits of the slot index below the level-1 bucket bits
  uint4* buf;       // [3][NO][cap_o] x 32 B
  uint32_t cap_o;
  uint32_t* cursor;  // [3][NO]
  uint32_t* prod_done;  // [4]: producers that finished a step = q (mod 4)
  uint32_t* cons_done;  // [4]
  unsigned long long* stats;  // [8] clock totals
  uint32_t mode;
  uint32_t Tp;  // rows per producer slice per step
  uint32_t S;   // smem table entries (multiple of 4)
  uint32_t NP;  // producer warps
  uint32_t* flags;
};

__device__ __forceinline__ uint32_t home4(uint64_t key, uint32_t nbk) {
  return (uint32_t)(((fmix64(key ^ 0x2545F4914F6CDD1Dull) >> 32) * (uint64_t)nbk) >> 32);
}

__global__ void __launch_bounds__(768, 1) k_route(RP p) {
  extern __shared__ __align__(16) uint8_t sm[];
  const uint32_t NO = gridDim.x, me = blockIdx.x, S = p.S;
  // shared layout: table (keys, cnt, lo, hi, f64), step table, producer staging
  uint64_t* tkey = (uint64_t*)sm;
  double* tf = (double*)(tkey + S);
  uint32_t* tcnt = (uint32_t*)(tf + S);
  uint32_t* tlo = tcnt + S;
  uint32_t* thi = tlo + S;
  uint32_t* stepoff = thi + S;  // B1 + 1
  uint32_t* hist = stepoff + p.B1 + 1;  // NO
  uint32_t* off = hist + NO;            // NO
  uint32_t* base = off + NO;            // NO
  volatile uint32_t* misc = base + NO;  // 8
  uint8_t* sown = (uint8_t*)(misc + 8);  // Tp
  uint4* stage = (uint4*)(((uintptr_t)(sown + p.Tp) + 15) & ~(uintptr_t)15);  // Tp x 32 B

  // step schedule (every thread computes it redundantly in smem via thread 0)
  if (threadIdx.x == 0) {
    uint32_t acc = 0;
    for (uint32_t b = 0; b < p.B1; ++b) {
      stepoff[b] = acc;
      acc += (uint32_t)((p.nrows[b] + (uint64_t)NO * p.Tp - 1) / ((uint64_t)NO * p.Tp));
    }
    stepoff[p.B1] = acc;
  }
  __syncthreads();
  const uint32_t ST = stepoff[p.B1];
  const uint32_t PT = p.NP * 32;
  auto bucket_of = [&](uint32_t s) {
    uint32_t lo = 0, hi = p.B1 - 1;
    while (lo < hi) {
      const uint32_t mid = (lo + hi + 1) >> 1;
      if (stepoff[mid] <= s) lo = mid; else hi = mid - 1;
    }
    return lo;
  };
  const uint64_t lowmask = (1ull << p.bshift) - 1;

  if (threadIdx.x < PT) {
    // ------------------------------- producers -------------------------------------------------
    const uint32_t t = threadIdx.x;
    const uint64_t pol = evict_first();
    constexpr int RPT = 8;  // Tp == PT * RPT
    for (uint32_t s = 0; s < ST; ++s) {
      const uint32_t b = bucket_of(s), j = s - stepoff[b], par = s % 3;
      const uint64_t nb = p.nrows[b];
      const uint64_t row0 = ((uint64_t)j * NO + me) * p.Tp;
      long long c0 = clock64();
      if (s >= 3 && t == 0) {
        const uint32_t need = NO * ((s - 3) / 4 + 1);
        while (ld_acq(p.cons_done + (s - 3) % 4) < need) __nanosleep(64);
      }
      for (uint32_t o = t; o < NO; o += PT) hist[o] = 0;
      bar_named(1, PT);
      long long c1 = clock64();
      if (t == 0) atomicAdd(&p.stats[0], (unsigned long long)(c1 - c0));
      uint64_t k[RPT], a[RPT], c[RPT];
      uint32_t own[RPT], rk[RPT];
#pragma unroll
      for (int r = 0; r < RPT; ++r) {
        const uint64_t row = row0 + (uint64_t)r * PT + t;
        own[r] = 0xFFFFFFFFu;
        if (row < nb && row < row0 + p.Tp) {
          const uint64_t i = (uint64_t)b * p.seg_stride + row;
          k[r] = ldn(p.key + i, pol);
          a[r] = ldn(p.v0 + i, pol);
          c[r] = ldn(p.v1 + i, pol);
        }
      }
#pragma unroll
      for (int r = 0; r < RPT; ++r) {
        const uint64_t row = row0 + (uint64_t)r * PT + t;
        if (row < nb && row < row0 + p.Tp) {
          const uint64_t sl = fmix64(k[r]) & p.mask;
          own[r] = (uint32_t)(((sl & lowmask) * NO) >> p.bshift);
          rk[r] = atomicAdd(&hist[own[r]], 1u);
        }
      }
      bar_named(1, PT);
      if (t < 32) {  // exclusive scan of hist into off
        uint32_t carry = 0;
        for (uint32_t o0 = 0; o0 < NO; o0 += 32) {
          const uint32_t o = o0 + t;
          const uint32_t x = o < NO ? hist[o] : 0u;
          uint32_t inc = x;
          for (int d = 1; d < 32; d <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, inc, d);
            if ((int)t >= d) inc += y;
          }
          if (o < NO) off[o] = carry + inc - x;
          carry += __shfl_sync(0xffffffffu, inc, 31);
        }
      }
      for (uint32_t o = t; o < NO; o += PT) {
        const uint32_t h = hist[o];
        if (h) {
          const uint32_t g = atomicAdd(&p.cursor[par * NO + o], h);
          base[o] = g;
          if (g + h > p.cap_o) atomicOr(p.flags, 2u);
        }
      }
      bar_named(1, PT);
#pragma unroll
      for (int r = 0; r < RPT; ++r)
        if (own[r] != 0xFFFFFFFFu) {
          const uint32_t e = off[own[r]] + rk[r];
          stage[2 * e] = make_uint4((uint32_t)k[r], (uint32_t)(k[r] >> 32), (uint32_t)a[r], (uint32_t)(a[r] >> 32));
          stage[2 * e + 1] = make_uint4((uint32_t)c[r], (uint32_t)(c[r] >> 32), 0u, 0u);
          sown[e] = (uint8_t)own[r];
        }
      bar_named(1, PT);
      const uint32_t tot = nb > row0 ? (uint32_t)(nb - row0 < (uint64_t)p.Tp ? nb - row0 : (uint64_t)p.Tp) : 0u;
      for (uint32_t e = t; e < tot && !(p.mode & 2); e += PT) {
        const uint32_t o = sown[e];
        const uint32_t pos = base[o] + (e - off[o]);
        if (pos >= p.cap_o) continue;
        uint4* dst = p.buf + 2 * (((uint64_t)par * NO + o) * p.cap_o + pos);
        dst[0] = stage[2 * e];
        dst[1] = stage[2 * e + 1];
      }
      __threadfence();
      bar_named(1, PT);
      if (t == 0) {
        atomicAdd(p.prod_done + s % 4, 1u);
        atomicAdd(&p.stats[1], (unsigned long long)(clock64() - c1));
      }
    }
  } else {
    // ------------------------------- consumers -------------------------------------------------
    const uint32_t CT = blockDim.x - PT, t = threadIdx.x - PT;
    for (uint32_t e = t; e < S; e += CT) {
      tkey[e] = kEmpty;
      tf[e] = 0.0;
      tcnt[e] = 0;
      tlo[e] = 0;
      thi[e] = 0;
    }
    const uint32_t nbk = S >> 2;
    auto flush = [&]() {
      for (uint32_t e = t; e < S; e += CT) {
        const uint64_t key = tkey[e];
        if (key == kEmpty) continue;
        uint64_t sl;
        if (g_locate(p.table, p.mask, key, sl)) {
          atomicAdd(&p.table[sl].cnt, (unsigned long long)tcnt[e]);
          atomicAdd(&p.table[sl].s0, ((unsigned long long)thi[e] << 32) | tlo[e]);
          atomicAdd(&p.table[sl].s1, tf[e]);
        } else {
          atomicOr(p.flags, 1u);
        }
        tkey[e] = kEmpty;
        tf[e] = 0.0;
        tcnt[e] = 0;
        tlo[e] = 0;
        thi[e] = 0;
      }
    };
    bar_named(2, CT);
    for (uint32_t s = 0; s < ST; ++s) {
      const uint32_t b = bucket_of(s), par = s % 3;
      long long c0 = clock64();
      if (t == 0) {
        const uint32_t need = NO * (s / 4 + 1);
        while (ld_acq(p.prod_done + s % 4) < need) __nanosleep(32);
        misc[0] = *(volatile uint32_t*)&p.cursor[par * NO + me];
      }
      bar_named(2, CT);
      long long c1 = clock64();
      if (t == 0) atomicAdd(&p.stats[2], (unsigned long long)(c1 - c0));
      unsigned long long dummy = 0;
      const uint32_t n = min(misc[0], p.cap_o);
      const uint4* reg = p.buf + 2 * (((uint64_t)par * NO + me) * p.cap_o);
      for (uint32_t i = t; i < n; i += CT) {
        const uint4 x = __ldcg(reg + 2 * i), y = __ldcg(reg + 2 * i + 1);
        const uint64_t key = ((uint64_t)x.y << 32) | x.x;
        const uint64_t v0 = ((uint64_t)x.w << 32) | x.z;
        const double v1 = __longlong_as_double((long long)(((uint64_t)y.y << 32) | y.x));
        if (p.mode & 1) {
          dummy += key ^ v0 ^ (uint64_t)__double_as_longlong(v1);
          continue;
        }
        uint32_t h = home4(key, nbk);
        int e = -1;
        for (int it = 0; it < 32 && e < 0; ++it) {
          const uint64_t* q = tkey + 4 * h;
          const uint64_t k0 = ((volatile uint64_t*)q)[0], k1 = ((volatile uint64_t*)q)[1],
                         k2 = ((volatile uint64_t*)q)[2], k3 = ((volatile uint64_t*)q)[3];
          int m = k0 == key ? 0 : k1 == key ? 1 : k2 == key ? 2 : k3 == key ? 3 : -1;
          if (m < 0) {
            const int z = k0 == kEmpty ? 0 : k1 == kEmpty ? 1 : k2 == kEmpty ? 2 : k3 == kEmpty ? 3 : -1;
            if (z >= 0) {
              const unsigned long long old = atomicCAS((unsigned long long*)(q + z), kEmpty, (unsigned long long)key);
              if (old == kEmpty || old == key) m = z;
            } else {
              h = h + 1 == nbk ? 0u : h + 1;
            }
          }
          if (m >= 0) e = (int)(4 * h + m);
        }
        if (e >= 0) {
          atomicAdd(&tcnt[e], 1u);
          const uint32_t lo = (uint32_t)v0, hi = (uint32_t)(v0 >> 32);
          const uint32_t old = atomicAdd(&tlo[e], lo);
          const uint32_t carry = (old + lo) < old ? 1u : 0u;
          if (hi + carry) atomicAdd(&thi[e], hi + carry);
          atomicAdd(&tf[e], v1);
        } else {
          uint64_t sl;
          if (g_locate(p.table, p.mask, key, sl)) {
            atomicAdd(&p.table[sl].cnt, 1ull);
            atomicAdd(&p.table[sl].s0, (unsigned long long)v0);
            atomicAdd(&p.table[sl].s1, v1);
          } else {
            atomicOr(p.flags, 1u);
          }
        }
      }
      if (dummy == 0x1234567) atomicOr(p.flags, 8u);
      bar_named(2, CT);
      long long c2 = clock64();
      if (t == 0) {
        p.cursor[par * NO + me] = 0;
        __threadfence();
        atomicAdd(p.cons_done + s % 4, 1u);
        atomicAdd(&p.stats[3], (unsigned long long)(c2 - c1));
      }
      if (s + 1 == ST || bucket_of(s + 1) != b) {
        flush();
        bar_named(2, CT);
        if (t == 0) atomicAdd(&p.stats[4], (unsigned long long)(clock64() - c2));
      }
    }
  }
}


// ================================================================================================
// v2: static per-(owner, producer) sub-regions (no global atomics on the hot path), TMA bulk loads of
// the producer's slice into a 2-stage shared-memory ring, a signal warp that publishes producer steps
// (so no producer waits on the release fence), consumers pipelined 4 chunks deep.
// ================================================================================================
struct RP2 {
  const uint64_t* key;
  const int64_t* v0;
  const double* v1;
  const uint64_t* nrows;
  uint32_t B1;
  uint64_t seg_stride;
  Slot* table;
  uint64_t mask;
  uint32_t bshift;
  uint4* sub;        // [3][NO owner][NO producer][CAPP] x 32 B
  uint32_t* cnt;     // [3][NO owner][NO producer]
  uint4* ovf;        // [3][NO][OCAP] x 32 B
  uint32_t* ovc;     // [3][NO]
  uint32_t CAPP, OCAP;
  uint32_t* prod_done;  // [4]
  uint32_t* cons_done;  // [4]
  unsigned long long* stats;
  uint32_t Tp, S, NP, CW;
  uint32_t* flags;
  uint32_t mode;
};

__device__ __forceinline__ void mbar_init(uint64_t* m, uint32_t c) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"((uint32_t)__cvta_generic_to_shared(m)), "r"(c) : "memory");
}
__device__ __forceinline__ void mbar_expect(uint64_t* m, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"((uint32_t)__cvta_generic_to_shared(m)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* m, uint32_t parity) {
  const uint32_t a = (uint32_t)__cvta_generic_to_shared(m);
  uint32_t done = 0;
  while (!done) {
    asm volatile(
        "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
        : "=r"(done)
        : "r"(a), "r"(parity)
        : "memory");
  }
}
__device__ __forceinline__ void tma_load(void* dst, const void* src, uint32_t bytes, uint64_t* m, uint64_t pol) {
  asm volatile("cp.async.bulk.shared::cta.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
                   (uint32_t)__cvta_generic_to_shared(dst)),
               "l"(src), "r"(bytes), "r"((uint32_t)__cvta_generic_to_shared(m)), "l"(pol)
               : "memory");
}
__device__ __forceinline__ void st256(void* p, uint64_t a, uint64_t b, uint64_t c, uint64_t d) {
  asm volatile("st.global.v4.b64 [%0], {%1, %2, %3, %4};" ::"l"(p), "l"(a), "l"(b), "l"(c), "l"(d) : "memory");
}
__device__ __forceinline__ void ld256cg(const void* p, uint64_t& a, uint64_t& b, uint64_t& c, uint64_t& d) {
  asm volatile("ld.global.cg.v4.b64 {%0, %1, %2, %3}, [%4];" : "=l"(a), "=l"(b), "=l"(c), "=l"(d) : "l"(p));
}
__device__ __forceinline__ uint32_t ldcg32(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.global.cg.u32 %0, [%1];" : "=r"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ void bar_arrive(int id, int n) { asm volatile("bar.arrive %0, %1;" ::"r"(id), "r"(n) : "memory"); }

struct Tbl {
  uint64_t* key;
  double* f;
  uint32_t* cnt;
  uint32_t* lo;
  uint32_t* hi;
  uint32_t nbk;
};

// probe + update of R rows held by this lane (convergent 4-way bucket probe, as bucket_body)
template <int R>
__device__ __forceinline__ void tbl_apply(const Tbl& T, const RP2& p, const uint64_t (&key)[R], const uint64_t (&v0)[R],
                                          const double (&v1)[R], uint32_t valid) {
  uint32_t h[R], e[R];
#pragma unroll
  for (int r = 0; r < R; ++r) {
    h[r] = home4(key[r], T.nbk);
    e[r] = 0;
  }
  uint32_t pending = valid, hit = 0;
  for (int it = 0; it < 32 && pending; ++it) {
#pragma unroll
    for (int r = 0; r < R; ++r) {
      if (!(pending >> r & 1)) continue;
      const uint64_t* q = T.key + 4 * h[r];
      const uint64_t k0 = ((volatile const uint64_t*)q)[0], k1 = ((volatile const uint64_t*)q)[1],
                     k2 = ((volatile const uint64_t*)q)[2], k3 = ((volatile const uint64_t*)q)[3];
      const uint64_t kk = key[r];
      int m = k0 == kk ? 0 : k1 == kk ? 1 : k2 == kk ? 2 : k3 == kk ? 3 : -1;
      if (m < 0) {
        const int z = k0 == kEmpty ? 0 : k1 == kEmpty ? 1 : k2 == kEmpty ? 2 : k3 == kEmpty ? 3 : -1;
        if (z >= 0) {
          const unsigned long long old = atomicCAS((unsigned long long*)(q + z), kEmpty, (unsigned long long)kk);
          if (old == kEmpty || old == kk) m = z;
        } else {
          h[r] = h[r] + 1 == T.nbk ? 0u : h[r] + 1;
        }
      }
      if (m >= 0) {
        e[r] = 4 * h[r] + (uint32_t)m;
        pending &= ~(1u << r);
        hit |= 1u << r;
      }
    }
  }
#pragma unroll
  for (int r = 0; r < R; ++r) {
    if (hit >> r & 1) {
      const uint32_t x = e[r];
      atomicAdd(&T.cnt[x], 1u);
      const uint32_t lo = (uint32_t)v0[r], hi = (uint32_t)(v0[r] >> 32);
      const uint32_t old = atomicAdd(&T.lo[x], lo);
      const uint32_t carry = (old + lo) < old ? 1u : 0u;
      if (hi + carry) atomicAdd(&T.hi[x], hi + carry);
      atomicAdd(&T.f[x], v1[r]);
    } else if (pending >> r & 1) {
      uint64_t sl;
      if (g_locate(p.table, p.mask, key[r], sl)) {
        atomicAdd(&p.table[sl].cnt, 1ull);
        atomicAdd(&p.table[sl].s0, (unsigned long long)v0[r]);
        atomicAdd(&p.table[sl].s1, v1[r]);
      } else {
        atomicOr(p.flags, 1u);
      }
    }
  }
}

__global__ void __launch_bounds__(1024, 1) k_route2(RP2 p) {
  extern __shared__ __align__(16) uint8_t sm[];
  const uint32_t NO = gridDim.x, me = blockIdx.x, S = p.S, Tp = p.Tp;
  // shared layout: input ring (2 stages x 3 columns x Tp x 8 B), table, schedule, histograms, mbarriers
  uint64_t* ring = (uint64_t*)sm;  // [2][3][Tp]
  uint64_t* tkey = ring + 6 * (size_t)Tp;
  double* tf = (double*)(tkey + S);
  uint32_t* tcnt = (uint32_t*)(tf + S);
  uint32_t* tlo = tcnt + S;
  uint32_t* thi = tlo + S;
  uint32_t* stepoff = thi + S;           // B1 + 1
  uint32_t* hist = stepoff + p.B1 + 1;   // [3][NO]
  uint64_t* mbar = (uint64_t*)(((uintptr_t)(hist + 3 * NO) + 7) & ~(uintptr_t)7);  // [2]
  uint32_t* cpre = (uint32_t*)(mbar + 2);  // NO + 2 (consumers)
  if (threadIdx.x == 0) {
    uint32_t acc = 0;
    for (uint32_t b = 0; b < p.B1; ++b) {
      stepoff[b] = acc;
      acc += (uint32_t)((p.nrows[b] + (uint64_t)NO * Tp - 1) / ((uint64_t)NO * Tp));
    }
    stepoff[p.B1] = acc;
    mbar_init(&mbar[0], 1);
    mbar_init(&mbar[1], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  for (uint32_t i = threadIdx.x; i < 3 * NO; i += blockDim.x) hist[i] = 0;
  __syncthreads();
  const uint32_t ST = stepoff[p.B1];
  const uint32_t PT = p.NP * 32, CT = p.CW * 32;
  auto bucket_of = [&](uint32_t s) {
    uint32_t lo = 0, hi = p.B1 - 1;
    while (lo < hi) {
      const uint32_t mid = (lo + hi + 1) >> 1;
      if (stepoff[mid] <= s) lo = mid; else hi = mid - 1;
    }
    return lo;
  };
  const uint64_t lowmask = (1ull << p.bshift) - 1;
  const uint64_t pol = evict_first();
  // slice of step s: rows [row0, row1) of bucket b
  auto slice = [&](uint32_t s, uint32_t& b, uint64_t& row0, uint32_t& n) {
    b = bucket_of(s);
    const uint32_t j = s - stepoff[b];
    const uint64_t nb = p.nrows[b];
    row0 = ((uint64_t)j * NO + me) * Tp;
    n = nb > row0 ? (uint32_t)(nb - row0 < Tp ? nb - row0 : Tp) : 0u;
  };
  auto issue = [&](uint32_t s) {  // thread 0 of the producers
    uint32_t b, n;
    uint64_t row0;
    slice(s, b, row0, n);
    const uint32_t st = s & 1;
    const uint32_t bytes = ((n * 8) + 15) & ~15u;
    mbar_expect(&mbar[st], 3 * bytes);
    if (bytes) {
      const uint64_t i = (uint64_t)b * p.seg_stride + row0;
      tma_load(ring + (size_t)(st * 3 + 0) * Tp, p.key + i, bytes, &mbar[st], pol);
      tma_load(ring + (size_t)(st * 3 + 1) * Tp, p.v0 + i, bytes, &mbar[st], pol);
      tma_load(ring + (size_t)(st * 3 + 2) * Tp, p.v1 + i, bytes, &mbar[st], pol);
    }
  };
  const uint32_t w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x < PT) {
    // ------------------------------- producers -------------------------------------------------
    const uint32_t t = threadIdx.x;
    if (t == 0) {
      if (ST > 0 && !(p.mode & 4)) issue(0);
      if (ST > 1 && !(p.mode & 4)) issue(1);
    }
    long long cw = 0, cwork = 0;
    for (uint32_t s = 0; s < ST; ++s) {
      const uint32_t par = s % 3, st = s & 1;
      uint32_t b, n;
      uint64_t row0;
      slice(s, b, row0, n);
      long long c0 = clock64();
      // buffer `par` is free once every consumer finished step s - 3
      if (s >= 3 && lane == 0) {
        const uint32_t need = NO * ((s - 3) / 4 + 1);
        const volatile uint32_t* cd = p.cons_done + (s - 3) % 4;
        while (*cd < need) __nanosleep(64);
        asm volatile("fence.acq_rel.gpu;" ::: "memory");
      }
      __syncwarp();
      for (uint32_t o = t; o < NO; o += PT) hist[((s + 1) % 3) * NO + o] = 0;  // used by step s - 2
      if (!(p.mode & 4)) mbar_wait(&mbar[st], (s >> 1) & 1);
      if (p.mode & 4) n = 0;
      long long c1 = clock64();
      cw += c1 - c0;
      const uint64_t* rk = ring + (size_t)(st * 3 + 0) * Tp;
      const uint64_t* ra = ring + (size_t)(st * 3 + 1) * Tp;
      const uint64_t* rc = ring + (size_t)(st * 3 + 2) * Tp;
      uint32_t* hp = hist + par * NO;
      for (uint32_t r = t; r < n; r += PT) {
        const uint64_t k = rk[r], a = ra[r], c = rc[r];
        const uint64_t sl = fmix64(k) & p.mask;
        const uint32_t o = (uint32_t)(((sl & lowmask) * NO) >> p.bshift);
        const uint32_t q = atomicAdd(&hp[o], 1u);
        if (!(p.mode & 2)) {
          if (q < p.CAPP) {
            st256(p.sub + 2 * ((((uint64_t)par * NO + o) * NO + me) * p.CAPP + q), k, a, c, 0);
          } else {
            const uint32_t pos = atomicAdd(&p.cnt[((uint64_t)par * NO + o) * (NO + 4) + NO], 1u);
            if (pos < p.OCAP) st256(p.ovf + 2 * (((uint64_t)par * NO + o) * p.OCAP + pos), k, a, c, 0);
            else atomicOr(p.flags, 2u);
          }
        }
      }
      bar_named(1, PT);  // ring stage consumed, hist[par] final
      if (t == 0 && s + 2 < ST && !(p.mode & 4)) issue(s + 2);
      for (uint32_t o = t; o < NO; o += PT) {
        const uint32_t h = hp[o];
        p.cnt[((uint64_t)par * NO + o) * (NO + 4) + me] = h < p.CAPP ? h : p.CAPP;
      }
      bar_arrive(3 + par, PT + 32);  // the signal warp publishes step s
      cwork += clock64() - c1;
    }
    if (t == 0) {
      atomicAdd(&p.stats[0], (unsigned long long)cw);
      atomicAdd(&p.stats[1], (unsigned long long)cwork);
    }
  } else if (threadIdx.x < PT + 32) {
    // ------------------------------- signal warp ----------------------------------------------
    for (uint32_t s = 0; s < ST; ++s) {
      bar_named(3 + s % 3, PT + 32);
      if (lane == 0) {
        __threadfence();
        atomicAdd(p.prod_done + s % 4, 1u);
      }
    }
  } else {
    // ------------------------------- consumers -------------------------------------------------
    if (threadIdx.x >= PT + 32 + CT) {  // consumer signal warp: publishes consumer steps
      for (uint32_t s = 0; s < ST; ++s) {
        bar_named(6 + s % 3, CT + 32);
        if (lane == 0) {
          __threadfence();
          atomicAdd(p.cons_done + s % 4, 1u);
        }
      }
      return;
    }
    const uint32_t t = threadIdx.x - PT - 32, cw_ = t >> 5;
    for (uint32_t e = t; e < S; e += CT) {
      tkey[e] = kEmpty;
      tf[e] = 0.0;
      tcnt[e] = 0;
      tlo[e] = 0;
      thi[e] = 0;
    }
    Tbl T{tkey, tf, tcnt, tlo, thi, S >> 2};
    const uint32_t RW = NO + 4;  // count row: NO producer counts, then the overflow cursor
    // every consumer warp is independent: it owns the producer chunks q = cw_ + CW * lane (<= 32 per
    // warp) and joins the others only through the signal warp's barrier (and at bucket ends)
    const uint32_t my_chunk = cw_ + p.CW * lane;
    const bool has_chunk = my_chunk < NO;
    bar_named(2, CT);
    long long cwt = 0, cwork = 0, cfl = 0;
    for (uint32_t s = 0; s < ST; ++s) {
      const uint32_t par = s % 3;
      const uint32_t b = bucket_of(s);
      long long c0 = clock64();
      if (lane == 0) {
        const uint32_t need = NO * (s / 4 + 1);
        const volatile uint32_t* pd = p.prod_done + s % 4;
        while (*pd < need) __nanosleep(32);
        asm volatile("fence.acq_rel.gpu;" ::: "memory");
      }
      __syncwarp();
      long long c1 = clock64();
      cwt += c1 - c0;
      const uint32_t* row = p.cnt + ((uint64_t)par * NO + me) * RW;
      const uint32_t n_mine = has_chunk && !(p.mode & 4) ? ldcg32(row + my_chunk) : 0u;
      uint32_t inc = n_mine;  // inclusive scan over the warp's chunks
#pragma unroll
      for (int d = 1; d < 32; d <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, inc, d);
        if ((int)lane >= d) inc += y;
      }
      const uint32_t excl = inc - n_mine;
      const uint32_t total = __shfl_sync(0xffffffffu, inc, 31);
      const uint4* base = p.sub + 2 * (((uint64_t)par * NO + me) * NO) * p.CAPP;
      constexpr int R = 4;
      for (uint32_t j0 = 0; j0 < total; j0 += 32 * R) {
        uint64_t key[R], a[R], c[R], d;
        double v1[R];
        uint32_t valid = 0;
#pragma unroll
        for (int r = 0; r < R; ++r) {
          const uint32_t j = j0 + 32 * r + lane;
          key[r] = kEmpty;
          // chunk of record j: the last lane q whose exclusive prefix is <= j
          const uint32_t ball = __ballot_sync(0xffffffffu, excl <= j0 + 32 * r);  // lanes <= any j of this row
          (void)ball;
          uint32_t q = 0;
#pragma unroll
          for (int st = 16; st >= 1; st >>= 1) {
            const uint32_t e = __shfl_sync(0xffffffffu, excl, q + st < 32 ? q + st : 31);
            if (q + st < 32 && e <= j) q += st;
          }
          const uint32_t eq = __shfl_sync(0xffffffffu, excl, q);
          if (j < total) {
            const uint32_t chunk = cw_ + p.CW * q;
            ld256cg(base + 2 * ((uint64_t)chunk * p.CAPP + (j - eq)), key[r], a[r], c[r], d);
            valid |= 1u << r;
          }
        }
#pragma unroll
        for (int r = 0; r < R; ++r) v1[r] = __longlong_as_double((long long)c[r]);
        if (!(p.mode & 1)) tbl_apply<R>(T, p, key, a, v1, valid);
      }
      if (cw_ == 0) {  // rows beyond a producer chunk's capacity (rare)
        const uint32_t novf = min(ldcg32(row + NO), p.OCAP);
        const uint4* ob = p.ovf + 2 * ((uint64_t)par * NO + me) * p.OCAP;
        for (uint32_t i = lane; i < novf; i += 32) {
          uint64_t key[1], a[1], c, d;
          double v1[1];
          ld256cg(ob + 2 * i, key[0], a[0], c, d);
          v1[0] = __longlong_as_double((long long)c);
          tbl_apply<1>(T, p, key, a, v1, 1u);
        }
        __syncwarp();
        if (lane == 0) p.cnt[((uint64_t)par * NO + me) * RW + NO] = 0;
      }
      __syncwarp();
      bar_arrive(6 + par, CT + 32);  // the consumer signal warp publishes step s once every warp arrived
      long long c2 = clock64();
      cwork += c2 - c1;
      if (s + 1 == ST || bucket_of(s + 1) != b) {
        bar_named(2, CT);
        for (uint32_t e = t; e < S; e += CT) {
          const uint64_t key = tkey[e];
          if (key == kEmpty) continue;
          uint64_t sl;
          if (g_locate(p.table, p.mask, key, sl)) {
            atomicAdd(&p.table[sl].cnt, (unsigned long long)tcnt[e]);
            atomicAdd(&p.table[sl].s0, ((unsigned long long)thi[e] << 32) | tlo[e]);
            atomicAdd(&p.table[sl].s1, tf[e]);
          } else {
            atomicOr(p.flags, 1u);
          }
          tkey[e] = kEmpty;
          tf[e] = 0.0;
          tcnt[e] = 0;
          tlo[e] = 0;
          thi[e] = 0;
        }
        bar_named(2, CT);
        cfl += clock64() - c2;
      }
    }
    if (t == 0) {
      atomicAdd(&p.stats[2], (unsigned long long)cwt);
      atomicAdd(&p.stats[3], (unsigned long long)cwork);
      atomicAdd(&p.stats[4], (unsigned long long)cfl);
    }
  }
}

static void run_v2(int sms, uint64_t tot, const uint64_t* d_key, const int64_t* d_v0, const double* d_v1,
                   const uint64_t* d_nrows, uint32_t B1, uint64_t seg_stride, Slot* t1, uint64_t cap, uint64_t mask,
                   uint32_t bshift, uint32_t Tp, uint32_t S, uint32_t NP, uint32_t CW, uint32_t CAPP, int reps,
                   uint32_t mode, uint32_t* flags, unsigned long long* stats) {
  RP2 p{};
  p.key = d_key;
  p.v0 = d_v0;
  p.v1 = d_v1;
  p.nrows = d_nrows;
  p.B1 = B1;
  p.seg_stride = seg_stride;
  p.table = t1;
  p.mask = mask;
  p.bshift = bshift;
  p.CAPP = CAPP;
  p.OCAP = 4096;
  CK(cudaMalloc(&p.sub, 3ull * sms * sms * CAPP * 32));
  CK(cudaMalloc(&p.cnt, 3ull * sms * (sms + 4) * 4));
  CK(cudaMemset(p.cnt, 0, 3ull * sms * (sms + 4) * 4));
  CK(cudaMalloc(&p.ovf, 3ull * sms * p.OCAP * 32));
  uint32_t* ctr;
  CK(cudaMalloc(&ctr, (3 * sms + 16) * 4));
  p.ovc = ctr;
  p.prod_done = ctr + 3 * sms;
  p.cons_done = ctr + 3 * sms + 4;
  p.stats = stats;
  p.Tp = Tp;
  p.S = S;
  p.NP = NP;
  p.CW = CW;
  p.flags = flags;
  p.mode = mode;
  const uint32_t block = (NP + 2 + CW) * 32;
  const size_t smem = (size_t)6 * Tp * 8 + (size_t)S * 28 + (B1 + 1) * 4 + 3 * sms * 4 + 16 + 64 + (sms + 2) * 4;
  printf("v2: Tp %u S %u NP %u CW %u CAPP %u block %u smem %zu L2 sub-regions %.1f MB\n", Tp, S, NP, CW, CAPP, block,
         smem, 3.0 * sms * sms * CAPP * 32 / 1e6);
  if (smem > 232448 || block > 1024) {
    printf("v2: does not fit\n");
    return;
  }
  CK(cudaFuncSetAttribute(k_route2, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  for (int rep = 0; rep < reps; ++rep) {
    k_init<<<sms * 8, 256>>>(t1, cap);
    CK(cudaMemset(ctr, 0, (3 * sms + 16) * 4));
    CK(cudaMemset(stats, 0, 64));
    CK(cudaMemset(flags, 0, 64));
    void* args[] = {&p};
    cudaEventRecord(e0);
    CK(cudaLaunchCooperativeKernel((void*)k_route2, dim3(sms), dim3(block), args, smem, 0));
    cudaEventRecord(e1);
    CK(cudaDeviceSynchronize());
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    uint32_t hf = 0;
    CK(cudaMemcpy(&hf, flags, 4, cudaMemcpyDeviceToHost));
    unsigned long long hs[8];
    CK(cudaMemcpy(hs, stats, 64, cudaMemcpyDeviceToHost));
    const double cyc = (double)sms * ms * 1.965e6;
    printf("route2: %.3f ms  %.1f G rows/s  %.0f GB/s (24 B/row)  flags %u | prod wait %.2f work %.2f | cons wait %.2f work %.2f flush %.2f\n",
           ms, tot / ms / 1e6, tot * 24.0 / ms / 1e6, hf, hs[0] / cyc, hs[1] / cyc, hs[2] / cyc, hs[3] / cyc, hs[4] / cyc);
  }
  cudaFree(p.sub);
  cudaFree(p.cnt);
  cudaFree(p.ovf);
  cudaFree(ctr);
}

int main(int argc, char** argv) {
  const uint64_t G = argc > 1 ? strtoull(argv[1], 0, 10) : 10000000ull;
  const uint64_t N = argc > 2 ? strtoull(argv[2], 0, 10) : 1000000000ull;
  const uint32_t B1 = argc > 3 ? atoi(argv[3]) : 32;
  const uint32_t cb = argc > 4 ? atoi(argv[4]) : 24;
  const uint32_t Tp = argc > 5 ? atoi(argv[5]) : 2048;
  const uint32_t S = argc > 6 ? atoi(argv[6]) : 4096;
  const uint32_t block = argc > 7 ? atoi(argv[7]) : 768;
  const uint32_t NP = argc > 8 ? atoi(argv[8]) : 8;
  const int reps = argc > 9 ? atoi(argv[9]) : 3;
  const uint32_t mode = argc > 10 ? atoi(argv[10]) : 0;
  const uint32_t ver = argc > 11 ? atoi(argv[11]) : 2;
  const uint32_t CW = argc > 12 ? atoi(argv[12]) : 16;
  const uint32_t CAPP = argc > 13 ? atoi(argv[13]) : 32;
  int sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  const uint64_t cap = 1ull << cb, mask = cap - 1;
  uint32_t lb1 = 0;
  while ((1u << lb1) < B1) ++lb1;
  const uint32_t bshift = cb - lb1;
  // groups per bucket (host)
  std::vector<std::vector<uint64_t>> per(B1);
  for (uint64_t g = 0; g < G; ++g) {
    const uint64_t key = splitmix(g * 7919 + 17) & ((1ull << 62) - 1);
    per[(fmix64(key) & mask) >> bshift].push_back(key);
  }
  std::vector<uint64_t> gk, goff(B1 + 1), nrows(B1);
  uint64_t maxr = 0, tot = 0;
  for (uint32_t b = 0; b < B1; ++b) {
    goff[b] = gk.size();
    gk.insert(gk.end(), per[b].begin(), per[b].end());
    nrows[b] = (uint64_t)((double)N * per[b].size() / G);
    maxr = std::max(maxr, nrows[b]);
    tot += nrows[b];
  }
  goff[B1] = gk.size();
  const uint64_t seg_stride = (maxr + 63) & ~63ull;
  printf("G %llu N %llu B1 %u cap 2^%u Tp %u S %u block %u NP %u sms %d: groups/owner %.0f (load %.2f) steps/bucket %.1f\n",
         (unsigned long long)G, (unsigned long long)tot, B1, cb, Tp, S, block, NP, sms, (double)G / B1 / sms,
         (double)G / B1 / sms / S, (double)tot / B1 / ((double)sms * Tp));
  uint64_t *d_key, *d_gk, *d_goff, *d_nrows;
  int64_t* d_v0;
  double* d_v1;
  CK(cudaMalloc(&d_key, seg_stride * B1 * 8));
  CK(cudaMalloc(&d_v0, seg_stride * B1 * 8));
  CK(cudaMalloc(&d_v1, seg_stride * B1 * 8));
  CK(cudaMalloc(&d_gk, gk.size() * 8));
  CK(cudaMalloc(&d_goff, goff.size() * 8));
  CK(cudaMalloc(&d_nrows, nrows.size() * 8));
  CK(cudaMemcpy(d_gk, gk.data(), gk.size() * 8, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(d_goff, goff.data(), goff.size() * 8, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(d_nrows, nrows.data(), nrows.size() * 8, cudaMemcpyHostToDevice));
  k_gen<<<dim3(sms * 4, 16), 256>>>(d_key, d_v0, d_v1, d_gk, d_goff, d_nrows, B1, seg_stride);
  CK(cudaDeviceSynchronize());
  Slot *t1, *t2;
  CK(cudaMalloc(&t1, cap * sizeof(Slot)));
  CK(cudaMalloc(&t2, cap * sizeof(Slot)));
  uint32_t* flags;
  CK(cudaMalloc(&flags, 64));
  unsigned long long* chk;
  CK(cudaMalloc(&chk, 64));
  const uint32_t cap_o = (uint32_t)(Tp * 1.25) + 256;
  uint4* buf;
  CK(cudaMalloc(&buf, 3ull * sms * cap_o * 32));
  uint32_t* ctr;
  CK(cudaMalloc(&ctr, (3 * sms + 16) * 4));
  unsigned long long* stats;
  CK(cudaMalloc(&stats, 64));
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  // reference
  k_init<<<sms * 8, 256>>>(t2, cap);
  CK(cudaMemset(flags, 0, 64));
  cudaEventRecord(e0);
  k_naive<<<dim3(sms * 8, 4), 256>>>(d_key, d_v0, d_v1, d_nrows, B1, seg_stride, t2, mask, flags);
  cudaEventRecord(e1);
  CK(cudaDeviceSynchronize());
  float ms = 0;
  cudaEventElapsedTime(&ms, e0, e1);
  printf("naive one-pass: %.2f ms (%.1f G rows/s)\n", ms, tot / ms / 1e6);
  if (ver == 2) {
    unsigned long long* st2;
    CK(cudaMalloc(&st2, 64));
    run_v2(sms, tot, d_key, d_v0, d_v1, d_nrows, B1, seg_stride, t1, cap, mask, bshift, Tp, S, NP, CW, CAPP, reps, mode,
           flags, st2);
  } else {
  // route kernel
  RP p{};
  p.key = d_key;
  p.v0 = d_v0;
  p.v1 = d_v1;
  p.nrows = d_nrows;
  p.B1 = B1;
  p.seg_stride = seg_stride;
  p.table = t1;
  p.mask = mask;
  p.bshift = bshift;
  p.buf = buf;
  p.cap_o = cap_o;
  p.cursor = ctr;
  p.prod_done = ctr + 3 * sms;
  p.cons_done = ctr + 3 * sms + 4;
  p.stats = stats;
  p.mode = mode;
  p.Tp = Tp;
  p.S = S;
  p.NP = NP;
  p.flags = flags;
  const size_t smem = (size_t)S * 28 + (B1 + 1) * 4 + 3 * sms * 4 + 32 + Tp + 16 + (size_t)Tp * 32;
  if (smem > 232448) {
    printf("smem %zu too large\n", smem);
    return 1;
  }
  CK(cudaFuncSetAttribute(k_route, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int nb = 0;
  CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_route, block, smem));
  printf("smem %zu B, blocks/SM %d, L2 buffer %.1f MB\n", smem, nb, 3.0 * sms * cap_o * 32 / 1e6);
  if (Tp != NP * 32 * 8) {
    printf("Tp must equal NP*32*8\n");
    return 1;
  }
  for (int rep = 0; rep < reps; ++rep) {
    k_init<<<sms * 8, 256>>>(t1, cap);
    CK(cudaMemset(ctr, 0, (3 * sms + 16) * 4));
    CK(cudaMemset(stats, 0, 64));
    CK(cudaMemset(flags, 0, 64));
    void* args[] = {&p};
    cudaEventRecord(e0);
    CK(cudaLaunchCooperativeKernel((void*)k_route, dim3(sms), dim3(block), args, smem, 0));
    cudaEventRecord(e1);
    CK(cudaDeviceSynchronize());
    cudaEventElapsedTime(&ms, e0, e1);
    uint32_t hf = 0;
    CK(cudaMemcpy(&hf, flags, 4, cudaMemcpyDeviceToHost));
    unsigned long long hs[8];
    CK(cudaMemcpy(hs, stats, 64, cudaMemcpyDeviceToHost));
    const double cyc = (double)sms * ms * 1.965e6;  // SM-cycles in the launch
    printf("route: %.3f ms  %.1f G rows/s  %.0f GB/s (24 B/row)  flags %u | prod wait %.2f work %.2f | cons wait %.2f work %.2f flush %.2f (fractions of SM time)\n",
           ms, tot / ms / 1e6, tot * 24.0 / ms / 1e6, hf, hs[0] / cyc, hs[1] / cyc, hs[2] / cyc, hs[3] / cyc, hs[4] / cyc);
  }
  }
  CK(cudaMemset(chk, 0, 64));
  k_check<<<sms * 8, 256>>>(t1, t2, cap, mask, chk);
  unsigned long long hc[4];
  CK(cudaMemcpy(hc, chk, 32, cudaMemcpyDeviceToHost));
  printf("check: groups route %llu naive %llu mismatches %llu rows %llu (expect %llu) -> %s\n", hc[0], hc[1], hc[2],
         hc[3], (unsigned long long)tot, (hc[0] == hc[1] && hc[2] == 0 && hc[3] == tot) ? "OK" : "FAIL");
  return 0;
}
