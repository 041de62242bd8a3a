// route3_bench.cu — design study v3 for the partitioned path (b) pass 2 "route + aggregate".
// Same dataflow as route_bench.cu v2 (level-1 buckets in HBM -> producers route rows to the owner CTA
// through per-(owner, producer) sub-regions in L2 -> consumers aggregate in shared memory), with the
// synchronisation rebuilt for latency:
//   * NBUF step buffers (template), monotonic counters mod NBUF+1;
//   * per CTA one poller warp per direction turns the global counters into a CTA-local "ready" word
//     (st.release.cta.shared), so working warps poll shared memory, not L2;
//   * per CTA one signal warp per direction publishes completed steps (bar.sync -> fence -> atomic),
//     so no working warp waits on a release fence.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -lineinfo -o route3_bench route3_bench.cu
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

struct Slot {
  unsigned long long key, cnt, s0;
  double s1;
};

__device__ __forceinline__ uint64_t evict_first() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ void bar_named(int id, int n) { asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory"); }
__device__ __forceinline__ void bar_arrive(int id, int n) { asm volatile("bar.arrive %0, %1;" ::"r"(id), "r"(n) : "memory"); }
__device__ __forceinline__ void st_rel_cta(uint32_t* p, uint32_t v) {
  asm volatile("st.release.cta.shared.u32 [%0], %1;" ::"r"((uint32_t)__cvta_generic_to_shared(p)), "r"(v) : "memory");
}
__device__ __forceinline__ uint32_t ld_acq_cta(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.cta.shared.u32 %0, [%1];" : "=r"(v) : "r"((uint32_t)__cvta_generic_to_shared(p)) : "memory");
  return v;
}
__device__ __forceinline__ void wait_local(const uint32_t* flag, uint32_t need) {
  while (ld_acq_cta(flag) < need) __nanosleep(20);
}
__device__ __forceinline__ void wait_global(const uint32_t* ctr, uint32_t need) {
  const volatile uint32_t* v = ctr;
  while (*v < need) __nanosleep(40);
  asm volatile("fence.acq_rel.gpu;" ::: "memory");
}
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
  while (!done)
    asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
                 : "=r"(done)
                 : "r"(a), "r"(parity)
                 : "memory");
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
      continue;
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

struct RP {
  const uint64_t* key;
  const int64_t* v0;
  const double* v1;
  const uint64_t* nrows;
  uint32_t B1;
  uint64_t seg_stride;
  Slot* table;
  uint64_t mask;
  uint32_t bshift;
  uint4* sub;     // [NBUF][NO owner][NO producer][CAPP] x 32 B
  uint32_t* cnt;  // [NBUF][NO owner][NO + 4]: producer counts, then the overflow cursor
  uint4* ovf;     // [NBUF][NO][OCAP] x 32 B
  uint32_t CAPP, OCAP;
  uint32_t* prod_done;  // [NBUF + 1]
  uint32_t* cons_done;  // [NBUF + 1]
  unsigned long long* stats;
  uint32_t Tp, S, NP, CW;
  uint32_t* flags;
  uint32_t mode;
  uint32_t l2frac;  // keys whose hash byte is below this go straight to the global table (L2 REDs)
};

__device__ __forceinline__ uint32_t home4(uint64_t key, uint32_t nbk) {
  return (uint32_t)(((fmix64(key ^ 0x2545F4914F6CDD1Dull) >> 32) * (uint64_t)nbk) >> 32);
}

struct Tbl {
  uint64_t* key;
  double* f;
  uint32_t* cnt;
  uint32_t* lo;
  uint32_t* hi;
  uint32_t nbk;
};

template <int R>
__device__ __forceinline__ void tbl_apply(const Tbl& T, const RP& p, const uint64_t (&key)[R], const uint64_t (&v0)[R],
                                          const double (&v1)[R], uint32_t valid) {
  uint32_t h[R], e[R];
  uint32_t glob = 0;
#pragma unroll
  for (int r = 0; r < R; ++r) {
    const uint64_t hh = fmix64(key[r] ^ 0x2545F4914F6CDD1Dull);
    h[r] = (uint32_t)(((hh >> 32) * (uint64_t)T.nbk) >> 32);
    if ((uint32_t)(hh & 255) < p.l2frac) glob |= 1u << r;
    e[r] = 0;
  }
  valid &= ~glob;
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
    } else if ((pending | glob) >> r & 1) {
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

// warp roles: [0, NP) producers | NP: producer signal | NP+1: producer-ready poller | NP+2: consumer-
// ready poller | NP+3: consumer signal | [NP+4, NP+4+CW) consumers
template <int NBUF>
__global__ void __launch_bounds__(1024, 1) k_route3(RP p) {
  extern __shared__ __align__(16) uint8_t sm[];
  constexpr uint32_t M = NBUF + 1;
  const uint32_t NO = gridDim.x, me = blockIdx.x, S = p.S, Tp = p.Tp;
  uint64_t* ring = (uint64_t*)sm;  // [2][3][Tp]
  uint64_t* tkey = ring + 6 * (size_t)Tp;
  double* tf = (double*)(tkey + S);
  uint32_t* tcnt = (uint32_t*)(tf + S);
  uint32_t* tlo = tcnt + S;
  uint32_t* thi = tlo + S;
  uint32_t* stepoff = thi + S;          // B1 + 1
  uint32_t* hist = stepoff + p.B1 + 1;  // [NBUF][NO]
  uint32_t* ready = hist + NBUF * NO;   // [0] producer steps ready, [1] consumer steps done (CTA-local view)
  uint64_t* mbar = (uint64_t*)(((uintptr_t)(ready + 4) + 7) & ~(uintptr_t)7);  // [2]
  if (threadIdx.x == 0) {
    uint32_t acc = 0;
    for (uint32_t b = 0; b < p.B1; ++b) {
      stepoff[b] = acc;
      acc += (uint32_t)((p.nrows[b] + (uint64_t)NO * Tp - 1) / ((uint64_t)NO * Tp));
    }
    stepoff[p.B1] = acc;
    ready[0] = 0;
    ready[1] = 0;
    mbar_init(&mbar[0], 1);
    mbar_init(&mbar[1], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  for (uint32_t i = threadIdx.x; i < NBUF * NO; i += blockDim.x) hist[i] = 0;
  __syncthreads();
  const uint32_t ST = stepoff[p.B1];
  const uint32_t PT = p.NP * 32, CT = p.CW * 32;
  const uint32_t w = threadIdx.x >> 5, lane = threadIdx.x & 31;
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
  auto slice = [&](uint32_t s, uint32_t& b, uint64_t& row0, uint32_t& n) {
    b = bucket_of(s);
    const uint32_t j = s - stepoff[b];
    const uint64_t nb = p.nrows[b];
    row0 = ((uint64_t)j * NO + me) * Tp;
    n = nb > row0 ? (uint32_t)(nb - row0 < Tp ? nb - row0 : Tp) : 0u;
  };
  auto issue = [&](uint32_t s) {
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
  const uint32_t RW = NO + 4;
  if (w < p.NP) {
    // ------------------------------- producers -------------------------------------------------
    const uint32_t t = threadIdx.x;
    if (t == 0 && !(p.mode & 4)) {
      if (ST > 0) issue(0);
      if (ST > 1) issue(1);
    }
    long long cw = 0, cwork = 0;
    for (uint32_t s = 0; s < ST; ++s) {
      const uint32_t par = s % NBUF, st = s & 1;
      uint32_t b, n;
      uint64_t row0;
      slice(s, b, row0, n);
      long long c0 = clock64();
      if (s >= NBUF) wait_local(&ready[1], s - NBUF + 1);  // buffer `par` consumed everywhere (step s - NBUF)
      for (uint32_t o = t; o < NO; o += PT) hist[((s + 1) % NBUF) * NO + o] = 0;  // last used by step s + 1 - NBUF
      if (!(p.mode & 4)) mbar_wait(&mbar[st], (s >> 1) & 1);
      else n = 0;
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
        if (q < p.CAPP) {
          st256(p.sub + 2 * ((((uint64_t)par * NO + o) * NO + me) * p.CAPP + q), k, a, c, 0);
        } else {
          const uint32_t pos = atomicAdd(&p.cnt[((uint64_t)par * NO + o) * RW + NO], 1u);
          if (pos < p.OCAP) st256(p.ovf + 2 * (((uint64_t)par * NO + o) * p.OCAP + pos), k, a, c, 0);
          else atomicOr(p.flags, 2u);
        }
      }
      bar_named(1, PT);  // ring stage consumed, hist[par] final
      if (t == 0 && s + 2 < ST && !(p.mode & 4)) issue(s + 2);
      for (uint32_t o = t; o < NO; o += PT) {
        const uint32_t h = hp[o];
        p.cnt[((uint64_t)par * NO + o) * RW + me] = h < p.CAPP ? h : p.CAPP;
      }
      bar_arrive(3 + par, PT + 32);
      cwork += clock64() - c1;
    }
    if (t == 0) {
      atomicAdd(&p.stats[0], (unsigned long long)cw);
      atomicAdd(&p.stats[1], (unsigned long long)cwork);
    }
  } else if (w == p.NP) {  // producer signal warp
    for (uint32_t s = 0; s < ST; ++s) {
      bar_named(3 + s % NBUF, PT + 32);
      if (lane == 0) {
        __threadfence();
        atomicAdd(p.prod_done + s % M, 1u);
      }
    }
  } else if (w == p.NP + 1) {  // producer-ready poller
    if (lane == 0)
      for (uint32_t s = 0; s < ST; ++s) {
        wait_global(p.prod_done + s % M, NO * (s / M + 1));
        st_rel_cta(&ready[0], s + 1);
      }
  } else if (w == p.NP + 2) {  // consumer-done poller
    if (lane == 0)
      for (uint32_t s = 0; s < ST; ++s) {
        wait_global(p.cons_done + s % M, NO * (s / M + 1));
        st_rel_cta(&ready[1], s + 1);
      }
  } else if (w == p.NP + 3) {  // consumer signal warp
    for (uint32_t s = 0; s < ST; ++s) {
      bar_named(3 + NBUF + s % NBUF, CT + 32);
      if (lane == 0) {
        __threadfence();
        atomicAdd(p.cons_done + s % M, 1u);
      }
    }
  } else {
    // ------------------------------- consumers -------------------------------------------------
    const uint32_t t = threadIdx.x - (p.NP + 4) * 32, cw_ = t >> 5;
    for (uint32_t e = t; e < S; e += CT) {
      tkey[e] = kEmpty;
      tf[e] = 0.0;
      tcnt[e] = 0;
      tlo[e] = 0;
      thi[e] = 0;
    }
    Tbl T{tkey, tf, tcnt, tlo, thi, S >> 2};
    const uint32_t my_chunk = cw_ + p.CW * lane;
    const bool has_chunk = my_chunk < NO;
    bar_named(2, CT);
    long long cwt = 0, cwork = 0, cfl = 0;
    for (uint32_t s = 0; s < ST; ++s) {
      const uint32_t par = s % NBUF;
      const uint32_t b = bucket_of(s);
      long long c0 = clock64();
      wait_local(&ready[0], s + 1);
      long long c1 = clock64();
      cwt += c1 - c0;
      const uint32_t* row = p.cnt + ((uint64_t)par * NO + me) * RW;
      const uint32_t n_mine = has_chunk && !(p.mode & 4) ? ldcg32(row + my_chunk) : 0u;
      uint32_t inc = n_mine;
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
      if (cw_ == 0 && !(p.mode & 4)) {
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
        if (lane == 0 && novf) p.cnt[((uint64_t)par * NO + me) * RW + NO] = 0;
      }
      __syncwarp();
      bar_arrive(3 + NBUF + par, CT + 32);
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

int main(int argc, char** argv) {
  const uint64_t G = argc > 1 ? strtoull(argv[1], 0, 10) : 10000000ull;
  const uint64_t N = argc > 2 ? strtoull(argv[2], 0, 10) : 1000000000ull;
  const uint32_t B1 = argc > 3 ? atoi(argv[3]) : 32;
  const uint32_t cb = argc > 4 ? atoi(argv[4]) : 24;
  const uint32_t Tp = argc > 5 ? atoi(argv[5]) : 2048;
  const uint32_t S = argc > 6 ? atoi(argv[6]) : 4096;
  const uint32_t NP = argc > 7 ? atoi(argv[7]) : 4;
  const uint32_t CW = argc > 8 ? atoi(argv[8]) : 20;
  const uint32_t CAPP = argc > 9 ? atoi(argv[9]) : 32;
  const int NBUF = argc > 10 ? atoi(argv[10]) : 3;
  const uint32_t mode = argc > 11 ? atoi(argv[11]) : 0;
  const int reps = argc > 12 ? atoi(argv[12]) : 2;
  const uint32_t l2frac = argc > 13 ? atoi(argv[13]) : 0;
  int sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  const uint64_t cap = 1ull << cb, mask = cap - 1;
  uint32_t lb1 = 0;
  while ((1u << lb1) < B1) ++lb1;
  const uint32_t bshift = cb - lb1;
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
  uint64_t *d_key, *d_gk, *d_goff, *d_nrows;
  int64_t* d_v0;
  double* d_v1;
  CK(cudaMalloc(&d_key, seg_stride * B1 * 8 + 64));
  CK(cudaMalloc(&d_v0, seg_stride * B1 * 8 + 64));
  CK(cudaMalloc(&d_v1, seg_stride * B1 * 8 + 64));
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
  unsigned long long *chk, *stats;
  CK(cudaMalloc(&chk, 64));
  CK(cudaMalloc(&stats, 64));
  k_init<<<sms * 8, 256>>>(t2, cap);
  CK(cudaMemset(flags, 0, 64));
  k_naive<<<dim3(sms * 8, 4), 256>>>(d_key, d_v0, d_v1, d_nrows, B1, seg_stride, t2, mask, flags);
  CK(cudaDeviceSynchronize());
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
  p.CAPP = CAPP;
  p.OCAP = 4096;
  CK(cudaMalloc(&p.sub, (size_t)NBUF * sms * sms * CAPP * 32));
  CK(cudaMalloc(&p.cnt, (size_t)NBUF * sms * (sms + 4) * 4));
  CK(cudaMemset(p.cnt, 0, (size_t)NBUF * sms * (sms + 4) * 4));
  CK(cudaMalloc(&p.ovf, (size_t)NBUF * sms * p.OCAP * 32));
  uint32_t* ctr;
  CK(cudaMalloc(&ctr, 64 * 4));
  p.prod_done = ctr;
  p.cons_done = ctr + 16;
  p.stats = stats;
  p.Tp = Tp;
  p.S = S;
  p.NP = NP;
  p.CW = CW;
  p.flags = flags;
  p.mode = mode;
  p.l2frac = l2frac;
  const uint32_t block = (NP + 4 + CW) * 32;
  const size_t smem = (size_t)6 * Tp * 8 + (size_t)S * 28 + (B1 + 1) * 4 + (size_t)NBUF * sms * 4 + 16 + 64;
  printf("v3: G %llu rows %llu B1 %u Tp %u S %u NP %u CW %u CAPP %u NBUF %d block %u smem %zu sub %.1f MB mode %u l2frac %u\n",
         (unsigned long long)G, (unsigned long long)tot, B1, Tp, S, NP, CW, CAPP, NBUF, block, smem,
         (double)NBUF * sms * sms * CAPP * 32 / 1e6, mode, l2frac);
  if (smem > 232448 || block > 1024) {
    printf("v3: does not fit\n");
    return 1;
  }
  void* kern = NBUF == 3 ? (void*)k_route3<3> : NBUF == 4 ? (void*)k_route3<4> : NBUF == 5 ? (void*)k_route3<5> : (void*)k_route3<6>;
  CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  for (int rep = 0; rep < reps; ++rep) {
    k_init<<<sms * 8, 256>>>(t1, cap);
    CK(cudaMemset(ctr, 0, 64 * 4));
    CK(cudaMemset(stats, 0, 64));
    CK(cudaMemset(flags, 0, 64));
    void* args[] = {&p};
    cudaEventRecord(e0);
    CK(cudaLaunchCooperativeKernel(kern, dim3(sms), dim3(block), args, smem, 0));
    cudaEventRecord(e1);
    CK(cudaDeviceSynchronize());
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    uint32_t hf = 0;
    CK(cudaMemcpy(&hf, flags, 4, cudaMemcpyDeviceToHost));
    unsigned long long hs[8];
    CK(cudaMemcpy(hs, stats, 64, cudaMemcpyDeviceToHost));
    const double cyc = (double)sms * ms * 1.965e6;
    printf("route3: %.3f ms  %.1f G rows/s  flags %u | prod wait %.2f work %.2f | cons wait %.2f work %.2f flush %.2f\n", ms,
           tot / ms / 1e6, hf, hs[0] / cyc, hs[1] / cyc, hs[2] / cyc, hs[3] / cyc, hs[4] / cyc);
  }
  if (!(mode & 5)) {
    CK(cudaMemset(chk, 0, 64));
    k_check<<<sms * 8, 256>>>(t1, t2, cap, mask, chk);
    unsigned long long hc[4];
    CK(cudaMemcpy(hc, chk, 32, cudaMemcpyDeviceToHost));
    printf("check: groups %llu naive %llu mismatches %llu rows %llu (expect %llu) -> %s\n", hc[0], hc[1], hc[2], hc[3],
           (unsigned long long)tot, (hc[0] == hc[1] && hc[2] == 0 && hc[3] == tot) ? "OK" : "FAIL");
  }
  return 0;
}
