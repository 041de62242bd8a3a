// smagg_bench.cu — throughput of shared-memory hash-table aggregation (the inner loop of the
// partitioned path (b) pass 2): rows are synthesised in registers from a per-CTA key set (no memory
// traffic), so the kernel time is the table work alone. Variants:
//   v0  SoA table, 4-way bucketed probe (4 x LDS.64), atomics: COUNT u32, SUM i64 as 2 x u32 + carry,
//       SUM f64 CAS loop (the prototype's tbl_apply)
//   v1  as v0 with the probe as 2 x LDS.128
//   v2  warp-exclusive table partitions (entries of a warp's partition are touched only by that warp):
//       rows are redistributed through shared memory by owner warp, then plain read-modify-write with
//       __match_any_sync grouping of equal entries (no atomics)
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -lineinfo -o smagg_bench smagg_bench.cu
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

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
__device__ __forceinline__ uint32_t home4(uint64_t key, uint32_t nbk) {
  return (uint32_t)(((fmix64(key ^ 0x2545F4914F6CDD1Dull) >> 32) * (uint64_t)nbk) >> 32);
}
__device__ __forceinline__ void lds128v(const uint64_t* p, uint64_t& a, uint64_t& b) {
  asm volatile("ld.volatile.shared.v2.u64 {%0, %1}, [%2];" : "=l"(a), "=l"(b) : "r"((uint32_t)__cvta_generic_to_shared(p)));
}

// row j of CTA c: key = keyset(c, hash(j) % G), v0, v1 from the same hash
__device__ __forceinline__ void synth(uint32_t c, uint64_t j, uint32_t G, uint64_t& key, uint64_t& v0, double& v1) {
  const uint64_t u = fmix64(j * 0x9E3779B97F4A7C15ull + c);
  const uint64_t g = __umul64hi(u, G);
  key = fmix64(g + ((uint64_t)c << 32)) & ((1ull << 62) - 1);
  v0 = (u >> 20) - (1ull << 43);
  v1 = (double)((int64_t)(u & 0xFFFFF) - (1 << 19)) / 64.0;
}

template <int R, int VAR>
__global__ void __launch_bounds__(1024, 1) k_agg(uint64_t rows_per_cta, uint32_t G, uint32_t S, unsigned long long* out) {
  extern __shared__ __align__(16) uint8_t sm[];
  uint64_t* tkey = (uint64_t*)sm;
  double* tf = (double*)(tkey + S);
  uint32_t* tcnt = (uint32_t*)(tf + S);
  uint32_t* tlo = tcnt + S;
  uint32_t* thi = tlo + S;
  uint64_t* s64 = (uint64_t*)(thi + S);  // v2: S x (sum0) as u64 (exclusive RMW)
  for (uint32_t e = threadIdx.x; e < S; e += blockDim.x) {
    tkey[e] = kEmpty;
    tf[e] = 0.0;
    tcnt[e] = 0;
    tlo[e] = 0;
    thi[e] = 0;
    if (VAR == 2) s64[e] = 0;
  }
  __syncthreads();
  const uint32_t nbk = S >> 2;
  const uint32_t lane = threadIdx.x & 31;
  const uint64_t T = (uint64_t)blockDim.x * R;
  for (uint64_t j0 = 0; j0 < rows_per_cta; j0 += T) {
    uint64_t key[R], v0[R];
    double v1[R];
#pragma unroll
    for (int r = 0; r < R; ++r) synth(blockIdx.x, j0 + (uint64_t)r * blockDim.x + threadIdx.x, G, key[r], v0[r], v1[r]);
    uint32_t h[R], e[R];
#pragma unroll
    for (int r = 0; r < R; ++r) {
      h[r] = home4(key[r], nbk);
      e[r] = 0;
    }
    uint32_t pending = (1u << R) - 1, hit = 0;
    for (int it = 0; it < 32 && pending; ++it) {
#pragma unroll
      for (int r = 0; r < R; ++r) {
        if (!(pending >> r & 1)) continue;
        const uint64_t* q = tkey + 4 * h[r];
        uint64_t k0, k1, k2, k3;
        if (VAR == 0) {
          k0 = ((volatile const uint64_t*)q)[0];
          k1 = ((volatile const uint64_t*)q)[1];
          k2 = ((volatile const uint64_t*)q)[2];
          k3 = ((volatile const uint64_t*)q)[3];
        } else {
          lds128v(q, k0, k1);
          lds128v(q + 2, k2, k3);
        }
        const uint64_t kk = key[r];
        int m = k0 == kk ? 0 : k1 == kk ? 1 : k2 == kk ? 2 : k3 == kk ? 3 : -1;
        if (m < 0) {
          const int z = k0 == kEmpty ? 0 : k1 == kEmpty ? 1 : k2 == kEmpty ? 2 : k3 == kEmpty ? 3 : -1;
          if (z >= 0) {
            const unsigned long long old = atomicCAS((unsigned long long*)(q + z), kEmpty, (unsigned long long)kk);
            if (old == kEmpty || old == kk) m = z;
          } else {
            h[r] = h[r] + 1 == nbk ? 0u : h[r] + 1;
          }
        }
        if (m >= 0) {
          e[r] = 4 * h[r] + (uint32_t)m;
          pending &= ~(1u << r);
          hit |= 1u << r;
        }
      }
    }
    if (VAR <= 1) {
#pragma unroll
      for (int r = 0; r < R; ++r) {
        if (!(hit >> r & 1)) continue;
        const uint32_t x = e[r];
        atomicAdd(&tcnt[x], 1u);
        const uint32_t lo = (uint32_t)v0[r], hi = (uint32_t)(v0[r] >> 32);
        const uint32_t old = atomicAdd(&tlo[x], lo);
        const uint32_t carry = (old + lo) < old ? 1u : 0u;
        if (hi + carry) atomicAdd(&thi[x], hi + carry);
        atomicAdd(&tf[x], v1[r]);
      }
    } else {
      // warp-level grouping of equal entries, then ONE atomic per distinct entry and field, applied by
      // the group's leader with the group's combined values (combine in registers via shuffles)
#pragma unroll
      for (int r = 0; r < R; ++r) {
        const bool ok = hit >> r & 1;
        const uint32_t x = ok ? e[r] : 0xFFFFFFFFu;
        const uint32_t grp = __match_any_sync(0xffffffffu, x);
        const uint32_t leader = __ffs(grp) - 1;
        uint64_t s0 = v0[r];
        double s1 = v1[r];
        uint32_t c = 1;
        if (__any_sync(0xffffffffu, __popc(grp) > 1)) {  // rare: combine each group's values in its leader
          uint32_t rest = grp & ~(1u << leader);
          s0 = lane == leader ? v0[r] : 0;
          s1 = lane == leader ? v1[r] : 0.0;
          while (__any_sync(0xffffffffu, rest)) {
            const uint32_t src = rest ? __ffs(rest) - 1 : lane;
            const uint64_t a = __shfl_sync(0xffffffffu, v0[r], src);
            const double b = __shfl_sync(0xffffffffu, v1[r], src);
            if (rest && lane == leader) {
              s0 += a;
              s1 += b;
            }
            if (rest) rest &= rest - 1;
          }
          c = __popc(grp);
        }
        if (ok && lane == leader) {
          atomicAdd(&tcnt[x], c);
          atomicAdd((unsigned long long*)&s64[x], (unsigned long long)s0);
          atomicAdd(&tf[x], s1);
        }
      }
    }
  }
  __syncthreads();
  unsigned long long acc = 0;
  for (uint32_t e = threadIdx.x; e < S; e += blockDim.x) acc += tcnt[e];
  atomicAdd(out, acc);
}


// v3: warp-exclusive partitions (simulates rows already routed to their owner warp): warp w sees only
// keys of its own set, hashed into its own S/32-entry partition; equal keys in a warp are grouped with
// __match_any_sync, the group leader probes and applies the combined values with plain loads/stores.
// AoS entries of 32 B: key | sum0 | sum1 | count, pad.  MODE 1: synth only, MODE 2: synth + probe.
template <int R, int MODE>
__global__ void __launch_bounds__(1024, 1) k_agg3(uint64_t rows_per_cta, uint32_t G, uint32_t S, unsigned long long* out) {
  extern __shared__ __align__(16) uint8_t sm[];
  uint64_t* ent = (uint64_t*)sm;  // S x 4 words
  for (uint32_t e = threadIdx.x; e < S; e += blockDim.x) {
    ent[4 * e] = kEmpty;
    ent[4 * e + 1] = 0;
    ent[4 * e + 2] = 0;
    ent[4 * e + 3] = 0;
  }
  __syncthreads();
  const uint32_t lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
  const uint32_t P = S / nw;  // entries per warp partition (multiple of 4)
  uint64_t* pe = ent + 4ull * P * w;
  const uint32_t nbk = P >> 2;
  const uint32_t Gw = G / nw + 1;
  const uint64_t T = (uint64_t)blockDim.x * R;
  unsigned long long dummy = 0;
  for (uint64_t j0 = 0; j0 < rows_per_cta; j0 += T) {
#pragma unroll
    for (int r = 0; r < R; ++r) {
      uint64_t key, v0;
      double v1;
      synth(blockIdx.x * 64 + w, j0 + (uint64_t)r * blockDim.x + threadIdx.x, Gw, key, v0, v1);
      if (MODE == 1) {
        dummy += key ^ v0 ^ (uint64_t)__double_as_longlong(v1);
        continue;
      }
      const uint32_t grp = __match_any_sync(0xffffffffu, (uint32_t)key ^ (uint32_t)(key >> 32));
      const uint32_t leader = __ffs(grp) - 1;
      uint64_t s0 = v0;
      double s1 = v1;
      uint32_t c = 1;
      if (__any_sync(0xffffffffu, __popc(grp) > 1)) {
        uint32_t rest = grp & ~(1u << leader);
        while (__any_sync(0xffffffffu, rest)) {
          const uint32_t src = rest ? __ffs(rest) - 1 : lane;
          const uint64_t a = __shfl_sync(0xffffffffu, v0, src);
          const double b = __shfl_sync(0xffffffffu, v1, src);
          if (rest && lane == leader) {
            s0 += a;
            s1 += b;
          }
          if (rest) rest &= rest - 1;
        }
        c = __popc(grp);
      }
      if (lane != leader) continue;
      uint32_t h = home4(key, nbk);
      int e = -1;
      for (int it = 0; it < 32 && e < 0; ++it) {
        const uint64_t* q = pe + 16 * h;  // bucket = 4 entries x 4 words
        const uint64_t k0 = q[0], k1 = q[4], k2 = q[8], k3 = q[12];
        int m = k0 == key ? 0 : k1 == key ? 1 : k2 == key ? 2 : k3 == key ? 3 : -1;
        if (m < 0) {
          const int z = k0 == kEmpty ? 0 : k1 == kEmpty ? 1 : k2 == kEmpty ? 2 : k3 == kEmpty ? 3 : -1;
          if (z >= 0) {  // only this warp writes its partition; distinct keys of the warp may race here
            const unsigned long long old = atomicCAS((unsigned long long*)(q + 4 * z), kEmpty, (unsigned long long)key);
            if (old == kEmpty || old == key) m = z;
          } else {
            h = h + 1 == nbk ? 0u : h + 1;
          }
        }
        if (m >= 0) e = (int)(4 * h + m);
      }
      if (MODE == 2) {
        dummy += e;
        continue;
      }
      if (e >= 0) {
        uint64_t* x = pe + 4 * e;
        const uint64_t a = x[1];
        const double b = __longlong_as_double((long long)x[2]);
        const uint64_t cc = x[3];
        x[1] = a + s0;
        x[2] = (uint64_t)__double_as_longlong(b + s1);
        x[3] = cc + c;
      }
    }
  }
  __syncthreads();
  unsigned long long acc = dummy == 0x1234 ? 1 : 0;
  for (uint32_t e = threadIdx.x; e < S; e += blockDim.x) acc += ent[4 * e] != kEmpty ? ent[4 * e + 3] : 0;
  atomicAdd(out, acc);
}


// v4: atomic-free aggregation. Per tile of 1024 x R rows: warp-level multisplit of the rows by owner
// warp (32 table partitions by hash bits; match_any ranks, per-warp counters, one block scan; no
// atomics), rows staged in shared memory by owner, then every warp aggregates its own rows into its
// own partition: probe (2 x LDS.128 per 4-entry bucket), equal entries grouped with match_any and
// combined by shuffles, then plain loads/stores by the group leader. Only claiming an empty entry is
// an atomic (CAS: once per group per table lifetime).
template <int R>
__global__ void __launch_bounds__(1024, 1) k_agg4(uint64_t rows_per_cta, uint32_t G, uint32_t S, unsigned long long* out) {
  extern __shared__ __align__(16) uint8_t sm[];
  const uint32_t T = blockDim.x * R;  // rows per tile
  uint64_t* tkey = (uint64_t*)sm;     // S
  uint64_t* ts0 = tkey + S;           // S  (int64 sum, plain RMW)
  double* ts1 = (double*)(ts0 + S);   // S
  uint32_t* tcnt = (uint32_t*)(ts1 + S);  // S
  uint64_t* sk = (uint64_t*)(tcnt + S);   // T staged keys
  uint64_t* sa = sk + T;                  // T
  double* sc = (double*)(sa + T);         // T
  uint32_t* wcnt = (uint32_t*)(sc + T);   // [32 dest][32 warp]
  uint32_t* wtot = wcnt + 1024;           // 32 + 1
  for (uint32_t e = threadIdx.x; e < S; e += blockDim.x) {
    tkey[e] = kEmpty;
    ts0[e] = 0;
    ts1[e] = 0.0;
    tcnt[e] = 0;
  }
  const uint32_t lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const uint32_t P = S >> 5;   // entries per warp partition
  const uint32_t nbk = P >> 2;
  const uint32_t lt = (1u << lane) - 1;
  __syncthreads();
  for (uint64_t j0 = 0; j0 < rows_per_cta; j0 += T) {
    uint64_t key[R], v0[R];
    double v1[R];
    uint32_t d[R], rk[R];
    wcnt[threadIdx.x] = 0;  // blockDim == 1024 == 32 x 32 counters
    __syncthreads();
#pragma unroll
    for (int r = 0; r < R; ++r) {
      synth(blockIdx.x, j0 + (uint64_t)r * blockDim.x + threadIdx.x, G, key[r], v0[r], v1[r]);
      d[r] = (uint32_t)(fmix64(key[r] ^ 0x2545F4914F6CDD1Dull) >> 59);  // owner warp (top 5 hash bits)
      const uint32_t m = __match_any_sync(0xffffffffu, d[r]);
      const uint32_t before = wcnt[d[r] * 32 + w];  // this warp's count for d so far (only this warp writes it)
      rk[r] = before + __popc(m & lt);
      __syncwarp();
      if ((m & lt) == 0) wcnt[d[r] * 32 + w] = before + __popc(m);
      __syncwarp();
    }
    __syncthreads();
    {  // exclusive scan of the 1024 counters in (dest, warp) order: thread t holds element t
      const uint32_t x = wcnt[threadIdx.x];
      uint32_t inc = x;
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
        if ((int)lane >= o) inc += y;
      }
      if (lane == 31) wtot[w] = inc;
      __syncthreads();
      if (w == 0) {
        const uint32_t v = wtot[lane];
        uint32_t vi = v;
        for (int o = 1; o < 32; o <<= 1) {
          const uint32_t y = __shfl_up_sync(0xffffffffu, vi, o);
          if ((int)lane >= o) vi += y;
        }
        wtot[lane] = vi - v;  // exclusive prefix of dest block `lane` (dest-major: row = dest)
        if (lane == 31) wtot[32] = vi;
      }
      __syncthreads();
      wcnt[threadIdx.x] = wtot[w] + inc - x;  // element (dest = w_row, warp = lane) -> its offset
    }
    __syncthreads();
#pragma unroll
    for (int r = 0; r < R; ++r) {
      const uint32_t pos = wcnt[d[r] * 32 + w] + rk[r];
      sk[pos] = key[r];
      sa[pos] = v0[r];
      sc[pos] = v1[r];
    }
    __syncthreads();
    // warp w aggregates destination block w: rows [start, end)
    const uint32_t start = wcnt[w * 32], end = (w == 31) ? wtot[32] : wcnt[(w + 1) * 32];
    uint64_t* pk = tkey + (size_t)P * w;
    for (uint32_t i0 = start; i0 < end; i0 += 32) {
      const uint32_t i = i0 + lane;
      const bool ok = i < end;
      const uint64_t kk = ok ? sk[i] : kEmpty;
      const uint64_t a = ok ? sa[i] : 0;
      const double c = ok ? sc[i] : 0.0;
      uint32_t h = ok ? (uint32_t)(((fmix64(kk ^ 0x2545F4914F6CDD1Dull) >> 27 & 0xFFFFFFFFull) * nbk) >> 32) : 0u;
      int e = -1;
      bool pend = ok;
      for (int it = 0; it < 32 && __any_sync(0xffffffffu, pend); ++it) {
        if (pend) {
          const uint64_t* q = pk + 4 * h;
          uint64_t k0, k1, k2, k3;
          lds128v(q, k0, k1);
          lds128v(q + 2, k2, k3);
          int m = k0 == kk ? 0 : k1 == kk ? 1 : k2 == kk ? 2 : k3 == kk ? 3 : -1;
          if (m < 0) {
            const int z = k0 == kEmpty ? 0 : k1 == kEmpty ? 1 : k2 == kEmpty ? 2 : k3 == kEmpty ? 3 : -1;
            if (z >= 0) {
              const unsigned long long old = atomicCAS((unsigned long long*)(q + z), kEmpty, (unsigned long long)kk);
              if (old == kEmpty || old == kk) m = z;
            } else {
              h = h + 1 == nbk ? 0u : h + 1;
            }
          }
          if (m >= 0) {
            e = (int)(4 * h + m);
            pend = false;
          }
        }
      }
      // group equal entries, combine in the leader, plain read-modify-write
      const uint32_t g = __match_any_sync(0xffffffffu, (uint32_t)e);
      const uint32_t leader = __ffs(g) - 1;
      uint64_t s0 = a;
      double s1 = c;
      if (__any_sync(0xffffffffu, __popc(g) > 1)) {
        uint32_t rest = g & ~(1u << leader);
        s0 = lane == leader ? a : 0;
        s1 = lane == leader ? c : 0.0;
        while (__any_sync(0xffffffffu, rest)) {
          const uint32_t src = rest ? __ffs(rest) - 1 : lane;
          const uint64_t x = __shfl_sync(0xffffffffu, a, src);
          const double y = __shfl_sync(0xffffffffu, c, src);
          if (rest && lane == leader) {
            s0 += x;
            s1 += y;
          }
          if (rest) rest &= rest - 1;
        }
      }
      if (e >= 0 && lane == leader) {
        const uint32_t x = P * w + (uint32_t)e;
        ts0[x] += s0;
        ts1[x] += s1;
        tcnt[x] += __popc(g);
      }
    }
    __syncthreads();
  }
  __syncthreads();
  unsigned long long acc = 0;
  for (uint32_t e = threadIdx.x; e < S; e += blockDim.x) acc += tcnt[e];
  atomicAdd(out, acc);
}

int main(int argc, char** argv) {
  const uint64_t rows = argc > 1 ? strtoull(argv[1], 0, 10) : 1000000000ull;
  const uint32_t G = argc > 2 ? atoi(argv[2]) : 2111;
  const uint32_t S = argc > 3 ? atoi(argv[3]) : 4096;
  const int block = argc > 4 ? atoi(argv[4]) : 1024;
  int sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  unsigned long long* out;
  CK(cudaMalloc(&out, 8));
  const uint64_t per = rows / sms / (block * 4) * (block * 4);
  const size_t smem = (size_t)S * (8 + 8 + 4 + 4 + 4 + 8) + (size_t)1024 * 2 * 24 + 4096 + 256;
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  auto run = [&](auto kern, const char* name) {
    CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    for (int rep = 0; rep < 2; ++rep) {
      CK(cudaMemset(out, 0, 8));
      cudaEventRecord(e0);
      kern<<<sms, block, smem>>>(per, G, S, out);
      cudaEventRecord(e1);
      CK(cudaDeviceSynchronize());
      float ms = 0;
      cudaEventElapsedTime(&ms, e0, e1);
      unsigned long long h = 0;
      CK(cudaMemcpy(&h, out, 8, cudaMemcpyDeviceToHost));
      const double tot = (double)per * sms;
      printf("%-28s G %u S %u block %d: %.3f ms  %.1f G rows/s  %.3f rows/clk/SM  (count %llu / %.0f)\n", name, G, S, block,
             ms, tot / ms / 1e6, tot / (ms * 1e-3 * 1.965e9 * sms), h, tot);
    }
  };
  run(k_agg<4, 0>, "v0 atomics, 4xLDS.64 probe");
  run(k_agg<4, 1>, "v1 atomics, 2xLDS.128 probe");
  run(k_agg<4, 2>, "v2 match_any + 3 atomics");
  run(k_agg<2, 1>, "v1 R=2");
  run(k_agg4<2>, "v4 multisplit, no atomics R=2");

  return 0;
}
