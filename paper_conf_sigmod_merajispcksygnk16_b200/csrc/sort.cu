// sort.cu — libblugby's sort offload (§3; include/blu_sort.h).
//
//   k_rs_upsweep / k_rs_scan / k_rs_downsweep   one pass of a stable LSD radix sort (8-bit digit):
//       every CTA owns one contiguous range of tiles; the upsweep counts its digits, one CTA scans
//       the digit-major count matrix into output offsets, the downsweep ranks each tile's keys with
//       warp matching (__match_any_sync: lanes with equal digits, the lowest one bumps a per-warp
//       counter) and scatters them after all earlier CTAs' and tiles' keys of the same digit —
//       stable, no global atomics. Used for the partial key buffer (u32 keys, "Duane sort"
//       [18]) and for the batched duplicate-range jobs (u64 keys = range id << 32 | partial key).
//   k_partial_keys        P:78 4-byte big-endian partial key of one word of every row
//   k_dup_mark / k_dup_count / k_dup_emit   P:84 duplicate ranges: run boundaries, block counts,
//       one-CTA scan, compaction into (start, len) or into the next level's active set
//   k_level_keys / k_level_scatter           one batched level of the job queue
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <string.h>
#include <time.h>

#include <algorithm>
#include <vector>

#include "blu_internal.h"
#include "blu_sort.h"

namespace blu {

namespace {

constexpr int kRT = 256;  // threads per radix CTA (= number of digits: thread d owns digit d)

template <typename KT>
struct RadixCfg {
  static constexpr int ITEMS = 8;                          // keys per thread per tile
  static constexpr int WARP_CHUNK = 32 * ITEMS;           // contiguous keys per warp
  static constexpr int TILE = kRT * ITEMS;
};

__device__ __forceinline__ void tile_span(uint64_t ntiles, uint64_t& t0, uint64_t& t1) {
  t0 = ntiles * blockIdx.x / gridDim.x;
  t1 = ntiles * (blockIdx.x + 1) / gridDim.x;
}

template <typename KT>
__device__ __forceinline__ uint32_t digit_of(KT k, uint32_t shift) {
  return (uint32_t)(k >> shift) & 255u;
}

template <typename KT>
__global__ void __launch_bounds__(kRT) k_rs_upsweep(const KT* __restrict__ keys, uint64_t n, uint32_t shift,
                                                    uint32_t* __restrict__ counts) {
  using C = RadixCfg<KT>;
  __shared__ uint32_t h[256];
  h[threadIdx.x] = 0;
  __syncthreads();
  const unsigned lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint64_t t0, t1;
  tile_span((n + C::TILE - 1) / C::TILE, t0, t1);
  for (uint64_t t = t0; t < t1; ++t) {
    const uint64_t b = t * C::TILE + (uint64_t)warp * C::WARP_CHUNK + lane;
#pragma unroll
    for (int i = 0; i < C::ITEMS; ++i) {
      const uint64_t e = b + (uint64_t)i * 32;
      const bool valid = e < n;
      const uint32_t d = valid ? digit_of(keys[e], shift) : 256u + lane;
      const uint32_t peers = __match_any_sync(0xffffffffu, d);
      if (valid && lane == (unsigned)(__ffs(peers) - 1)) atomicAdd(&h[d], (uint32_t)__popc(peers));
    }
  }
  __syncthreads();
  counts[(uint64_t)threadIdx.x * gridDim.x + blockIdx.x] = h[threadIdx.x];
}

// Exclusive scan, in place, of a[0..L) (one CTA of 1024 threads, contiguous chunk per thread).
__global__ void __launch_bounds__(1024) k_rs_scan(uint32_t* a, uint64_t L) {
  __shared__ uint32_t ws[32];
  const uint64_t per = (L + blockDim.x - 1) / blockDim.x;
  const uint64_t b = per * threadIdx.x, e = b + per < L ? b + per : L;
  uint32_t s = 0;
  for (uint64_t i = b; i < e; ++i) s += a[i];
  const unsigned lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  uint32_t inc = s;
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
    if ((int)lane >= o) inc += y;
  }
  if (lane == 31) ws[w] = inc;
  __syncthreads();
  if (w == 0) {
    const uint32_t v = ws[lane];
    uint32_t vi = v;
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, vi, o);
      if ((int)lane >= o) vi += y;
    }
    ws[lane] = vi - v;
  }
  __syncthreads();
  uint32_t run = ws[w] + inc - s;
  for (uint64_t i = b; i < e; ++i) {
    const uint32_t x = a[i];
    a[i] = run;
    run += x;
  }
}

// Exclusive scan of each digit's row of the count matrix (CTA d scans counts[d][0..G), coalesced,
// 256 at a time); the row total goes to digit_tot[d]. The downsweep adds the digit bases itself.
__global__ void __launch_bounds__(kRT) k_rs_scan_rows(uint32_t* __restrict__ counts, uint32_t G,
                                                      uint32_t* __restrict__ digit_tot) {
  __shared__ uint32_t ws[kRT / 32];
  uint32_t* row = counts + (uint64_t)blockIdx.x * G;
  const unsigned lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  uint32_t carry = 0;
  for (uint32_t c0 = 0; c0 < G; c0 += kRT) {
    const uint32_t c = c0 + threadIdx.x;
    const uint32_t x = c < G ? row[c] : 0u;
    uint32_t inc = x;
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
      if ((int)lane >= o) inc += y;
    }
    if (lane == 31) ws[w] = inc;
    __syncthreads();
    uint32_t before = 0, tot = 0;
    for (unsigned q = 0; q < kRT / 32; ++q) {
      if (q < w) before += ws[q];
      tot += ws[q];
    }
    if (c < G) row[c] = carry + before + inc - x;
    carry += tot;
    __syncthreads();
  }
  if (threadIdx.x == 0) digit_tot[blockIdx.x] = carry;
}

template <typename KT>
__global__ void __launch_bounds__(kRT, 4) k_rs_downsweep(const KT* __restrict__ kin, const uint32_t* __restrict__ vin,
                                                      KT* __restrict__ kout, uint32_t* __restrict__ vout, uint64_t n,
                                                      uint32_t shift, const uint32_t* __restrict__ offsets,
                                                      const uint32_t* __restrict__ digit_tot) {
  using C = RadixCfg<KT>;
  __shared__ uint32_t base[256];
  __shared__ uint32_t ttot[256];
  __shared__ uint32_t tstart[256];
  __shared__ uint32_t wsum[kRT / 32];
  __shared__ uint32_t wcnt[kRT / 32][256];
  __shared__ KT sk[C::TILE];
  __shared__ uint32_t sv[C::TILE];
  const unsigned lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint32_t lt_mask = (1u << lane) - 1u;
  {  // digit bases: exclusive scan of the 256 digit totals (thread d owns digit d)
    const uint32_t x = digit_tot[threadIdx.x];
    uint32_t inc = x;
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
      if ((int)lane >= o) inc += y;
    }
    if (lane == 31) ttot[warp] = inc;
    __syncthreads();
    uint32_t before = 0;
    for (unsigned q = 0; q < warp; ++q) before += ttot[q];
    base[threadIdx.x] = before + inc - x + offsets[(uint64_t)threadIdx.x * gridDim.x + blockIdx.x];
    __syncthreads();
  }
  uint64_t t0, t1;
  tile_span((n + C::TILE - 1) / C::TILE, t0, t1);
  // warp-striped tile: warp w owns keys [w * WARP_CHUNK, +WARP_CHUNK); item i of lane l is key
  // i * 32 + l of that chunk, so (warp, i, lane) order is input order (stability)
  KT k[C::ITEMS];
  uint32_t v[C::ITEMS], rank[C::ITEMS];
  auto load_tile = [&](uint64_t tt) {
    const uint64_t bb = tt * C::TILE + (uint64_t)warp * C::WARP_CHUNK + lane;
#pragma unroll
    for (int i = 0; i < C::ITEMS; ++i) {
      const uint64_t e = bb + (uint64_t)i * 32;
      k[i] = e < n ? kin[e] : (KT)0;
      v[i] = e < n ? vin[e] : 0u;
    }
  };
  if (t0 < t1) load_tile(t0);
  for (uint64_t t = t0; t < t1; ++t) {
#pragma unroll
    for (int w = 0; w < kRT / 32; ++w) wcnt[w][threadIdx.x] = 0;
    __syncthreads();
    const uint64_t b = t * C::TILE + (uint64_t)warp * C::WARP_CHUNK + lane;
#pragma unroll
    for (int i = 0; i < C::ITEMS; ++i) {
      const bool valid = b + (uint64_t)i * 32 < n;
      const uint32_t d = valid ? digit_of(k[i], shift) : 256u + lane;
      const uint32_t peers = __match_any_sync(0xffffffffu, d);
      const int leader = __ffs(peers) - 1;
      uint32_t c = 0;
      if (valid && (int)lane == leader) {
        c = wcnt[warp][d];
        wcnt[warp][d] = c + (uint32_t)__popc(peers);
      }
      c = __shfl_sync(0xffffffffu, c, leader);
      rank[i] = c + (uint32_t)__popc(peers & lt_mask);
      __syncwarp();
    }
    __syncthreads();
    uint32_t tot_d;
    {  // per digit: exclusive prefix over the warps, tile total
      uint32_t run = 0;
#pragma unroll
      for (int w = 0; w < kRT / 32; ++w) {
        const uint32_t x = wcnt[w][threadIdx.x];
        wcnt[w][threadIdx.x] = run;
        run += x;
      }
      tot_d = run;
    }
    {  // tile-local start of each digit: exclusive scan of the tile totals over the 256 digits
      uint32_t inc = tot_d;
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
        if ((int)lane >= o) inc += y;
      }
      if (lane == 31) wsum[warp] = inc;
      __syncthreads();
      uint32_t before = 0;
      for (unsigned q = 0; q < warp; ++q) before += wsum[q];
      tstart[threadIdx.x] = before + inc - tot_d;
      ttot[threadIdx.x] = tot_d;
    }
    __syncthreads();
    // stage the tile in digit order in shared memory ...
#pragma unroll
    for (int i = 0; i < C::ITEMS; ++i) {
      if (b + (uint64_t)i * 32 >= n) continue;
      const uint32_t d = digit_of(k[i], shift);
      const uint32_t lp = tstart[d] + wcnt[warp][d] + rank[i];
      sk[lp] = k[i];
      sv[lp] = v[i];
    }
    // the tile is staged: the next one's loads go out now and are in flight during the write-out
    if (t + 1 < t1) load_tile(t + 1);
    __syncthreads();
    // ... then write it out: consecutive threads write consecutive addresses of each digit's run
    const uint64_t tile0 = t * C::TILE;
    const uint32_t cnt = (uint32_t)(n - tile0 < (uint64_t)C::TILE ? n - tile0 : (uint64_t)C::TILE);
    for (uint32_t e = threadIdx.x; e < cnt; e += kRT) {
      const KT key = sk[e];
      const uint32_t d = digit_of(key, shift);
      const uint32_t pos = base[d] + (e - tstart[d]);
      kout[pos] = key;
      vout[pos] = sv[e];
    }
    __syncthreads();
    base[threadIdx.x] += ttot[threadIdx.x];
  }
}

// OR and AND of all keys: a digit whose 8 bits agree in both is the same for every key, and its
// LSD pass is the identity permutation (skipped).
template <typename KT>
__global__ void k_key_bits(const KT* __restrict__ keys, uint64_t n, unsigned long long* __restrict__ or_and) {
  unsigned long long o = 0, a = ~0ull;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    const unsigned long long k = (unsigned long long)keys[i];
    o |= k;
    a &= k;
  }
  for (int s = 16; s; s >>= 1) {
    o |= __shfl_xor_sync(0xffffffffu, o, s);
    a &= __shfl_xor_sync(0xffffffffu, a, s);
  }
  if ((threadIdx.x & 31) == 0) {
    atomicOr(or_and, o);
    atomicAnd(or_and + 1, a);
  }
}

// big-endian 4-byte partial key of word `word` (bytes past W read as 0); payload = row index.
template <typename KT>
__global__ void k_partial_keys(const uint8_t* __restrict__ rows, uint64_t n, uint32_t W, uint32_t word,
                               KT* __restrict__ keys, uint32_t* __restrict__ payload) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t p = 4 * word;
    uint32_t k;
    if (p + 4 <= W && (W & 3) == 0 && ((uintptr_t)rows & 3) == 0) {
      k = __byte_perm(__ldg((const unsigned int*)(rows + i * W + p)), 0, 0x0123);  // bswap
    } else {
      k = 0;
      for (uint32_t q = 0; q < 4; ++q) k = (k << 8) | (p + q < W ? rows[i * W + p + q] : 0u);
    }
    keys[i] = (KT)k;
    if (payload) payload[i] = (uint32_t)i;
  }
}

// ---- duplicate ranges: marks -> block counts -> scan -> emit ---------------------------------------
constexpr int kDT = 256, kDR = 16;  // threads, elements per thread (4096 per block)
constexpr uint64_t kDB = (uint64_t)kDT * kDR;

template <typename KT>
__device__ __forceinline__ void dup_flags(const KT* k, uint64_t m, uint64_t j, bool& act, bool& start, bool& end) {
  const bool sp = j > 0 && k[j] == k[j - 1];
  const bool sn = j + 1 < m && k[j] == k[j + 1];
  act = sp || sn;
  start = act && !sp;
  end = act && !sn;
}

// per block: number of active elements (in a duplicate range) and of range starts
template <typename KT>
__global__ void __launch_bounds__(kDT) k_dup_count(const KT* __restrict__ k, uint64_t m, uint32_t* __restrict__ cnt_act,
                                                   uint32_t* __restrict__ cnt_start) {
  uint32_t a = 0, s = 0;
  for (int r = 0; r < kDR; ++r) {
    const uint64_t j = (uint64_t)blockIdx.x * kDB + (uint64_t)r * kDT + threadIdx.x;
    if (j >= m) break;
    bool act, st, en;
    dup_flags(k, m, j, act, st, en);
    a += act;
    s += st;
  }
  __shared__ uint32_t wa[kDT / 32], wsum[kDT / 32];
  for (int o = 16; o; o >>= 1) {
    a += __shfl_xor_sync(0xffffffffu, a, o);
    s += __shfl_xor_sync(0xffffffffu, s, o);
  }
  if ((threadIdx.x & 31) == 0) {
    wa[threadIdx.x >> 5] = a;
    wsum[threadIdx.x >> 5] = s;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    uint32_t ta = 0, ts = 0;
    for (int w = 0; w < kDT / 32; ++w) {
      ta += wa[w];
      ts += wsum[w];
    }
    cnt_act[blockIdx.x] = ta;
    cnt_start[blockIdx.x] = ts;
  }
}

// Emit, in order, per active element j: its position act_pos (the caller's position list, or j
// itself if NULL) into next_pos and its range id (0-based, in order) into next_seg; per range its
// start and its end (exclusive; k_range_lens turns it into a length) into r_start / r_len (if
// non-NULL, ids < cap).
template <typename KT>
__global__ void __launch_bounds__(kDT) k_dup_emit(const KT* __restrict__ k, uint64_t m, const uint32_t* __restrict__ off_act,
                                                  const uint32_t* __restrict__ off_start, const uint32_t* __restrict__ act_pos,
                                                  uint32_t* __restrict__ next_pos, uint32_t* __restrict__ next_seg,
                                                  uint64_t* __restrict__ r_start, uint64_t* __restrict__ r_len, uint64_t cap) {
  __shared__ uint32_t wa[kDT / 32], wsum[kDT / 32];
  uint32_t base_a = off_act[blockIdx.x], base_s = off_start[blockIdx.x];
  const unsigned lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  for (int r = 0; r < kDR; ++r) {
    const uint64_t j = (uint64_t)blockIdx.x * kDB + (uint64_t)r * kDT + threadIdx.x;
    bool act = false, st = false, en = false;
    if (j < m) dup_flags(k, m, j, act, st, en);
    const uint32_t ba = __ballot_sync(0xffffffffu, act), bs = __ballot_sync(0xffffffffu, st);
    if (lane == 0) {
      wa[w] = __popc(ba);
      wsum[w] = __popc(bs);
    }
    __syncthreads();
    uint32_t pa = 0, ps = 0, ta = 0, ts = 0;
    for (unsigned q = 0; q < kDT / 32; ++q) {
      if (q < w) {
        pa += wa[q];
        ps += wsum[q];
      }
      ta += wa[q];
      ts += wsum[q];
    }
    pa += __popc(ba & ((1u << lane) - 1u));
    ps += __popc(bs & ((1u << lane) - 1u));
    const uint32_t ia = base_a + pa;                      // index among active elements
    const uint32_t seg = base_s + ps + (st ? 1u : 0u) - 1u;  // range id (inclusive count - 1)
    if (act) {
      if (next_pos) next_pos[ia] = act_pos ? act_pos[j] : (uint32_t)j;
      if (next_seg) next_seg[ia] = seg;
    }
    if (r_start && seg < cap) {
      if (st) r_start[seg] = j;
      if (en) r_len[seg] = j + 1;
    }
    __syncthreads();
    base_a += ta;
    base_s += ts;
  }
}

__global__ void k_range_lens(const uint64_t* __restrict__ r_start, uint64_t* __restrict__ r_len, uint64_t cnt) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < cnt; i += (uint64_t)gridDim.x * blockDim.x)
    r_len[i] -= r_start[i];
}

// One batched level: key = (range id << 32) | partial key `word` of the row at buffer position
// pos[j]; payload = that row id.
// The row reads are random 4-byte gathers: each thread keeps 4 of them in flight (elements j,
// j + stride, j + 2 stride, j + 3 stride) instead of one.
__global__ void k_level_keys(const uint8_t* __restrict__ rows, uint32_t W, uint32_t word, const uint32_t* __restrict__ pos,
                             const uint32_t* __restrict__ seg, const uint32_t* __restrict__ perm, uint64_t m,
                             uint64_t* __restrict__ keys, uint32_t* __restrict__ payload) {
  const uint32_t p = 4 * word;
  const bool aligned = (W & 3) == 0 && p + 4 <= W && ((uintptr_t)rows & 3) == 0;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t j0 = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; j0 < m; j0 += 4 * stride) {
    uint32_t row[4], k[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const uint64_t j = j0 + u * stride;
      row[u] = j < m ? __ldg(perm + __ldg(pos + j)) : 0u;
    }
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const uint64_t j = j0 + u * stride;
      k[u] = 0;
      if (j >= m) continue;
      if (aligned) {
        k[u] = __ldg((const unsigned int*)(rows + (uint64_t)row[u] * W + p));
      } else {
        for (uint32_t q = 0; q < 4; ++q) k[u] = (k[u] << 8) | (p + q < W ? rows[(uint64_t)row[u] * W + p + q] : 0u);
        k[u] = __byte_perm(k[u], 0, 0x0123);  // undone below: both branches yield big-endian order
      }
    }
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const uint64_t j = j0 + u * stride;
      if (j >= m) continue;
      keys[j] = ((uint64_t)__ldg(seg + j) << 32) | __byte_perm(k[u], 0, 0x0123);
      payload[j] = row[u];
    }
  }
}

// Sorted level results back into the positions its ranges occupy (same ranges, same order).
__global__ void k_level_scatter(const uint32_t* __restrict__ pos, const uint32_t* __restrict__ rows_sorted, uint64_t m,
                                uint32_t* __restrict__ perm) {
  for (uint64_t j = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; j < m; j += (uint64_t)gridDim.x * blockDim.x)
    perm[pos[j]] = rows_sorted[j];
}

// ---- segmented window sort (levels >= 1 whose duplicate ranges are all short) -------------------
// The level's active list holds its ranges contiguously with consecutive range ids (seg), so sorting
// the batched (seg << 32 | key) array only has to order elements WITHIN each range. When no range is
// longer than kSW / 2, two passes of in-shared-memory sorts over fixed windows do it: windows
// [w*kSW, (w+1)*kSW), then windows shifted by kSW / 2. A range inside a first-pass window is sorted
// by it; a range across a first-pass boundary lies inside one shifted window (length <= kSW / 2),
// and a shifted window re-sorting already sorted parts leaves them in place. Each window is a stable
// LSD radix sort in shared memory on (seg - first seg in window, key): 12 + 32 bits, 8-bit digits,
// digits that are constant across the window skipped. Replaces the 6-7 global radix passes of such
// a level (S1 level 2: ~915K ranges of ~109 rows) by two reads and writes of the level's keys.
// Window size kSW elements, kST = kSW / 4 threads (4 elements each); 2048-element windows fit three
// CTAs per SM, 4096-element windows one (BLU_SORT_SEG_W).
template <int kSW>
constexpr size_t seg_smem() { return (size_t)kSW * (8 + 8 + 4 + 4) + (kSW / 128) * 256 * 4 + 2 * 256 * 4 + 64; }

template <int kSW>
__global__ void __launch_bounds__(kSW / 4) k_seg_window_sort(uint64_t* __restrict__ keys, uint32_t* __restrict__ rows,
                                                             uint64_t m, uint64_t off) {
  constexpr int kST = kSW / 4, kNW = kST / 32;
  extern __shared__ __align__(16) uint8_t smraw[];
  uint64_t* ka = (uint64_t*)smraw;
  uint64_t* kb = ka + kSW;
  uint32_t* ra = (uint32_t*)(kb + kSW);
  uint32_t* rb = ra + kSW;
  uint32_t (*wcnt)[256] = (uint32_t(*)[256])(rb + kSW);
  uint32_t* tot = (uint32_t*)(wcnt + kNW);
  uint32_t* dstart = tot + 256;
  uint32_t* misc = dstart + 256;  // [0] OR lo, [1] OR hi, [2] AND lo, [3] AND hi, [4..11] warp sums
  const unsigned tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint32_t lt_mask = (1u << lane) - 1u;
  for (uint64_t b0 = off + (uint64_t)blockIdx.x * kSW; b0 < m; b0 += (uint64_t)gridDim.x * kSW) {
    const uint32_t cnt = (uint32_t)(m - b0 < (uint64_t)kSW ? m - b0 : (uint64_t)kSW);
    const uint32_t seg0 = (uint32_t)(keys[b0] >> 32);
    if (tid == 0) {
      misc[0] = misc[1] = 0u;
      misc[2] = misc[3] = ~0u;
    }
    __syncthreads();
    uint32_t o0 = 0, o1 = 0, a0 = ~0u, a1 = ~0u;
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const uint32_t e = warp * 128 + i * 32 + lane;
      if (e < cnt) {
        const uint64_t k = keys[b0 + e];
        const uint64_t lk = ((uint64_t)((uint32_t)(k >> 32) - seg0) << 32) | (k & 0xFFFFFFFFull);
        ka[e] = lk;
        ra[e] = rows[b0 + e];
        o0 |= (uint32_t)lk, o1 |= (uint32_t)(lk >> 32), a0 &= (uint32_t)lk, a1 &= (uint32_t)(lk >> 32);
      }
    }
    o0 = __reduce_or_sync(0xffffffffu, o0), o1 = __reduce_or_sync(0xffffffffu, o1);
    a0 = __reduce_and_sync(0xffffffffu, a0), a1 = __reduce_and_sync(0xffffffffu, a1);
    if (lane == 0) {
      atomicOr(&misc[0], o0), atomicOr(&misc[1], o1);
      atomicAnd(&misc[2], a0), atomicAnd(&misc[3], a1);
    }
    __syncthreads();
    const uint64_t vary = ((uint64_t)(misc[1] ^ misc[3]) << 32) | (misc[0] ^ misc[2]);
    uint64_t* ks = ka;
    uint64_t* kd = kb;
    uint32_t* rs = ra;
    uint32_t* rd = rb;
    for (uint32_t shift = 0; shift < 48; shift += 8) {
      if (((vary >> shift) & 255ull) == 0) continue;  // constant digit: the pass is the identity
#pragma unroll
      for (int q = 0; q < 8; ++q) wcnt[warp][q * 32 + lane] = 0u;
      __syncthreads();
      uint32_t dg[4], rk[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const uint32_t e = warp * 128 + i * 32 + lane;
        const bool valid = e < cnt;
        const uint32_t d = valid ? (uint32_t)(ks[e] >> shift) & 255u : 256u + lane;
        const uint32_t peers = __match_any_sync(0xffffffffu, d);
        const int leader = __ffs(peers) - 1;
        uint32_t c = 0;
        if (valid && (int)lane == leader) {
          c = wcnt[warp][d];
          wcnt[warp][d] = c + (uint32_t)__popc(peers);
        }
        c = __shfl_sync(0xffffffffu, c, leader);
        dg[i] = d;
        rk[i] = c + (uint32_t)__popc(peers & lt_mask);
        __syncwarp();
      }
      __syncthreads();
      if (tid < 256) {  // per digit: exclusive prefix over the warps, and the digit total
        uint32_t run = 0;
        for (int w = 0; w < kNW; ++w) {
          const uint32_t x = wcnt[w][tid];
          wcnt[w][tid] = run;
          run += x;
        }
        uint32_t inc = run;  // exclusive scan of the 256 digit totals (8 warps)
        for (int o = 1; o < 32; o <<= 1) {
          const uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
          if ((int)lane >= o) inc += y;
        }
        if (lane == 31) misc[4 + warp] = inc;
        tot[tid] = inc - run;
      }
      __syncthreads();
      if (tid < 256) {
        uint32_t before = 0;
        for (unsigned q = 0; q < warp; ++q) before += misc[4 + q];
        dstart[tid] = before + tot[tid];
      }
      __syncthreads();
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const uint32_t e = warp * 128 + i * 32 + lane;
        if (e < cnt) {
          const uint32_t pos = dstart[dg[i]] + wcnt[warp][dg[i]] + rk[i];
          kd[pos] = ks[e];
          rd[pos] = rs[e];
        }
      }
      __syncthreads();
      uint64_t* tk = ks; ks = kd; kd = tk;
      uint32_t* tr = rs; rs = rd; rd = tr;
    }
    for (uint32_t e = tid; e < cnt; e += kST) {
      const uint64_t lk = ks[e];
      keys[b0 + e] = ((uint64_t)((uint32_t)(lk >> 32) + seg0) << 32) | (lk & 0xFFFFFFFFull);
      rows[b0 + e] = rs[e];
    }
    __syncthreads();
  }
}

// ---- warp-per-range sort (levels whose ranges are all <= 256 rows) -------------------------------
// One warp sorts one range in registers with a bitonic network over (key << 32 | index in range):
// the index makes every element distinct, so the order is the stable one. N = 32 R elements,
// element i = r * 32 + lane in register r; partners at distance >= 32 are in the same lane
// (registers r, r ^ j/32), closer ones in lane ^ j (shuffle). Rows follow their index after the sort.
template <int R>
__device__ __forceinline__ void warp_range_sort(uint64_t* __restrict__ keys, uint32_t* __restrict__ rows,
                                                uint32_t start, uint32_t len, unsigned lane) {
  constexpr int N = 32 * R;
  uint64_t v[R];
  const uint32_t seg = (uint32_t)(keys[start] >> 32);
#pragma unroll
  for (int r = 0; r < R; ++r) {
    const uint32_t i = r * 32 + lane;
    v[r] = i < len ? (keys[start + i] << 32) | i : ~0ull;
  }
#pragma unroll
  for (int k = 2; k <= N; k <<= 1) {
#pragma unroll
    for (int j = k >> 1; j > 0; j >>= 1) {
      if (j >= 32) {
        const int jr = j / 32;
#pragma unroll
        for (int r = 0; r < R; ++r) {
          if (r & jr) continue;
          const uint32_t i = r * 32 + lane;
          const bool up = (i & k) == 0;
          const uint64_t a = v[r], b = v[r + jr];
          if ((a > b) == up) {
            v[r] = b;
            v[r + jr] = a;
          }
        }
      } else {
#pragma unroll
        for (int r = 0; r < R; ++r) {
          const uint32_t i = r * 32 + lane;
          const uint64_t o = __shfl_xor_sync(0xffffffffu, v[r], j);
          const bool up = (i & k) == 0, low = (lane & j) == 0;
          v[r] = (low == up) ? (v[r] < o ? v[r] : o) : (v[r] > o ? v[r] : o);
        }
      }
    }
  }
  uint32_t rr[R];
#pragma unroll
  for (int r = 0; r < R; ++r) {
    const uint32_t i = r * 32 + lane;
    rr[r] = i < len ? rows[start + (uint32_t)(v[r] & 0xFFFFFFFFull)] : 0u;
  }
  __syncwarp();
#pragma unroll
  for (int r = 0; r < R; ++r) {
    const uint32_t i = r * 32 + lane;
    if (i < len) {
      keys[start + i] = ((uint64_t)seg << 32) | (v[r] >> 32);
      rows[start + i] = rr[r];
    }
  }
}

__global__ void __launch_bounds__(256) k_seg_warp_sort(uint64_t* __restrict__ keys, uint32_t* __restrict__ rows,
                                                      const uint32_t* __restrict__ starts, uint64_t nr, uint64_t m) {
  const unsigned lane = threadIdx.x & 31;
  const uint64_t nwarps = (uint64_t)gridDim.x * (blockDim.x >> 5);
  for (uint64_t s = (uint64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); s < nr; s += nwarps) {
    const uint32_t start = starts[s], end = s + 1 < nr ? starts[s + 1] : (uint32_t)m, len = end - start;
    if (len <= 1) continue;
    if (len <= 32) warp_range_sort<1>(keys, rows, start, len, lane);
    else if (len <= 64) warp_range_sort<2>(keys, rows, start, len, lane);
    else if (len <= 128) warp_range_sort<4>(keys, rows, start, len, lane);
    else warp_range_sort<8>(keys, rows, start, len, lane);
  }
}

// Longest run of equal range ids in seg[0..m): run starts (per range id) then run lengths.
__global__ void k_seg_starts(const uint32_t* __restrict__ seg, uint64_t m, uint32_t* __restrict__ starts) {
  for (uint64_t j = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; j < m; j += (uint64_t)gridDim.x * blockDim.x)
    if (j == 0 || seg[j] != seg[j - 1]) starts[seg[j]] = (uint32_t)j;
}
__global__ void k_seg_maxlen(const uint32_t* __restrict__ seg, uint64_t m, const uint32_t* __restrict__ starts,
                             uint32_t* __restrict__ mx) {
  uint32_t best = 0;
  for (uint64_t j = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; j < m; j += (uint64_t)gridDim.x * blockDim.x)
    if (j + 1 == m || seg[j] != seg[j + 1]) best = max(best, (uint32_t)(j + 1) - starts[seg[j]]);
  best = __reduce_max_sync(0xffffffffu, best);
  if ((threadIdx.x & 31) == 0 && best) atomicMax(mx, best);
}

int sms_now() {
  int dev = 0, s = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&s, cudaDevAttrMultiProcessorCount, dev);
  return s;
}

uint32_t elem_grid(uint64_t n) {
  const uint64_t g = (n + 255) / 256;
  return (uint32_t)std::max<uint64_t>(1, std::min<uint64_t>(g, (uint64_t)sms_now() * 16));
}

struct CachedBuf {  // workspace from the block cache (callers synchronise before it is released)
  void* p = nullptr;
  cudaError_t alloc(size_t b) { return cache_get(&p, std::max<size_t>(b, 16)); }
  ~CachedBuf() {
    if (p) cache_put(p);
  }
};

struct DevBuf {  // stream-ordered scratch
  void* p = nullptr;
  cudaStream_t st;
  explicit DevBuf(cudaStream_t s) : st(s) {}
  cudaError_t alloc(size_t b) { return cudaMallocAsync(&p, std::max<size_t>(b, 16), st); }
  ~DevBuf() {
    if (p) cudaFreeAsync(p, st);
  }
};

// Per-launch CUDA events around the downsweeps (blu_sort_stats_t), read after the caller syncs.
struct RsTiming {  // events are created once per thread and reused (creating them takes driver locks)
  std::vector<cudaEvent_t> ev;
  size_t used = 0;
  uint64_t bytes = 0;
  cudaEvent_t next() {
    if (used == ev.size()) {
      cudaEvent_t e;
      cudaEventCreate(&e);
      ev.push_back(e);
    }
    return ev[used++];
  }
  void reset() {
    used = 0;
    bytes = 0;
  }
};
thread_local RsTiming t_rs;

// Stable LSD radix sort of the low `bits` key bits: (kin, vin) -> (kout, vout); kt/vt scratch (n).
template <typename KT>
cudaError_t radix_sort(const KT* kin, const uint32_t* vin, KT* kout, uint32_t* vout, KT* kt, uint32_t* vt, uint64_t n,
                       uint32_t bits, uint32_t* counts, uint32_t grid, cudaStream_t st, RsTiming* tm = nullptr) {
  if (n == 0) return cudaSuccess;
  // digits that vary (one small reduction + one synchronisation)
  int digits[8], passes = 0;
  {
    unsigned long long* oa = (unsigned long long*)(counts + (size_t)256 * (grid + 1));
    cudaError_t e = cudaMemsetAsync(oa, 0, 8, st);
    if (!e) e = cudaMemsetAsync(oa + 1, 0xFF, 8, st);
    if (e) return e;
    k_key_bits<KT><<<elem_grid(n), 256, 0, st>>>(kin, n, oa);
    count_launch(1);
    unsigned long long h[2];
    if ((e = cudaMemcpyAsync(h, oa, 16, cudaMemcpyDeviceToHost, st)) || (e = cudaStreamSynchronize(st))) return e;
    const int nd = std::max(1, (int)((bits + 7) / 8));
    for (int p = 0; p < nd; ++p)
      if ((((h[0] ^ h[1]) >> (8 * p)) & 255ull) != 0) digits[passes++] = p;
  }
  if (passes == 0) {  // every key equal: the stable order is the input order
    cudaError_t e = cudaMemcpyAsync(kout, kin, n * sizeof(KT), cudaMemcpyDeviceToDevice, st);
    if (!e) e = cudaMemcpyAsync(vout, vin, n * 4, cudaMemcpyDeviceToDevice, st);
    return e;
  }
  const KT* sk = kin;
  const uint32_t* sv = vin;
  for (int p = 0; p < passes; ++p) {
    const bool to_out = ((passes - 1 - p) % 2) == 0;
    KT* dk = to_out ? kout : kt;
    uint32_t* dv = to_out ? vout : vt;
    const uint32_t shift = 8u * (uint32_t)digits[p];
    k_rs_upsweep<KT><<<grid, kRT, 0, st>>>(sk, n, shift, counts);
    k_rs_scan_rows<<<256, kRT, 0, st>>>(counts, grid, counts + (size_t)256 * grid);
    if (tm) cudaEventRecord(tm->next(), st);
    k_rs_downsweep<KT><<<grid, kRT, 0, st>>>(sk, sv, dk, dv, n, shift, counts, counts + (size_t)256 * grid);
    if (tm) {
      cudaEventRecord(tm->next(), st);
      tm->bytes += 2ull * n * (sizeof(KT) + 4);
    }
    count_launch(3);
    sk = dk;
    sv = dv;
  }
  return cudaGetLastError();
}

uint32_t radix_grid() { return (uint32_t)sms_now() * 8; }  // 8 x 256 threads per SM


blu_status_t cuda_err(cudaError_t e, const char* what) {
  cudaGetLastError();
  if (e == cudaErrorMemoryAllocation) return fail(BLU_E_OOM, "%s: %s", what, cudaGetErrorString(e));
  return fail(BLU_E_CUDA, "%s: %s", what, cudaGetErrorString(e));
}

#define SCK(x, what)                                 \
  do {                                               \
    cudaError_t e_ = (x);                            \
    if (e_ != cudaSuccess) return cuda_err(e_, what); \
  } while (0)

// Duplicate ranges of sorted keys k[0..m): counts, host scan result (#active, #ranges), emit.
template <typename KT>
blu_status_t dup_pass(const KT* k, uint64_t m, const uint32_t* act_pos, uint32_t* next_pos, uint32_t* next_seg,
                      uint64_t* r_start, uint64_t* r_len, uint64_t cap, uint64_t* n_act, uint64_t* n_rng,
                      cudaStream_t st, void* ws = nullptr) {
  *n_act = *n_rng = 0;
  if (m == 0) return BLU_OK;
  const uint64_t nb = (m + kDB - 1) / kDB;
  DevBuf w(st);
  if (!ws) {
    SCK(w.alloc(nb * 8 + 16), "dup workspace");
    ws = w.p;
  }
  uint32_t* ca = (uint32_t*)ws;
  uint32_t* cs = ca + nb;
  uint32_t* tot = cs + nb;  // 2 totals
  k_dup_count<KT><<<(unsigned)nb, kDT, 0, st>>>(k, m, ca, cs);
  // totals: sum of the last offsets + counts after the scans
  SCK(cudaMemcpyAsync(tot, ca + nb - 1, 4, cudaMemcpyDeviceToDevice, st), "dup totals");
  SCK(cudaMemcpyAsync(tot + 1, cs + nb - 1, 4, cudaMemcpyDeviceToDevice, st), "dup totals");
  k_rs_scan<<<1, 1024, 0, st>>>(ca, nb);
  k_rs_scan<<<1, 1024, 0, st>>>(cs, nb);
  k_dup_emit<KT><<<(unsigned)nb, kDT, 0, st>>>(k, m, ca, cs, act_pos, next_pos, next_seg, r_start, r_len, cap);
  count_launch(4);
  uint32_t h[4];
  SCK(cudaMemcpyAsync(h, ca + nb - 1, 4, cudaMemcpyDeviceToHost, st), "dup D2H");
  SCK(cudaMemcpyAsync(h + 1, cs + nb - 1, 4, cudaMemcpyDeviceToHost, st), "dup D2H");
  SCK(cudaMemcpyAsync(h + 2, tot, 8, cudaMemcpyDeviceToHost, st), "dup D2H");
  SCK(cudaStreamSynchronize(st), "dup sync");
  *n_act = (uint64_t)h[0] + h[2];
  *n_rng = (uint64_t)h[1] + h[3];
  if (r_start && *n_rng) {
    const uint64_t c = std::min(cap, *n_rng);
    k_range_lens<<<elem_grid(c), 256, 0, st>>>(r_start, r_len, c);
    count_launch(1);
    SCK(cudaGetLastError(), "range lens");
  }
  return BLU_OK;
}

}  // namespace

// Ascending sort of n u64 keys with the radix sort above (the KMV estimate's candidate merge, kmv.cu).
// ws: caller-owned device scratch of sort_u64_scratch_bytes(n) bytes, released stream-ordered by the
// caller. Synchronises `st` once (the constant-digit check).
size_t sort_u64_scratch_bytes(uint64_t n) { return (size_t)n * (8 + 3 * 4) + (size_t)256 * (radix_grid() + 1) * 4 + 64; }
cudaError_t sort_u64_keys(const uint64_t* kin, uint64_t* kout, uint64_t n, void* ws, cudaStream_t st) {
  if (!n) return cudaSuccess;
  const uint32_t grid = radix_grid();
  uint64_t* kt = (uint64_t*)ws;
  uint32_t* vin = (uint32_t*)(kt + n);  // payloads are not used: any content
  uint32_t* vout = vin + n;
  uint32_t* vt = vout + n;
  uint32_t* counts = vt + n;
  return radix_sort<uint64_t>(kin, vin, kout, vout, kt, vt, n, 64, counts, grid, st);
}

}  // namespace blu

using namespace blu;

extern "C" {

blu_status_t blu_sort_partial_keys(const uint8_t* rows, uint64_t n, uint32_t W, uint32_t word, uint32_t* keys_out,
                                   void* stream) {
  env_snapshot();
  if (n && (!rows || !keys_out)) return fail(BLU_E_INVALID, "NULL pointer");
  if (W < 4 || W > 1024 || (W & 3) || 4 * word >= W) return fail(BLU_E_INVALID, "bad W %u / word %u", W, word);
  if (!n) return BLU_OK;
  cudaStream_t st = (cudaStream_t)stream;
  k_partial_keys<uint32_t><<<elem_grid(n), 256, 0, st>>>(rows, n, W, word, keys_out, nullptr);
  count_launch(1);
  SCK(cudaGetLastError(), "partial keys");
  return BLU_OK;
}

blu_status_t blu_sort_pairs(const uint32_t* keys_in, const uint32_t* payload_in, uint64_t n, uint32_t* keys_out,
                            uint32_t* payload_out, void* stream) {
  env_snapshot();
  if (n && (!keys_in || !payload_in || !keys_out || !payload_out)) return fail(BLU_E_INVALID, "NULL pointer");
  if (n >= (1ull << 32)) return fail(BLU_E_INVALID, "n >= 2^32");
  if (n && ((const void*)keys_out == (const void*)keys_in || (const void*)payload_out == (const void*)payload_in))
    return fail(BLU_E_INVALID, "outputs alias inputs");
  if (!n) return BLU_OK;
  cudaStream_t st = (cudaStream_t)stream;
  setup_pool();
  const uint32_t grid = radix_grid();
  DevBuf w(st);
  SCK(w.alloc((size_t)n * 8 + (size_t)256 * (grid + 1) * 4 + 64), "sort workspace");
  uint32_t* kt = (uint32_t*)w.p;
  uint32_t* vt = kt + n;
  uint32_t* counts = vt + n;
  SCK(radix_sort<uint32_t>(keys_in, payload_in, keys_out, payload_out, kt, vt, n, 32, counts, grid, st), "radix sort");
  return BLU_OK;
}

blu_status_t blu_sort_dup_ranges(const uint32_t* sorted_keys, uint64_t n, uint64_t* starts, uint64_t* lens, uint64_t cap,
                                 uint64_t* n_ranges, void* stream) {
  env_snapshot();
  if (!n_ranges || (n && !sorted_keys) || (cap && (!starts || !lens))) return fail(BLU_E_INVALID, "NULL pointer");
  if (n >= (1ull << 32)) return fail(BLU_E_INVALID, "n >= 2^32");
  uint64_t na = 0;
  setup_pool();
  return dup_pass<uint32_t>(sorted_keys, n, nullptr, nullptr, nullptr, cap ? starts : nullptr, cap ? lens : nullptr, cap, &na,
                            n_ranges, (cudaStream_t)stream);
}

blu_status_t blu_sort_rows(const uint8_t* rows, uint64_t n, uint32_t W, uint32_t* perm_out, void* stream,
                           blu_sort_stats_t* stats) {
  env_snapshot();
  if (n && (!rows || !perm_out)) return fail(BLU_E_INVALID, "NULL pointer");
  if (W < 4 || W > 1024 || (W & 3)) return fail(BLU_E_INVALID, "W must be a multiple of 4 in [4, 1024] (got %u)", W);
  if (n >= (1ull << 32)) return fail(BLU_E_INVALID, "n >= 2^32");
  if (stats) memset(stats, 0, sizeof *stats);
  if (!n) return BLU_OK;
  cudaStream_t st = (cudaStream_t)stream;
  const uint32_t grid = radix_grid();
  static thread_local cudaEvent_t e0 = nullptr, e1 = nullptr;
  if (stats && !e0) {
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
  }
  setup_pool();
  auto level_time = [&](uint32_t l) {
    if (!stats || l >= 256) return;
    cudaEventRecord(e1, st);
    cudaEventSynchronize(e1);
    cudaEventElapsedTime(&stats->ms[l], e0, e1);
  };
  // workspace: level-0 keys/payload scratch (u32) + level keys (u64 x3) + payload x3 + pos/seg x2;
  // from the block cache (every level ends with a synchronisation, so it is idle on return)
  static const bool dbg = benv("BLU_SORT_DEBUG") != nullptr;
  const bool no_seg = benv("BLU_SORT_NO_SEG") != nullptr;  // always the batched global radix sort
  const bool no_warp = benv("BLU_SORT_NO_WARP") != nullptr;  // window sort even for ranges <= 256
  const char* sgw = benv("BLU_SORT_SEG_W");
  const int seg_w = sgw ? atoi(sgw) : 2048;
  auto hnow = [] {
    timespec ts;
    clock_gettime(CLOCK_MONOTONIC, &ts);
    return ts.tv_sec * 1e3 + ts.tv_nsec * 1e-6;
  };
  const double h0 = hnow();
  CachedBuf w;
  const size_t need = (size_t)n * (4 + 4 + 8 + 8 + 8 + 4 + 4 + 4 + 4 * 4) + (size_t)256 * (grid + 1) * 4 + 256 +
                      ((n + kDB - 1) / kDB) * 8 + 64;
  SCK(w.alloc(need), "sort workspace");
  if (dbg) fprintf(stderr, "[blu_sort] workspace %.3f ms\n", hnow() - h0);
  uint8_t* q = (uint8_t*)w.p;
  auto take = [&](size_t b) {
    uint8_t* r = q;
    q += (b + 15) & ~(size_t)15;
    return r;
  };
  uint32_t* k32a = (uint32_t*)take(n * 4);
  uint32_t* k32b = (uint32_t*)take(n * 4);
  uint64_t* k64a = (uint64_t*)take(n * 8);
  uint64_t* k64b = (uint64_t*)take(n * 8);
  uint64_t* k64c = (uint64_t*)take(n * 8);  // radix scratch (never an input of the same sort)
  uint32_t* pa = (uint32_t*)take(n * 4);
  uint32_t* pb = (uint32_t*)take(n * 4);
  uint32_t* pc = (uint32_t*)take(n * 4);
  uint32_t* pos0 = (uint32_t*)take(n * 4);
  uint32_t* seg0 = (uint32_t*)take(n * 4);
  uint32_t* pos1 = (uint32_t*)take(n * 4);
  uint32_t* seg1 = (uint32_t*)take(n * 4);
  uint32_t* counts = (uint32_t*)take((size_t)256 * (grid + 1) * 4 + 64);
  void* dws = take(((n + kDB - 1) / kDB) * 8 + 16);  // duplicate-range block counts
  if (stats) cudaEventRecord(e0, st);
  // level 0: the whole buffer is one job ("Initially there is only one job")
  k_partial_keys<uint32_t><<<elem_grid(n), 256, 0, st>>>(rows, n, W, 0, k32a, pa);
  count_launch(1);
  RsTiming& rtm = t_rs;
  rtm.reset();
  RsTiming* tm = stats ? &rtm : nullptr;
  SCK(radix_sort<uint32_t>(k32a, pa, k32b, perm_out, (uint32_t*)k64c, pc, n, 32, counts, grid, st, tm), "level 0 sort");
  uint64_t m = 0, nr = 0;
  blu_status_t s = dup_pass<uint32_t>(k32b, n, nullptr, pos0, seg0, nullptr, nullptr, 0, &m, &nr, st, dws);
  if (s != BLU_OK) return s;
  uint32_t level = 1;
  if (stats) {
    stats->ranges[0] = nr;
    stats->active[0] = m;
    level_time(0);
  }
  // level l: every duplicate range left is a job sorted by its next 4 bytes; all of them in
  // one batched sort keyed by (range id, partial key)
  for (uint32_t word = 1; m > 0 && 4 * word < W; ++word, ++level) {
    if (stats) cudaEventRecord(e0, st);
    uint32_t bits_seg = 0;
    while (bits_seg < 32 && (1ull << bits_seg) < nr) ++bits_seg;
    k_level_keys<<<elem_grid(m), 256, 0, st>>>(rows, W, word, pos0, seg0, perm_out, m, k64a, pa);
    count_launch(1);
    // all ranges short (<= kSW / 2): two passes of shared-memory window sorts, in place
    uint32_t maxlen = ~0u;
    const int sw = seg_w == 2048 ? 2048 : 4096;
    if (!no_seg) {
      uint32_t* mx = counts + (size_t)256 * (grid + 1) + 8;
      SCK(cudaMemsetAsync(mx, 0, 4, st), "seg maxlen");
      k_seg_starts<<<elem_grid(m), 256, 0, st>>>(seg0, m, seg1);
      k_seg_maxlen<<<elem_grid(m), 256, 0, st>>>(seg0, m, seg1, mx);
      count_launch(2);
      SCK(cudaMemcpyAsync(&maxlen, mx, 4, cudaMemcpyDeviceToHost, st), "seg maxlen D2H");
      SCK(cudaStreamSynchronize(st), "seg maxlen sync");
    }
    const uint64_t* lk = k64b;
    const uint32_t* lrows = pb;
    if (maxlen <= 256 && !no_warp) {  // one warp per range, bitonic in registers
      if (tm) cudaEventRecord(tm->next(), st);
      k_seg_warp_sort<<<(uint32_t)sms_now() * 8, 256, 0, st>>>(k64a, pa, seg1, nr, m);
      if (tm) {
        cudaEventRecord(tm->next(), st);
        tm->bytes += 2ull * m * (8 + 4);
      }
      count_launch(1);
      SCK(cudaGetLastError(), "seg warp sort");
      lk = k64a;
      lrows = pa;
    } else if (maxlen <= (uint32_t)sw / 2) {
      static bool attr = false;
      if (!attr) {
        SCK(cudaFuncSetAttribute(k_seg_window_sort<4096>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 (int)seg_smem<4096>()), "seg sort smem");
        SCK(cudaFuncSetAttribute(k_seg_window_sort<2048>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 (int)seg_smem<2048>()), "seg sort smem");
        attr = true;
      }
      const uint32_t per_sm = sw == 2048 ? 3 : 1;
      const uint32_t wg =
          (uint32_t)std::max<uint64_t>(1, std::min<uint64_t>((m + sw - 1) / sw, (uint64_t)sms_now() * per_sm));
      if (tm) cudaEventRecord(tm->next(), st);
      if (sw == 2048) {
        k_seg_window_sort<2048><<<wg, 512, seg_smem<2048>(), st>>>(k64a, pa, m, 0);
        if (m > 1024) k_seg_window_sort<2048><<<wg, 512, seg_smem<2048>(), st>>>(k64a, pa, m, 1024);
      } else {
        k_seg_window_sort<4096><<<wg, 1024, seg_smem<4096>(), st>>>(k64a, pa, m, 0);
        if (m > 2048) k_seg_window_sort<4096><<<wg, 1024, seg_smem<4096>(), st>>>(k64a, pa, m, 2048);
      }
      if (tm) {
        cudaEventRecord(tm->next(), st);
        tm->bytes += 2ull * 2 * m * (8 + 4);
      }
      count_launch(2);
      SCK(cudaGetLastError(), "seg window sort");
      lk = k64a;
      lrows = pa;
    } else {
      SCK(radix_sort<uint64_t>(k64a, pa, k64b, pb, k64c, pc, m, 32 + bits_seg, counts, grid, st, tm), "level sort");
    }
    k_level_scatter<<<elem_grid(m), 256, 0, st>>>(pos0, lrows, m, perm_out);
    count_launch(1);
    uint64_t m2 = 0, nr2 = 0;
    s = dup_pass<uint64_t>(lk, m, pos0, pos1, seg1, nullptr, nullptr, 0, &m2, &nr2, st, dws);
    if (s != BLU_OK) return s;
    std::swap(pos0, pos1);
    std::swap(seg0, seg1);
    m = m2;
    nr = nr2;
    if (dbg) fprintf(stderr, "[blu_sort] level %u done at %.3f ms (m=%llu)\n", level, hnow() - h0, (unsigned long long)m);
    if (stats && level < 256) {
      stats->ranges[level] = nr;
      stats->active[level] = m;
      level_time(level);
    }
  }
  if (stats) {
    stats->levels = level;
    cudaStreamSynchronize(st);
    for (size_t i = 0; i + 1 < rtm.used; i += 2) {
      float x = 0;
      cudaEventElapsedTime(&x, rtm.ev[i], rtm.ev[i + 1]);
      stats->downsweep_ms += x;
      stats->downsweep_launches += 1;
    }
    stats->downsweep_bytes = rtm.bytes;
  }
  SCK(cudaGetLastError(), "sort rows");
  return BLU_OK;
}

}  // extern "C"
