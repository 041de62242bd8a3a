// blu_device.cuh — libblugby's device code: helpers and the bodies of the hot kernels.
//
// Compiled twice: ahead of time by nvcc into libblugby.so with GenericSpec (the schema is read from
// the kernel parameters at run time), and at run time by NVRTC with a per-plan JitSpec whose key
// dtypes, dictionary strides, value dtypes and state-field program are compile-time constants
// (jit.cpp). The same source therefore produces both the generic kernels and the specialised,
// straight-line ones. No host headers: under NVRTC the integer typedefs come from the JIT preamble.
#pragma once

#ifndef BLU_JIT
#include "blu_params.h"
#endif

namespace blu {

// Schema read from AggParams::lay at run time.
struct GenericSpec {
  static constexpr bool kStatic = false;
  static constexpr int HOTREG = 0;
  static constexpr int MMBOUND = 0;
};

// ------------------------------------------------------------------------------------------------
// device helpers
// ------------------------------------------------------------------------------------------------
__device__ __forceinline__ uint64_t fmix64(uint64_t h) {  // Murmur3 finalizer (P:153 cites Murmur)
  h ^= h >> 33;
  h *= 0xff51afd7ed558ccdull;
  h ^= h >> 33;
  h *= 0xc4ceb9fe1a85ec53ull;
  h ^= h >> 33;
  return h;
}

// home slot of a key in the shared-memory front (bits independent of the table's slot bits)
__device__ __forceinline__ uint32_t front_home(uint64_t key, uint32_t S) {
  return (uint32_t)(fmix64(key ^ 0x5bd1e995ull) >> 40) & (S - 1);
}

// Order-preserving map of IEEE-754 f64 bits onto int64 (an involution).
__device__ __forceinline__ int64_t ord_f64(uint64_t bits) {
  int64_t b = (int64_t)bits;
  return b ^ ((b >> 63) & 0x7FFFFFFFFFFFFFFFll);
}
__device__ __forceinline__ uint64_t unord_f64(int64_t o) { return (uint64_t)(o ^ ((o >> 63) & 0x7FFFFFFFFFFFFFFFll)); }

__device__ __forceinline__ uint64_t evict_first_policy() {
  uint64_t pol;
  asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  return pol;
}
__device__ __forceinline__ int4 ld_stream_v4(const void* p, uint64_t pol) {
  int4 r;
  asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.s32 {%0,%1,%2,%3}, [%4], %5;"
      : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
      : "l"(p), "l"(pol));
  return r;
}
// 256-bit streaming load (LDG.E.256 on sm_100a): one instruction per 32 contiguous bytes per lane.
// Needs PTX ISA 8.8 (CUDA >= 12.9); the JIT passes BLU_LDG256 from the NVRTC version it loaded.
#ifndef BLU_LDG256
#if defined(__CUDACC_VER_MAJOR__) && (__CUDACC_VER_MAJOR__ > 12 || (__CUDACC_VER_MAJOR__ == 12 && __CUDACC_VER_MINOR__ >= 9))
#define BLU_LDG256 1
#else
#define BLU_LDG256 0
#endif
#endif
__device__ __forceinline__ void ld_stream_v4u64(const void* p, uint64_t pol, uint64_t& a, uint64_t& b, uint64_t& c,
                                                uint64_t& d) {
#if BLU_LDG256
  asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u64 {%0,%1,%2,%3}, [%4], %5;"
      : "=l"(a), "=l"(b), "=l"(c), "=l"(d)
      : "l"(p), "l"(pol));
#else
  const int4 x = ld_stream_v4(p, pol), y = ld_stream_v4((const uint8_t*)p + 16, pol);
  a = (uint64_t)(uint32_t)x.x | ((uint64_t)(uint32_t)x.y << 32);
  b = (uint64_t)(uint32_t)x.z | ((uint64_t)(uint32_t)x.w << 32);
  c = (uint64_t)(uint32_t)y.x | ((uint64_t)(uint32_t)y.y << 32);
  d = (uint64_t)(uint32_t)y.z | ((uint64_t)(uint32_t)y.w << 32);
#endif
}
__device__ __forceinline__ int32_t ld_stream_s32(const void* p, uint64_t pol) {
  int32_t r;
  asm("ld.global.nc.L1::no_allocate.L2::cache_hint.s32 %0, [%1], %2;" : "=r"(r) : "l"(p), "l"(pol));
  return r;
}
__device__ __forceinline__ uint64_t ld_stream_u64(const void* p, uint64_t pol) {
  uint64_t r;
  asm("ld.global.nc.L1::no_allocate.L2::cache_hint.u64 %0, [%1], %2;" : "=l"(r) : "l"(p), "l"(pol));
  return r;
}

// Row mapping: a warp owns 32*R consecutive rows; lane l owns rows lb + (r>>1)*64 + (r&1) for
// R = 4 (pairs 2l, 2l+1 and 64+2l, 65+2l), lb + r for R = 2, lb for R = 1, with lb the lane base
// below. Every load instruction of a warp then covers one contiguous span (256 B for i32 pairs,
// 512 B for 8-byte pairs): whole 32-byte sectors, no half-sector re-requests.
template <int R, bool PAIR = true>
__device__ __forceinline__ uint64_t lane_base(uint64_t tile_row0, unsigned warp, unsigned lane) {
  if (!PAIR) return tile_row0 + ((uint64_t)warp * 32 + lane) * R;  // quad: R consecutive rows
  return tile_row0 + (uint64_t)warp * 32 * R + (R >= 2 ? 2 * lane : lane);
}
template <int R, bool PAIR = true>
__device__ __forceinline__ uint64_t row_of(uint64_t lb, int r) {
  if (!PAIR) return lb + r;
  return R == 4 ? lb + (uint64_t)(r >> 1) * 64 + (r & 1) : lb + r;
}

__device__ __forceinline__ int2 ld_stream_v2(const void* p, uint64_t pol) {
  int2 r;
  asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.s32 {%0,%1}, [%2], %3;" : "=r"(r.x), "=r"(r.y) : "l"(p), "l"(pol));
  return r;
}

// Load this lane's R rows of one column as 64-bit patterns (i32 sign-extended). Rows >= n read 0.
// vec: bit 0 = every column 16-byte aligned, bit 1 = 32-byte aligned (256-bit loads allowed).
template <int R, bool PAIR = true>
__device__ __forceinline__ void load_rows(const void* base, int dt, uint64_t lb, uint64_t n, uint32_t vec,
                                          uint64_t pol, uint64_t (&out)[R]) {
  if (!PAIR && R >= 4) {  // quad mapping: rows lb..lb+R-1 (path (a): 16-byte loads, 4 i32 rows each)
    if (dt == BLU_I32) {
      const int32_t* p = (const int32_t*)base + lb;
      if (vec && lb + R <= n) {
#pragma unroll
        for (int q = 0; q < R; q += 4) {
          int4 v = ld_stream_v4(p + q, pol);
          out[q] = (uint64_t)(int64_t)v.x;
          out[(q + 1) % R] = (uint64_t)(int64_t)v.y;
          out[(q + 2) % R] = (uint64_t)(int64_t)v.z;
          out[(q + 3) % R] = (uint64_t)(int64_t)v.w;
        }
      } else {
#pragma unroll
        for (int r = 0; r < R; ++r) out[r] = lb + r < n ? (uint64_t)(int64_t)ld_stream_s32(p + r, pol) : 0ull;
      }
    } else {
      const uint64_t* p = (const uint64_t*)base + lb;
      if ((vec & 2) && R % 4 == 0 && lb + R <= n) {  // 32 contiguous bytes per lane: whole sectors
#pragma unroll
        for (int r = 0; r < R; r += 4) ld_stream_v4u64(p + r, pol, out[r], out[(r + 1) % R], out[(r + 2) % R], out[(r + 3) % R]);
      } else if (vec && lb + R <= n) {
#pragma unroll
        for (int r = 0; r < R; r += 2) {
          int4 v = ld_stream_v4(p + r, pol);
          out[r] = (uint64_t)(uint32_t)v.x | ((uint64_t)(uint32_t)v.y << 32);
          out[(r + 1) % R] = (uint64_t)(uint32_t)v.z | ((uint64_t)(uint32_t)v.w << 32);
        }
      } else {
#pragma unroll
        for (int r = 0; r < R; ++r) out[r] = lb + r < n ? ld_stream_u64(p + r, pol) : 0ull;
      }
    }
    return;
  }
  if (dt == BLU_I32) {
    const int32_t* p = (const int32_t*)base;
    if (R >= 2) {
#pragma unroll
      for (int h = 0; h < R / 2; ++h) {
        const uint64_t r0 = lb + (uint64_t)h * 64;
        if (vec && r0 + 1 < n) {
          int2 v = ld_stream_v2(p + r0, pol);
          out[2 * h] = (uint64_t)(int64_t)v.x;
          out[(2 * h + 1) % R] = (uint64_t)(int64_t)v.y;
        } else {
          out[2 * h] = r0 < n ? (uint64_t)(int64_t)ld_stream_s32(p + r0, pol) : 0ull;
          out[(2 * h + 1) % R] = r0 + 1 < n ? (uint64_t)(int64_t)ld_stream_s32(p + r0 + 1, pol) : 0ull;
        }
      }
    } else {
      out[0] = lb < n ? (uint64_t)(int64_t)ld_stream_s32(p + lb, pol) : 0ull;
    }
  } else {
    const uint64_t* p = (const uint64_t*)base;
    if (R >= 2) {
#pragma unroll
      for (int h = 0; h < R / 2; ++h) {
        const uint64_t r0 = lb + (uint64_t)h * 64;
        if (vec && r0 + 1 < n) {
          int4 v = ld_stream_v4(p + r0, pol);
          out[2 * h] = (uint64_t)(uint32_t)v.x | ((uint64_t)(uint32_t)v.y << 32);
          out[(2 * h + 1) % R] = (uint64_t)(uint32_t)v.z | ((uint64_t)(uint32_t)v.w << 32);
        } else {
          out[2 * h] = r0 < n ? ld_stream_u64(p + r0, pol) : 0ull;
          out[(2 * h + 1) % R] = r0 + 1 < n ? ld_stream_u64(p + r0 + 1, pol) : 0ull;
        }
      }
    } else {
      out[0] = lb < n ? ld_stream_u64(p + lb, pol) : 0ull;
    }
  }
}

// L2 prefetch of the column bytes of rows [r0, r1) (one prefetch per 128-byte line, spread over the
// CTA): issued one tile ahead so HBM reads stay in flight while the CTA works on the current tile.
template <class SP>
__device__ __forceinline__ void prefetch_rows_l2(const AggParams& p, uint64_t r0, uint64_t r1) {
  if (r0 >= r1) return;
  const int nk = p.lay.n_keys, nv = p.lay.n_vals;
  for (int c = 0; c < nk + nv; ++c) {
    const bool is_key = c < nk;
    const int dt = is_key ? p.lay.key_dtype[c] : p.lay.val_dtype[c - nk];
    const uint32_t w = dt == BLU_I32 ? 4 : 8;
    const uint8_t* base = (const uint8_t*)(is_key ? p.key[c] : p.val[c - nk]);
    const uintptr_t a0 = ((uintptr_t)(base + r0 * w)) & ~(uintptr_t)127, a1 = (uintptr_t)(base + r1 * w);
    for (uintptr_t a = a0 + (uintptr_t)threadIdx.x * 128; a < a1; a += (uintptr_t)blockDim.x * 128)
      asm volatile("prefetch.global.L2 [%0];" ::"l"(a));
  }
}

// Identity (the mask value of P:151) of a field in its encoded 64-bit form.
__device__ __forceinline__ uint64_t identity64(int k) {
  switch (k) {
    case FK_MINI32: return (uint64_t)(int64_t)INT32_MAX;
    case FK_MAXI32: return (uint64_t)(int64_t)INT32_MIN;
    case FK_MINI64: case FK_MINF64: return (uint64_t)INT64_MAX;
    case FK_MAXI64: case FK_MAXF64: return (uint64_t)INT64_MIN;
    default: return 0ull;
  }
}

// ---- per-field update primitives, specialised on the field kind at compile time ----------------
// The kind of every field is warp-uniform, so kernels dispatch ONCE per field per tile (a uniform
// switch) and then run straight-line updates for all R rows of the tile.
template <int K>
struct KC {
  static constexpr int v = K;
};

// Compile-time loop: f(KC<I>{}) for I in [B, E).
template <int B, int E, class F>
__device__ __forceinline__ void sfor(F&& f) {
  if constexpr (B < E) {
    f(KC<B>{});
    sfor<B + 1, E>(f);
  }
}

template <class Fn>
__device__ __forceinline__ void dispatch_kind(int kind, Fn&& fn) {
  switch (kind) {
    case FK_COUNT: fn(KC<FK_COUNT>{}); break;
    case FK_SUMI: fn(KC<FK_SUMI>{}); break;
    case FK_SUMF: fn(KC<FK_SUMF>{}); break;
    case FK_MINI32: fn(KC<FK_MINI32>{}); break;
    case FK_MAXI32: fn(KC<FK_MAXI32>{}); break;
    case FK_MINI64: fn(KC<FK_MINI64>{}); break;
    case FK_MAXI64: fn(KC<FK_MAXI64>{}); break;
    case FK_MINF64: fn(KC<FK_MINF64>{}); break;
    default: fn(KC<FK_MAXF64>{}); break;
  }
}

// Encoded value of a field: f64 MIN/MAX through ord_f64 (RAW row values only).
template <int K, bool RAW>
__device__ __forceinline__ uint64_t enc(uint64_t x) {
  if (RAW && (K == FK_MINF64 || K == FK_MAXF64)) return (uint64_t)ord_f64(x);
  return x;
}

// Warp-level L2 prefetch of rows [r0, min(r0 + rows, n)) of every key and value column: lane l takes
// the column's 128-byte lines l, l + 32, ... (C4: 3 i32 keys + i32 + 2 i64 values over 128 rows =
// 32 lines, one per lane). Issued for the warp's next tile before it works on the current one.
template <class SP>
__device__ __forceinline__ void prefetch_warp_rows_l2(const AggParams& p, uint64_t r0, uint64_t rows, uint64_t n,
                                                      unsigned lane) {
  if (r0 >= n) return;
  const uint64_t r1 = r0 + rows < n ? r0 + rows : n;
  auto col = [&](const void* base, uint32_t w) {
    const uintptr_t a0 = ((uintptr_t)base + r0 * w) & ~(uintptr_t)127, a1 = (uintptr_t)base + r1 * w;
    for (uintptr_t a = a0 + (uintptr_t)lane * 128; a < a1; a += 32 * 128) asm volatile("prefetch.global.L2 [%0];" ::"l"(a));
  };
  if constexpr (SP::kStatic) {
    sfor<0, SP::NK>([&](auto kc) {
      constexpr int k = decltype(kc)::v;
      col(p.key[k], SP::KDT[k] == BLU_I32 ? 4u : 8u);
    });
    sfor<0, SP::NV>([&](auto cc) {
      constexpr int c = decltype(cc)::v;
      col(p.val[c], SP::VDT[c] == BLU_I32 ? 4u : 8u);
    });
  } else {
    for (int k = 0; k < p.lay.n_keys; ++k) col(p.key[k], p.lay.key_dtype[k] == BLU_I32 ? 4u : 8u);
    for (int c = 0; c < p.lay.n_vals; ++c) col(p.val[c], p.lay.val_dtype[c] == BLU_I32 ? 4u : 8u);
  }
}

// Bulk L2 prefetch of a contiguous byte range by the TMA unit (one instruction for the whole range):
// cp.async.bulk.prefetch.L2 needs a 16-byte aligned address and a multiple of 16 bytes.
__device__ __forceinline__ void bulk_prefetch_l2(const void* p, uint64_t bytes) {
  const uintptr_t a0 = (uintptr_t)p & ~(uintptr_t)15, a1 = ((uintptr_t)p + bytes + 15) & ~(uintptr_t)15;
  if (a1 > a0)
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(a0), "r"((uint32_t)(a1 - a0)) : "memory");
}

// Rows [r0, r1) of every key and value column prefetched into L2 by the TMA unit (JIT kernels).
template <class SP>
__device__ __forceinline__ void bulk_prefetch_rows_l2(const AggParams& p, uint64_t r0, uint64_t r1) {
  if constexpr (SP::kStatic) {
    if (r0 >= r1) return;
    sfor<0, SP::NK>([&](auto kc) {
      constexpr int k = decltype(kc)::v;
      constexpr uint64_t w = SP::KDT[k] == BLU_I32 ? 4 : 8;
      bulk_prefetch_l2((const uint8_t*)p.key[k] + r0 * w, (r1 - r0) * w);
    });
    sfor<0, SP::NV>([&](auto cc) {
      constexpr int c = decltype(cc)::v;
      constexpr uint64_t w = SP::VDT[c] == BLU_I32 ? 4 : 8;
      bulk_prefetch_l2((const uint8_t*)p.val[c] + r0 * w, (r1 - r0) * w);
    });
  }
}

// Shared-memory table (path (a) and the hot-key front): SoA per field, S entries per field.
// Encodings: COUNT u32; SUMI as two u32 arrays lo[S], hi[S] — native 32-bit ATOMS with an explicit
// carry (64-bit shared atomics are CAS loops on sm_100a); SUMF f64 (CAS loop);
// MIN/MAX i32 native ATOMS.MIN/MAX; 64-bit MIN/MAX read first, atomic only if it improves (after
// warm-up a running min/max almost never changes, so almost every row costs one LDS).
template <int K, bool RAW>
__device__ __forceinline__ void s_upd(uint8_t* base, uint32_t e, uint32_t S, uint64_t x) {
  x = enc<K, RAW>(x);
  if constexpr (K == FK_COUNT) {
    atomicAdd((uint32_t*)base + e, (uint32_t)x);
  } else if constexpr (K == FK_SUMI) {
    uint32_t lo = (uint32_t)x, hi = (uint32_t)(x >> 32);
    uint32_t old = atomicAdd((uint32_t*)base + e, lo);
    hi += (uint32_t)(old + lo < old);
    if (hi) atomicAdd((uint32_t*)base + S + e, hi);
  } else if constexpr (K == FK_SUMF) {
    atomicAdd((double*)base + e, __longlong_as_double((long long)x));
  } else if constexpr (K == FK_MINI32) {
    int v = (int)x;
    int* q = (int*)base + e;
    if (v < *(volatile int*)q) atomicMin(q, v);
  } else if constexpr (K == FK_MAXI32) {
    int v = (int)x;
    int* q = (int*)base + e;
    if (v > *(volatile int*)q) atomicMax(q, v);
  } else if constexpr (K == FK_MINI64 || K == FK_MINF64) {
    long long v = (long long)x;
    long long* q = (long long*)base + e;
    if (v < *(volatile long long*)q) atomicMin(q, v);
  } else {
    long long v = (long long)x;
    long long* q = (long long*)base + e;
    if (v > *(volatile long long*)q) atomicMax(q, v);
  }
}

__device__ __forceinline__ void smem_init_entry(uint8_t* base, int k, uint32_t e, uint32_t S) {
  switch (k) {
    case FK_COUNT: ((uint32_t*)base)[e] = 0u; break;
    case FK_SUMI: ((uint32_t*)base)[e] = 0u; ((uint32_t*)base)[S + e] = 0u; break;
    case FK_SUMF: ((uint64_t*)base)[e] = 0ull; break;
    case FK_MINI32: ((int*)base)[e] = INT32_MAX; break;
    case FK_MAXI32: ((int*)base)[e] = INT32_MIN; break;
    default: ((uint64_t*)base)[e] = identity64(k); break;
  }
}

// A shared-memory entry's state as the encoded 64-bit value to combine into global memory.
template <int K>
__device__ __forceinline__ uint64_t s_read(const uint8_t* base, uint32_t e, uint32_t S) {
  if constexpr (K == FK_COUNT) return (uint64_t)((const uint32_t*)base)[e];
  else if constexpr (K == FK_SUMI)
    return (uint64_t)((const uint32_t*)base)[e] | ((uint64_t)((const uint32_t*)base)[S + e] << 32);
  else if constexpr (K == FK_MINI32 || K == FK_MAXI32) return (uint64_t)(int64_t)((const int*)base)[e];
  else return ((const uint64_t*)base)[e];
}

// Global AoS slot field (path b): fire-and-forget reductions REDG.E.ADD.64 / ADD.F64 / MIN.S64 ...
template <int K, bool RAW>
__device__ __forceinline__ void g_upd(uint8_t* a, uint64_t x) {
  x = enc<K, RAW>(x);
  if constexpr (K == FK_COUNT || K == FK_SUMI) atomicAdd((unsigned long long*)a, (unsigned long long)x);
  else if constexpr (K == FK_SUMF) atomicAdd((double*)a, __longlong_as_double((long long)x));
  else if constexpr (K == FK_MINI32) atomicMin((int*)a, (int)x);
  else if constexpr (K == FK_MAXI32) atomicMax((int*)a, (int)x);
  else if constexpr (K == FK_MINI64 || K == FK_MINF64) atomicMin((long long*)a, (long long)x);
  else atomicMax((long long*)a, (long long)x);
}

// Global dense state field (paths a / b'): every field 8 bytes (i32 MIN/MAX widened).
template <int K, bool RAW>
__device__ __forceinline__ void d_upd(uint64_t* a, uint64_t x) {
  x = enc<K, RAW>(x);
  if constexpr (K == FK_COUNT || K == FK_SUMI) atomicAdd((unsigned long long*)a, (unsigned long long)x);
  else if constexpr (K == FK_SUMF) atomicAdd((double*)a, __longlong_as_double((long long)x));
  else if constexpr (K == FK_MINI32 || K == FK_MINI64 || K == FK_MINF64) atomicMin((long long*)a, (long long)x);
  else atomicMax((long long*)a, (long long)x);
}

__device__ __forceinline__ uint64_t* dense_addr(const AggParams& p, int j, uint64_t g) {
  const Field& f = p.lay.f[j];
  return (uint64_t*)p.dense[f.sgroup] + (uint64_t)f.sidx * p.lay.domain + g;
}

// Linear probing from fmix64(key) & mask; read-before-CAS; keys are write-once (EMPTY -> key), so
// a stale read can only show EMPTY and the CAS resolves it ("next empty slot").
__device__ __forceinline__ bool hash_locate(uint8_t* table, uint64_t mask, uint32_t sb, uint64_t key,
                                            uint64_t first, uint64_t idx, uint32_t max_probe, uint64_t& out) {
  uint64_t cur = first;
  for (uint32_t p = 0; p < max_probe; ++p) {
    unsigned long long* kp = (unsigned long long*)(table + idx * sb);
    if (p) cur = __ldcg(kp);
    if (cur == key) { out = idx; return true; }
    if (cur == kEmpty) {
      unsigned long long old = atomicCAS(kp, (unsigned long long)kEmpty, (unsigned long long)key);
      if (old == kEmpty || old == key) { out = idx; return true; }
    }
    idx = (idx + 1) & mask;
  }
  return false;
}

// Pack the key columns of rows [row, row+R) (S1, CCAT P:111): sparse -> code; dense -> mixed radix
// sum code_j * stride_j. Invalid codes raise FLAG_KEY_RANGE; rows >= n are not valid.
template <class SP, int R, bool PAIR = true>
__device__ __forceinline__ uint32_t pack_keys(const AggParams& p, uint64_t row, uint64_t n, uint64_t pol,
                                              uint64_t (&key)[R]) {
  uint32_t valid = 0;
#pragma unroll
  for (int r = 0; r < R; ++r) {
    key[r] = 0;
    if (row_of<R, PAIR>(row, r) < n) valid |= 1u << r;
  }
  uint32_t bad = 0;
  if constexpr (SP::kStatic) {  // JIT: key dtypes, dictionary sizes and strides are constants
    if constexpr (SP::SPARSE) {
      uint64_t c[R];
      constexpr int dt = SP::KDT[0];
      load_rows<R, PAIR>(p.key[0], dt, row, n, p.vec_ok, pol, c);
#pragma unroll
      for (int r = 0; r < R; ++r) {
        key[r] = c[r];
        if constexpr (SP::PADK) {
          if (c[r] == kEmpty) valid &= ~(1u << r);  // padding record
        }
        if ((int64_t)c[r] < 0) bad |= 1u << r;
      }
    } else {
      sfor<0, SP::NK>([&](auto kc) {
        constexpr int k = decltype(kc)::v;
        constexpr int dt = SP::KDT[k];
        constexpr uint64_t d = SP::DICT[k], st = SP::STRIDE[k];
        uint64_t c[R];
        load_rows<R, PAIR>(p.key[k], dt, row, n, p.vec_ok, pol, c);
#pragma unroll
        for (int r = 0; r < R; ++r) {
          if (c[r] >= d) bad |= 1u << r;
          key[r] += c[r] * st;
        }
      });
    }
  } else if (p.lay.sparse) {
    uint64_t c[R];
    load_rows<R, PAIR>(p.key[0], p.lay.key_dtype[0], row, n, p.vec_ok, pol, c);
#pragma unroll
    for (int r = 0; r < R; ++r) {
      key[r] = c[r];
      if (p.lay.pad_keys && c[r] == kEmpty) valid &= ~(1u << r);  // padding record
      if ((int64_t)c[r] < 0) bad |= 1u << r;
    }
  } else {
    for (int k = 0; k < p.lay.n_keys; ++k) {
      uint64_t c[R];
      load_rows<R, PAIR>(p.key[k], p.lay.key_dtype[k], row, n, p.vec_ok, pol, c);
      const uint64_t d = p.lay.dict[k], s = p.lay.stride[k];
#pragma unroll
      for (int r = 0; r < R; ++r) {
        if (c[r] >= d) bad |= 1u << r;  // unsigned: negatives are huge
        key[r] += c[r] * s;
      }
    }
  }
  bad &= valid;
  if (bad) atomicOr(p.flags, FLAG_KEY_RANGE);
  return valid & ~bad;
}

// Load this lane's rows of every value column (JIT: dtypes are constants).
template <class SP, int NV, int R, bool PAIR = true>
__device__ __forceinline__ void load_vals(const AggParams& p, uint64_t row, uint64_t n, uint64_t pol,
                                          uint64_t (&v)[NV][R]) {
  if constexpr (SP::kStatic) {
    sfor<0, SP::NV>([&](auto cc) {
      constexpr int c = decltype(cc)::v;
      constexpr int dt = SP::VDT[c];
      load_rows<R, PAIR>(p.val[c], dt, row, n, p.vec_ok, pol, v[c]);
    });
  } else {
#pragma unroll
    for (int c = 0; c < NV; ++c)
      if (c < p.lay.n_vals) load_rows<R, PAIR>(p.val[c], p.lay.val_dtype[c], row, n, p.vec_ok, pol, v[c]);
  }
}

// MIN/MAX skip bounds of a shared-memory table (SP::MMBOUND, JIT only, opt-in: measured no faster on
// C2, slower on C4 — DESIGN.md §7h). For each MIN field the CTA
// publishes B >= max over the table's live entries of their current (encoded) MIN; a row whose value
// is >= B cannot lower the MIN of any entry, so it skips the read-before-atomic of s_upd (MAX
// symmetric). An entry's MIN only ever decreases, so every value ever computed from it stays an
// upper bound of its current MIN: a bound may be stale, never wrong, and concurrent publishers need
// no ordering. Every warp, every kMMRefresh of its own tiles, takes the max over its 1/nwarps slice
// of the entries (part[warp]) and publishes the max over all warps' parts; no warp carries more of
// this work than another (tiles are assigned statically, so one busy warp would hold the CTA at its
// final barrier). Parts start at the identity: nothing is skipped until every warp has refreshed.
constexpr int kMMRefresh = 16;
template <class SP>
constexpr int mm_count() {
  int n = 0;
  for (int j = 0; j < SP::NF; ++j)
    if (SP::COL[j] >= 0 && (SP::KIND[j] >= FK_MINI32 && SP::KIND[j] <= FK_MAXF64)) ++n;
  return n;
}
template <class SP>
constexpr int mm_slot(int j) {  // index of MIN/MAX field j among the table's MIN/MAX fields
  int n = 0;
  for (int i = 0; i < j; ++i)
    if (SP::COL[i] >= 0 && (SP::KIND[i] >= FK_MINI32 && SP::KIND[i] <= FK_MAXF64)) ++n;
  return n;
}
template <int K>
constexpr bool is_min_kind() { return K == FK_MINI32 || K == FK_MINI64 || K == FK_MINF64; }
template <int K>
constexpr bool is_max_kind() { return K == FK_MAXI32 || K == FK_MAXI64 || K == FK_MAXF64; }
template <class SP>
struct MMShared {
  static constexpr int N = mm_count<SP>() > 0 ? mm_count<SP>() : 1;
  long long pub[N];
  long long part[32][N];
};
template <class SP>
__device__ __forceinline__ MMShared<SP>& mm_shared() {
  __shared__ MMShared<SP> m;
  return m;
}
template <class SP>
constexpr bool mm_on() {  // path (a) dense tables: BLU_GBY_MMBOUND >= 1
  if constexpr (SP::kStatic) return SP::MMBOUND != 0 && mm_count<SP>() > 0;
  else return false;
}
template <class SP>
constexpr bool mm_front_on() {  // rank front: BLU_GBY_MMBOUND=2 only (C4: spills at 96 registers)
  if constexpr (SP::kStatic) return SP::MMBOUND >= 2 && mm_count<SP>() > 0;
  else return false;
}

// MIN/MAX update of an encoded value x behind the skip bound: the read-before-atomic is a
// predicated shared load (no branch around it); a skipped read leaves `cur` at the value that makes
// the row "no better", so only an improving row reaches the atomic.
template <int K>
__device__ __forceinline__ void s_mm_bounded(uint8_t* base, uint32_t e, uint64_t x, long long bnd) {
  constexpr bool MN = is_min_kind<K>();
  const uint32_t pass = MN ? (long long)x < bnd : (long long)x > bnd;
  if constexpr (K == FK_MINI32 || K == FK_MAXI32) {
    int* q = (int*)base + e;
    int cur = MN ? INT32_MIN : INT32_MAX;
    asm volatile("{ .reg .pred p; setp.ne.b32 p, %2, 0; @p ld.volatile.shared.b32 %0, [%1]; }"
                 : "+r"(cur) : "r"((uint32_t)__cvta_generic_to_shared(q)), "r"(pass));
    if (MN ? (int)x < cur : (int)x > cur) {
      if (MN) atomicMin(q, (int)x); else atomicMax(q, (int)x);
    }
  } else {
    long long* q = (long long*)base + e;
    long long cur = MN ? INT64_MIN : INT64_MAX;
    asm volatile("{ .reg .pred p; setp.ne.b32 p, %2, 0; @p ld.volatile.shared.b64 %0, [%1]; }"
                 : "+l"(cur) : "r"((uint32_t)__cvta_generic_to_shared(q)), "r"(pass));
    if (MN ? (long long)x < cur : (long long)x > cur) {
      if (MN) atomicMin(q, (long long)x); else atomicMax(q, (long long)x);
    }
  }
}

// before the CTA's first tile (ordered by the barrier after the table initialisation)
template <class SP, bool ON>
__device__ __forceinline__ void mm_init() {
  if constexpr (ON) {
    MMShared<SP>& m = mm_shared<SP>();
    sfor<0, SP::NF>([&](auto jc) {
      constexpr int j = decltype(jc)::v;
      if constexpr (SP::COL[j] >= 0 && (is_min_kind<SP::KIND[j]>() || is_max_kind<SP::KIND[j]>())) {
        constexpr int q = mm_slot<SP>(j);
        const long long id = (long long)identity64(SP::KIND[j]);
        if (threadIdx.x < 32) m.part[threadIdx.x][q] = id;
        if (threadIdx.x == 0) m.pub[q] = id;
      }
    });
  }
}

// The calling warp (converged): refresh its part over entries of its slice of [0, n) except `skip0`,
// `skip1` (entries whose rows bypass the table, e.g. the rank front's register-held hottest keys),
// then publish the max (MIN fields) / min (MAX fields) over all warps' parts.
#ifdef BLU_MM_INLINE
#define BLU_MM_REFRESH_ATTR __forceinline__
#else
#define BLU_MM_REFRESH_ATTR __noinline__
#endif
template <class SP>
__device__ BLU_MM_REFRESH_ATTR void mm_refresh(const uint8_t* sm, uint32_t n, uint32_t skip0, uint32_t skip1) {
  if constexpr (mm_on<SP>()) {
    MMShared<SP>& m = mm_shared<SP>();
    const unsigned lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
    const uint32_t lo = (uint32_t)((uint64_t)n * warp / nw), hi = (uint32_t)((uint64_t)n * (warp + 1) / nw);
    sfor<0, SP::NF>([&](auto jc) {
      constexpr int j = decltype(jc)::v;
      constexpr int K = SP::KIND[j];
      if constexpr (SP::COL[j] >= 0 && (is_min_kind<K>() || is_max_kind<K>())) {
        constexpr int q = mm_slot<SP>(j);
        constexpr bool MN = is_min_kind<K>();
        const uint8_t* b = sm + SP::SOFF[j];
        long long acc = (long long)identity64(MN ? FK_MAXI64 : FK_MINI64);
        for (uint32_t e = lo + lane; e < hi; e += 32) {
          if (e == skip0 || e == skip1) continue;
          const long long x = (K == FK_MINI32 || K == FK_MAXI32) ? (long long)((const volatile int*)b)[e]
                                                                  : ((const volatile long long*)b)[e];
          acc = MN ? max(acc, x) : min(acc, x);
        }
#pragma unroll
        for (int o = 16; o; o >>= 1) {
          const long long y = __shfl_xor_sync(0xffffffffu, acc, o);
          acc = MN ? max(acc, y) : min(acc, y);
        }
        if (lane == 0) ((volatile long long*)m.part[warp])[q] = acc;
        __syncwarp();
        long long all = lane < nw ? ((const volatile long long*)m.part[lane])[q]
                                  : (long long)identity64(MN ? FK_MAXI64 : FK_MINI64);
#pragma unroll
        for (int o = 16; o; o >>= 1) {
          const long long y = __shfl_xor_sync(0xffffffffu, all, o);
          all = MN ? max(all, y) : min(all, y);
        }
        if (lane == 0) ((volatile long long*)m.pub)[q] = all;
      }
    });
  }
}

// Apply every field to the rows in `mask` of a shared-memory table at entries e[r].
template <class SP, int NV, int R, bool MMB = false>
__device__ __forceinline__ void smem_apply_rows(const AggParams& p, uint8_t* sm, const uint32_t (&e)[R],
                                                uint32_t mask, const uint64_t (&v)[NV][R]) {
  const uint32_t S = p.S;
#ifdef BLU_FIELD_MAJOR  // experiment switch (BLU_GBY_JIT_DEFS): the previous field-major order
  if constexpr (SP::kStatic) {
    sfor<0, SP::NF>([&](auto jc) {
      constexpr int j = decltype(jc)::v;
      constexpr int K = SP::KIND[j], c = SP::COL[j];
      uint8_t* b = sm + p.soff[j];
#pragma unroll
      for (int r = 0; r < R; ++r)
        if (mask >> r & 1) {
          if constexpr (c < 0) s_upd<FK_COUNT, true>(b, e[r], S, 1ull);
          else s_upd<K, true>(b, e[r], S, v[c][r]);
        }
    });
    return;
  }
#endif
  if constexpr (SP::kStatic) {  // JIT: straight-line updates; one branch per row, not per (field, row)
#ifndef BLU_SOFF_PARAM  // table entries and field offsets are compile-time constants of the launch
    constexpr uint32_t ST = SP::STAB;
#else
    const uint32_t ST = S;
#endif
    long long bnd[SP::NF > 0 ? SP::NF : 1];
    sfor<0, SP::NF>([&](auto jc) {
      constexpr int j = decltype(jc)::v;
      if constexpr (MMB && SP::COL[j] >= 0 && (is_min_kind<SP::KIND[j]>() || is_max_kind<SP::KIND[j]>()))
        bnd[j] = ((const volatile long long*)mm_shared<SP>().pub)[mm_slot<SP>(j)];
    });
#pragma unroll
    for (int r = 0; r < R; ++r)
      if (mask >> r & 1) {
        sfor<0, SP::NF>([&](auto jc) {
          constexpr int j = decltype(jc)::v;
          constexpr int K = SP::KIND[j], c = SP::COL[j];
#ifndef BLU_SOFF_PARAM
          uint8_t* b = sm + SP::SOFF[j];
#else
          uint8_t* b = sm + p.soff[j];
#endif
          if constexpr (c < 0) {
            s_upd<FK_COUNT, true>(b, e[r], ST, 1ull);
          } else if constexpr (MMB && is_min_kind<K>()) {
            s_mm_bounded<K>(b, e[r], enc<K, true>(v[c][r]), bnd[j]);
          } else if constexpr (MMB && is_max_kind<K>()) {
            s_mm_bounded<K>(b, e[r], enc<K, true>(v[c][r]), bnd[j]);
          } else {
            s_upd<K, true>(b, e[r], ST, v[c][r]);
          }
        });
      }
    return;
  }
  for (uint32_t m = p.cntmask; m; m &= m - 1) {
    uint8_t* b = sm + p.soff[__ffs(m) - 1];
#pragma unroll
    for (int r = 0; r < R; ++r)
      if (mask >> r & 1) s_upd<FK_COUNT, true>(b, e[r], S, 1ull);
  }
#pragma unroll
  for (int c = 0; c < NV; ++c) {
    if (c >= p.lay.n_vals) break;
    for (uint32_t m = p.colmask[c]; m; m &= m - 1) {
      const int j = __ffs(m) - 1;
      uint8_t* b = sm + p.soff[j];
      dispatch_kind(p.lay.f[j].kind, [&](auto kc) {
        constexpr int K = decltype(kc)::v;
#pragma unroll
        for (int r = 0; r < R; ++r)
          if (mask >> r & 1) s_upd<K, true>(b, e[r], S, v[c][r]);
      });
    }
  }
}

// Apply every field to the rows in `mask` of the global target: AoS slots (hash) or dense state.
template <class SP, int NV, int R, bool DIRECT>
__device__ __forceinline__ void global_apply_rows(const AggParams& p, const uint64_t (&slot)[R], uint32_t mask,
                                                  const uint64_t (&v)[NV][R]) {
  const Layout& L = p.lay;
  uint8_t* tb = (uint8_t*)p.table;
#ifdef BLU_FIELD_MAJOR
  if constexpr (SP::kStatic) {
    sfor<0, SP::NF>([&](auto jc) {
      constexpr int j = decltype(jc)::v;
      constexpr int K = SP::KIND[j], c = SP::COL[j], KK = c < 0 ? FK_COUNT : K;
      constexpr int sg = SP::SGROUP[j], goff = SP::GOFF[j];
      constexpr uint64_t base = (uint64_t)SP::SIDX[j] * SP::DOMAIN, slot_b = SP::SLOT;
#pragma unroll
      for (int r = 0; r < R; ++r)
        if (mask >> r & 1) {
          const uint64_t x = c < 0 ? 1ull : v[c < 0 ? 0 : c][r];
          if constexpr (DIRECT) d_upd<KK, true>((uint64_t*)p.dense[sg] + base + slot[r], x);
          else g_upd<KK, true>(tb + slot[r] * slot_b + goff, x);
        }
    });
    return;
  }
#endif
  if constexpr (SP::kStatic) {  // JIT: slot size, field offsets and dense groups are constants
#pragma unroll
    for (int r = 0; r < R; ++r)
      if (mask >> r & 1) {  // one branch per row; its REDs go out back to back
        sfor<0, SP::NF>([&](auto jc) {
          constexpr int j = decltype(jc)::v;
          constexpr int K = SP::KIND[j], c = SP::COL[j], KK = c < 0 ? FK_COUNT : K;
          constexpr int sg = SP::SGROUP[j], goff = SP::GOFF[j];
          constexpr uint64_t base = (uint64_t)SP::SIDX[j] * SP::DOMAIN, slot_b = SP::SLOT;
          const uint64_t x = c < 0 ? 1ull : v[c < 0 ? 0 : c][r];
          if constexpr (DIRECT) d_upd<KK, true>((uint64_t*)p.dense[sg] + base + slot[r], x);
          else g_upd<KK, true>(tb + slot[r] * slot_b + goff, x);
        });
      }
    return;
  }
  for (uint32_t m = p.cntmask; m; m &= m - 1) {
    const int j = __ffs(m) - 1;
#pragma unroll
    for (int r = 0; r < R; ++r)
      if (mask >> r & 1) {
        if (DIRECT) d_upd<FK_COUNT, true>(dense_addr(p, j, slot[r]), 1ull);
        else g_upd<FK_COUNT, true>(tb + slot[r] * L.slot_bytes + L.f[j].goff, 1ull);
      }
  }
#pragma unroll
  for (int c = 0; c < NV; ++c) {
    if (c >= L.n_vals) break;
    for (uint32_t m = p.colmask[c]; m; m &= m - 1) {
      const int j = __ffs(m) - 1;
      dispatch_kind(L.f[j].kind, [&](auto kc) {
        constexpr int K = decltype(kc)::v;
#pragma unroll
        for (int r = 0; r < R; ++r)
          if (mask >> r & 1) {
            if (DIRECT) d_upd<K, true>(dense_addr(p, j, slot[r]), v[c][r]);
            else g_upd<K, true>(tb + slot[r] * L.slot_bytes + L.f[j].goff, v[c][r]);
          }
      });
    }
  }
}

// ------------------------------------------------------------------------------------------------
// S5a: path (a) dense shared-memory aggregation (§4.3.2)
// ------------------------------------------------------------------------------------------------
// ---- path (a) fused init / finalize helpers ---------------------------------------------------
__device__ __forceinline__ void st_release_gpu(uint32_t* a, uint32_t v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(a), "r"(v) : "memory");
}
__device__ __forceinline__ uint32_t ld_acquire_gpu(const uint32_t* a) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(a) : "memory");
  return v;
}
__device__ __forceinline__ uint32_t atom_add_acq_rel_gpu(uint32_t* a, uint32_t v) {
  uint32_t old;
  asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], %2;" : "=r"(old) : "l"(a), "r"(v) : "memory");
  return old;
}

// Dense-state identities per group: int64 SUM / f64 SUM -> 0, MIN -> INT64_MAX, MAX -> INT64_MIN.
__device__ __forceinline__ void dense_init_all(const AggParams& p) {
  const uint64_t D = p.lay.domain;
  for (int g = 0; g < 4; ++g) {
    const uint64_t n = (uint64_t)p.lay.n_group[g] * D;
    const uint64_t v = g == SG_MIN ? (uint64_t)INT64_MAX : g == SG_MAX ? (uint64_t)INT64_MIN : 0ull;
    for (uint64_t i = threadIdx.x; i < n; i += blockDim.x) ((uint64_t*)p.dense[g])[i] = v;
  }
}

__device__ __forceinline__ void store_bits(void* out, uint64_t pos, int dtype, uint64_t bits) {
  if (dtype == BLU_I32) ((int32_t*)out)[pos] = (int32_t)(uint32_t)bits;
  else ((uint64_t*)out)[pos] = bits;
}

// One CTA compacts the D-entry dense state (occupancy = COUNT > 0) into the result columns in key
// order: block-wide ballot/popc prefix per chunk of blockDim entries.
__device__ __forceinline__ void dense_finalize_block(const AggParams& p, const FinalParams& fp) {
  __shared__ uint32_t wcnt[32];
  __shared__ uint64_t base_s;
  const Layout& L = p.lay;
  const uint64_t D = L.domain;
  const Field& cf = L.f[L.count_field];
  const unsigned lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  if (threadIdx.x == 0) base_s = 0;
  __syncthreads();
  for (uint64_t c0 = 0; c0 < D; c0 += blockDim.x) {
    const uint64_t e = c0 + threadIdx.x;
    const bool occ = e < D && __ldcg((const long long*)p.dense[cf.sgroup] + (uint64_t)cf.sidx * D + e) > 0;
    const unsigned bal = __ballot_sync(0xffffffffu, occ);
    if (lane == 0) wcnt[warp] = __popc(bal);
    __syncthreads();
    uint32_t before = 0, tot = 0;
    for (unsigned w = 0; w < nw; ++w) {
      if (w < warp) before += wcnt[w];
      tot += wcnt[w];
    }
    before += __popc(bal & ((1u << lane) - 1u));
    if (occ) {
      const uint64_t pos = base_s + before;
      for (int k = 0; k < L.n_keys; ++k) store_bits(fp.out_keys[k], pos, L.key_dtype[k], (e / L.stride[k]) % L.dict[k]);
      for (int o = 0; o < fp.n_out; ++o) {
        const Field& f = L.f[fp.out_field[o]];
        uint64_t x = __ldcg((const unsigned long long*)p.dense[f.sgroup] + (uint64_t)f.sidx * D + e);
        if (fp.out_kind[o] == 1) {  // AVG = (double)SUM / (double)COUNT (reading A12)
          const Field& f2 = L.f[fp.out_field2[o]];
          const uint64_t cnt = __ldcg((const unsigned long long*)p.dense[f2.sgroup] + (uint64_t)f2.sidx * D + e);
          const double sm_ = f.kind == FK_SUMF ? __longlong_as_double((long long)x) : (double)(long long)x;
          x = (uint64_t)__double_as_longlong(sm_ / (double)(long long)cnt);
        } else if (f.kind == FK_MINF64 || f.kind == FK_MAXF64) {
          x = unord_f64((int64_t)x);
        }
        store_bits(fp.out_vals[o], pos, fp.out_dtype[o], x);
      }
    }
    __syncthreads();
    if (threadIdx.x == 0) base_s += tot;
    __syncthreads();
  }
  if (threadIdx.x == 0) *fp.n_groups = base_s;
}

// ---- software-pipelined row stream (NVRTC-specialised kernels only: dense PIPE, global MODE 3) --
// A warp issues the loads of its next tile before it unpacks and aggregates the current one, so the
// HBM reads of tile t+1 are in flight during the work on tile t (without it, every tile waited the
// full load latency right after issuing: 53% of C4's stall samples sat on the first use of a load).
// Loaded words stay raw (i32 columns: one register; 8-byte columns: two) until the tile is unpacked.
template <class SP, int R>
struct RawTile {
  static constexpr int NKC = SP::NK, NVC = SP::NV > 0 ? SP::NV : 1;
  uint32_t klo[NKC][R], khi[NKC][R], vlo[NVC][R], vhi[NVC][R];
};

struct NoRawTile {};
template <class SP, int R, bool PIPE>
struct RawTileSel { using type = NoRawTile; };
template <class SP, int R>
struct RawTileSel<SP, R, true> { using type = RawTile<SP, R>; };
template <class SP, int R, bool PIPE>
using RawTileFor = typename RawTileSel<SP, R, PIPE>::type;

// Issue the loads of this lane's R rows of one column (PAIR mapping, R even); rows >= n read 0.
template <int R, bool W64>
__device__ __forceinline__ void load_raw(const void* base, uint64_t lb, uint64_t n, uint32_t vec, uint64_t pol,
                                         uint32_t (&lo)[R], uint32_t (&hi)[R]) {
#pragma unroll
  for (int h = 0; h < R / 2; ++h) {
    const uint64_t r0 = lb + (uint64_t)h * 64;
    if (vec && r0 + 1 < n) {
      if constexpr (W64) {
        const int4 x = ld_stream_v4((const uint64_t*)base + r0, pol);
        lo[2 * h] = (uint32_t)x.x, hi[2 * h] = (uint32_t)x.y, lo[2 * h + 1] = (uint32_t)x.z, hi[2 * h + 1] = (uint32_t)x.w;
      } else {
        const int2 x = ld_stream_v2((const int32_t*)base + r0, pol);
        lo[2 * h] = (uint32_t)x.x, lo[2 * h + 1] = (uint32_t)x.y;
      }
    } else {
#pragma unroll
      for (int q = 0; q < 2; ++q) {
        const uint64_t rr = r0 + q;
        if constexpr (W64) {
          const uint64_t x = rr < n ? ld_stream_u64((const uint64_t*)base + rr, pol) : 0ull;
          lo[2 * h + q] = (uint32_t)x, hi[2 * h + q] = (uint32_t)(x >> 32);
        } else {
          lo[2 * h + q] = rr < n ? (uint32_t)ld_stream_s32((const int32_t*)base + rr, pol) : 0u;
        }
      }
    }
  }
}

template <class SP, int R>
__device__ __forceinline__ void tile_load(const AggParams& p, uint64_t lb, uint64_t n, uint64_t pol, RawTile<SP, R>& T) {
  sfor<0, SP::NK>([&](auto kc) {
    constexpr int k = decltype(kc)::v;
    load_raw<R, SP::KDT[k] != BLU_I32>(p.key[k], lb, n, p.vec_ok, pol, T.klo[k], T.khi[k]);
  });
  sfor<0, SP::NV>([&](auto cc) {
    constexpr int c = decltype(cc)::v;
    load_raw<R, SP::VDT[c] != BLU_I32>(p.val[c], lb, n, p.vec_ok, pol, T.vlo[c], T.vhi[c]);
  });
}

// Raw words -> packed keys (S1, CCAT P:111, with the range check of pack_keys) and 64-bit values.
template <class SP, int NV, int R>
__device__ __forceinline__ uint32_t tile_unpack(const AggParams& p, const RawTile<SP, R>& T, uint64_t lb, uint64_t n,
                                                uint64_t (&key)[R], uint64_t (&v)[NV][R]) {
  uint32_t valid = 0, bad = 0;
#pragma unroll
  for (int r = 0; r < R; ++r) {
    key[r] = 0;
    if (row_of<R>(lb, r) < n) valid |= 1u << r;
  }
  sfor<0, SP::NK>([&](auto kc) {
    constexpr int k = decltype(kc)::v;
#pragma unroll
    for (int r = 0; r < R; ++r) {
      const uint64_t c = SP::KDT[k] == BLU_I32 ? (uint64_t)(int64_t)(int32_t)T.klo[k][r]
                                               : ((uint64_t)T.khi[k][r] << 32 | T.klo[k][r]);
      if constexpr (SP::SPARSE) {
        key[r] = c;
        if constexpr (SP::PADK) {
          if (c == kEmpty) valid &= ~(1u << r);  // padding record
        }
        if ((int64_t)c < 0) bad |= 1u << r;
#ifndef BLU_PACK64
      } else if constexpr (SP::DOMAIN <= 0xFFFFFFFFull && SP::KDT[k] == BLU_I32 && SP::DICT[k] <= 0x80000000ull) {
        // dense domain below 2^32: 32-bit mixed radix (one IMAD per column instead of a 64-bit one);
        // a negative i32 code is >= 2^31 unsigned, so the same compare rejects it
        const uint32_t c32 = T.klo[k][r];
        if (c32 >= (uint32_t)SP::DICT[k]) bad |= 1u << r;
        key[r] = (uint64_t)((uint32_t)key[r] + c32 * (uint32_t)SP::STRIDE[k]);
#endif
      } else {
        if (c >= SP::DICT[k]) bad |= 1u << r;  // unsigned: negatives are huge
        key[r] += c * SP::STRIDE[k];
      }
    }
  });
  bad &= valid;
  if (bad) atomicOr(p.flags, FLAG_KEY_RANGE);
#pragma unroll
  for (int c = 0; c < NV; ++c)
#pragma unroll
    for (int r = 0; r < R; ++r) v[c][r] = 0;
  sfor<0, SP::NV>([&](auto cc) {
    constexpr int c = decltype(cc)::v;
#pragma unroll
    for (int r = 0; r < R; ++r)
      v[c][r] = SP::VDT[c] == BLU_I32 ? (uint64_t)(int64_t)(int32_t)T.vlo[c][r]
                                      : ((uint64_t)T.vhi[c][r] << 32 | T.vlo[c][r]);
  });
  return valid & ~bad;
}

// FUSE (small inputs, where launch latency dominates): S4 init and S8 compaction run inside this
// kernel. Kept out of the large-input instantiation, whose register budget it would squeeze.
template <class SP, int NV, int R, bool FUSE = false, bool PAIRMAP = false, bool PIPE = false>
__device__ __forceinline__ void dense_body(const AggParams& p, const FinalParams& fp) {
  extern __shared__ __align__(16) uint8_t sm[];
  const Layout& L = p.lay;
  const uint32_t D = p.S;
  if (FUSE && p.fuse_init && blockIdx.x == 0) {  // S4 fused: CTA 0 initialises the global dense state
    dense_init_all(p);
    __syncthreads();
    // one gpu-scope release after the barrier (cumulative over the CTA's writes it orders) instead
    // of a sequentially consistent fence in every thread (MEMBAR.SC.GPU: 9% of C1's stall samples)
    if (threadIdx.x == 0) st_release_gpu(&p.sync[0], 1u);
  }
  for (int j = 0; j < L.n_fields; ++j)
    for (uint32_t e = threadIdx.x; e < D; e += blockDim.x) smem_init_entry(sm + p.soff[j], L.f[j].kind, e, D);
  mm_init<SP, mm_on<SP>()>();
  __syncthreads();

  const uint64_t pol = evict_first_policy();
  const uint64_t n = p.n_rows;
  const uint64_t tile = (uint64_t)blockDim.x * R;
  const uint64_t ntiles = (n + tile - 1) / tile;
  uint32_t flag_seen = 0;
  uint32_t mm_it = 0;  // this warp's tiles since its last MIN/MAX bound refresh
  if constexpr (PIPE) {  // next tile's loads in flight during this tile's shared-memory updates
    const unsigned warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    RawTile<SP, R> A, B;
    uint64_t t = blockIdx.x;
    if (t < ntiles) tile_load<SP, R>(p, lane_base<R>(t * tile, warp, lane), n, pol, A);
    while (t < ntiles) {
      const uint64_t tn = t + gridDim.x;
      const uint32_t fl = *(volatile uint32_t*)p.flags;
      if (tn < ntiles) tile_load<SP, R>(p, lane_base<R>(tn * tile, warp, lane), n, pol, B);
      uint64_t key[R];
      uint64_t v[NV][R];
      const uint32_t valid = tile_unpack<SP, NV, R>(p, A, lane_base<R>(t * tile, warp, lane), n, key, v);
      uint32_t e[R];
#pragma unroll
      for (int r = 0; r < R; ++r) e[r] = (uint32_t)key[r];
      smem_apply_rows<SP, NV, R, mm_on<SP>()>(p, sm, e, valid, v);
      if (mm_on<SP>() && ++mm_it % kMMRefresh == 0) mm_refresh<SP>(sm, D, ~0u, ~0u);
      if (__any_sync(0xffffffffu, fl)) break;
      A = B;
      t = tn;
    }
  }
  for (uint64_t t = blockIdx.x; !PIPE && t < ntiles; t += gridDim.x) {
    if (flag_seen) break;
    flag_seen = __any_sync(0xffffffffu, *(volatile uint32_t*)p.flags);  // warp-uniform, seen next tile
    const uint64_t row = lane_base<R, PAIRMAP>(t * tile, threadIdx.x >> 5, threadIdx.x & 31);
    uint64_t key[R];
    const uint32_t valid = pack_keys<SP, R, PAIRMAP>(p, row, n, pol, key);
    uint64_t v[NV][R];
    load_vals<SP, NV, R, PAIRMAP>(p, row, n, pol, v);
    uint32_t e[R];
#pragma unroll
    for (int r = 0; r < R; ++r) e[r] = (uint32_t)key[r];
    smem_apply_rows<SP, NV, R, mm_on<SP>()>(p, sm, e, valid, v);
    if (mm_on<SP>() && ++mm_it % kMMRefresh == 0) mm_refresh<SP>(sm, D, ~0u, ~0u);
  }
  __syncthreads();
  if (FUSE && p.fuse_init) {  // the dense state must be initialised before this CTA flushes into it
    if (threadIdx.x == 0)
      while (ld_acquire_gpu(&p.sync[0]) == 0u) __nanosleep(64);
    __syncthreads();
  }
  // S7: CTA -> global merge with native 64-bit REDs ("the small hash tables in shared memory
  // are merged to a global hash table in device memory").
  const uint8_t* cnt = sm + p.soff[L.count_field];
  for (uint32_t e = threadIdx.x; e < D; e += blockDim.x) {
    if (((const uint32_t*)cnt)[e] == 0) continue;
    for (int j = 0; j < L.n_fields; ++j) {
      uint8_t* b = sm + p.soff[j];
      dispatch_kind(L.f[j].kind, [&](auto kc) {
        constexpr int K = decltype(kc)::v;
        d_upd<K, false>(dense_addr(p, j, e), s_read<K>(b, e, D));
      });
    }
  }
  if (FUSE && fp.enabled) {  // S8 fused: the last CTA to finish compacts the dense state
    __shared__ int am_last;
    __syncthreads();  // this CTA's REDs are ordered before thread 0's acq_rel arrival
    if (threadIdx.x == 0) am_last = atom_add_acq_rel_gpu(&p.sync[1], 1u) == gridDim.x - 1;
    __syncthreads();  // ... and the last arrival's acquire before the whole CTA's reads
    if (am_last) dense_finalize_block(p, fp);
  }
}

// ------------------------------------------------------------------------------------------------
// S5b: path (b) global hash table / path (b') direct-mapped, optional shared-memory hot-key front
// ------------------------------------------------------------------------------------------------
// ---- kernel 3: one row lock per slot, then every aggregate with plain L2 accesses -------
__device__ __forceinline__ void row_lock_acquire(uint32_t* l) {
  for (;;) {
    uint32_t old;
    asm volatile("atom.acquire.gpu.global.cas.b32 %0, [%1], 0, 1;" : "=r"(old) : "l"(l) : "memory");
    if (old == 0) return;
    __nanosleep(32);
  }
}
__device__ __forceinline__ void row_lock_release(uint32_t* l) {
  asm volatile("st.release.gpu.global.b32 [%0], 0;" ::"l"(l) : "memory");
}

// field update under the row lock (the stored encodings of g_upd: 4-byte i32 MIN/MAX, ordered f64)
template <int K>
__device__ __forceinline__ void locked_upd(uint8_t* a, uint64_t raw) {
  const uint64_t x = enc<K, true>(raw);
  if constexpr (K == FK_COUNT || K == FK_SUMI) {
    __stcg((unsigned long long*)a, __ldcg((const unsigned long long*)a) + x);
  } else if constexpr (K == FK_SUMF) {
    const double o = __longlong_as_double((long long)__ldcg((const unsigned long long*)a));
    __stcg((unsigned long long*)a, (unsigned long long)__double_as_longlong(o + __longlong_as_double((long long)x)));
  } else if constexpr (K == FK_MINI32 || K == FK_MAXI32) {
    const int o = __ldcg((const int*)a), v = (int)x;
    if (K == FK_MINI32 ? v < o : v > o) __stcg((int*)a, v);
  } else if constexpr (K == FK_MINI64 || K == FK_MINF64) {
    const long long o = (long long)__ldcg((const unsigned long long*)a);
    if ((long long)x < o) __stcg((unsigned long long*)a, x);
  } else {
    const long long o = (long long)__ldcg((const unsigned long long*)a);
    if ((long long)x > o) __stcg((unsigned long long*)a, x);
  }
}

// Kernel 3: for each row in `mask`, lock its slot, apply every aggregate, unlock ("each thread
// locks the entire row of the hash table after it finds out that its key matches ... goes through all
// the aggregation functions and applies them one by one. Finally, the thread releases the lock").
template <class SP, int NV, int R>
__device__ __forceinline__ void global_apply_rows_locked(const AggParams& p, const uint64_t (&slot)[R], uint32_t mask,
                                                         const uint64_t (&v)[NV][R]) {
  const Layout& L = p.lay;
  uint8_t* tb = (uint8_t*)p.table;
#pragma unroll
  for (int r = 0; r < R; ++r) {
    if (!(mask >> r & 1)) continue;
    uint8_t* s = tb + slot[r] * L.slot_bytes;
    uint32_t* lk = (uint32_t*)(s + L.lock_off);
    row_lock_acquire(lk);
    if constexpr (SP::kStatic) {
      sfor<0, SP::NF>([&](auto jc) {
        constexpr int j = decltype(jc)::v;
        constexpr int c = SP::COL[j], KK = c < 0 ? FK_COUNT : SP::KIND[j], goff = SP::GOFF[j];
        locked_upd<KK>(s + goff, c < 0 ? 1ull : v[c < 0 ? 0 : c][r]);
      });
    } else {
      for (int j = 0; j < L.n_fields; ++j) {
        const int c = L.f[j].col;
        uint64_t x = 1ull;
#pragma unroll
        for (int cc = 0; cc < NV; ++cc)
          if (cc == c) x = v[cc][r];
        dispatch_kind(c < 0 ? (int)FK_COUNT : L.f[j].kind, [&](auto kc) {
          constexpr int K = decltype(kc)::v;
          locked_upd<K>(s + L.f[j].goff, x);
        });
      }
    }
    row_lock_release(lk);
  }
}

// ---- JIT front path with warp-level pre-aggregation (skewed keys) -----------------------------
template <int K>
__device__ __forceinline__ uint64_t combine_vals(uint64_t a, uint64_t b) {
  if constexpr (K == FK_SUMI || K == FK_COUNT) return a + b;
  else if constexpr (K == FK_SUMF) return (uint64_t)__double_as_longlong(__longlong_as_double((long long)a) + __longlong_as_double((long long)b));
  else if constexpr (K == FK_MINI32 || K == FK_MINI64) return (int64_t)a < (int64_t)b ? a : b;
  else if constexpr (K == FK_MAXI32 || K == FK_MAXI64) return (int64_t)a > (int64_t)b ? a : b;
  else if constexpr (K == FK_MINF64) return __longlong_as_double((long long)a) < __longlong_as_double((long long)b) ? a : b;
  else return __longlong_as_double((long long)a) > __longlong_as_double((long long)b) ? a : b;
}

// For each of the lane's R rows: lanes holding the same key (__match_any_sync) reduce every field
// onto the lowest such lane with a successor-doubling shuffle tree (log2 of the largest group per
// warp steps); only that leader probes the shared-memory front and applies the combined update
// (COUNT adds the group size). Zipf hot keys then cost one shared atomic per field per warp instead
// of one per row. Rows whose key is not in the front go to the global table with the same
// combined values.
template <class SP, int NV, int R, bool DIRECT>
__device__ __forceinline__ void front_dedupe_rows(const AggParams& p, uint8_t* sm, const uint64_t (&key)[R],
                                                  uint32_t valid, const uint64_t (&v)[NV][R]) {
  const unsigned lane = threadIdx.x & 31;
  const uint32_t S = p.S;
  uint64_t* fk = (uint64_t*)(sm + p.key_off);
  uint8_t* tb = (uint8_t*)p.table;
#pragma unroll
  for (int r = 0; r < R; ++r) {
    const bool vr = valid >> r & 1;
    const uint64_t mk = vr ? key[r] : ((1ull << 63) | lane);
    const uint32_t peers = __match_any_sync(0xffffffffu, mk);
    const uint32_t np = __popc(peers);
    const uint32_t rank = __popc(peers & ((1u << lane) - 1u));
    const uint32_t above = lane == 31 ? 0u : (peers & (0xffffffffu << (lane + 1)));
    int sk = above ? __ffs(above) - 1 : -1;
    const uint32_t maxnp = __reduce_max_sync(0xffffffffu, np);
    uint64_t xr[SP::NF];
    sfor<0, SP::NF>([&](auto jc) {
      constexpr int j = decltype(jc)::v;
      constexpr int c = SP::COL[j];
      xr[j] = c < 0 ? (uint64_t)np : v[c < 0 ? 0 : c][r];
    });
    for (uint32_t k = 1; k < maxnp; k <<= 1) {
      const int src = sk < 0 ? (int)lane : sk;
      const bool take = sk >= 0 && (rank & (2 * k - 1)) == 0;
      sfor<0, SP::NF>([&](auto jc) {
        constexpr int j = decltype(jc)::v;
        constexpr int c = SP::COL[j], K = SP::KIND[j];
        if constexpr (c >= 0) {
          const uint64_t y = __shfl_sync(0xffffffffu, xr[j], src);
          if (take) xr[j] = combine_vals<K>(xr[j], y);
        }
      });
      const int s2 = __shfl_sync(0xffffffffu, sk, src);
      sk = sk < 0 ? -1 : s2;
    }
    if (!vr || rank != 0) continue;
    // leader: linear probe of the front (up to 8 slots)
    uint32_t e = (uint32_t)(fmix64(key[r] ^ 0x5bd1e995ull) >> 40) & (S - 1);
    bool hit = false;
#pragma unroll 1
    for (int q = 0; q < 8; ++q) {
      const uint64_t cur = *(volatile uint64_t*)(fk + e);
      if (cur == key[r]) { hit = true; break; }
      if (cur == kEmpty) {
        unsigned long long old = atomicCAS((unsigned long long*)(fk + e), (unsigned long long)kEmpty,
                                           (unsigned long long)key[r]);
        if (old == kEmpty || old == key[r]) { hit = true; break; }
      }
      e = (e + 1) & (S - 1);
    }
    if (hit) {
      sfor<0, SP::NF>([&](auto jc) {
        constexpr int j = decltype(jc)::v;
        constexpr int KK = SP::COL[j] < 0 ? FK_COUNT : SP::KIND[j];
        s_upd<KK, true>(sm + p.soff[j], e, S, xr[j]);
      });
    } else if constexpr (DIRECT) {
      sfor<0, SP::NF>([&](auto jc) {
        constexpr int j = decltype(jc)::v;
        constexpr int KK = SP::COL[j] < 0 ? FK_COUNT : SP::KIND[j];
        constexpr int sg = SP::SGROUP[j];
        constexpr uint64_t base = (uint64_t)SP::SIDX[j] * SP::DOMAIN;
        d_upd<KK, true>((uint64_t*)p.dense[sg] + base + key[r], xr[j]);
      });
    } else {
      constexpr uint64_t slot_b = SP::SLOT;
      const uint64_t idx = fmix64(key[r]) & p.cap_mask;
      const uint64_t first = __ldcg((const unsigned long long*)(tb + idx * slot_b));
      uint64_t sl;
      if (!hash_locate(tb, p.cap_mask, (uint32_t)slot_b, key[r], first, idx, p.max_probe, sl)) {
        atomicOr(p.flags, FLAG_OVERFLOW);
        continue;
      }
      sfor<0, SP::NF>([&](auto jc) {
        constexpr int j = decltype(jc)::v;
        constexpr int KK = SP::COL[j] < 0 ? FK_COUNT : SP::KIND[j];
        constexpr int goff = SP::GOFF[j];
        g_upd<KK, true>(tb + sl * slot_b + goff, xr[j]);
      });
    }
  }
  __syncwarp();
}

// Rank front with warp-level combining (SP::DEDUPE, JIT only): for each of the lane's R rows, lanes
// whose rows hit the same front entry (__match_any_sync on the entry) combine every field's value
// onto the lowest such lane with a successor-doubling shuffle tree, and only that lane updates the
// shared table (COUNT adds the group size). Under Zipf skew the second, third, ... hottest keys
// repeat inside a warp; each repeat is a same-address lane in every shared atomic of the row.
template <class SP, int NV, int R>
__device__ __forceinline__ void rank_dedupe_apply(const AggParams& p, uint8_t* sm, const uint32_t (&fe)[R],
                                                  uint32_t hit, const uint64_t (&v)[NV][R]) {
  const unsigned lane = threadIdx.x & 31;
#ifndef BLU_SOFF_PARAM
  constexpr uint32_t ST = SP::STAB;
#else
  const uint32_t ST = p.S;
#endif
#pragma unroll
  for (int r = 0; r < R; ++r) {
    const bool hr = hit >> r & 1;
    const uint32_t peers = __match_any_sync(0xffffffffu, hr ? fe[r] : (0x80000000u | lane));
    const uint32_t np = __popc(peers);
    const uint32_t maxnp = __reduce_max_sync(0xffffffffu, hr ? np : 1u);
    uint64_t xr[SP::NF];
    sfor<0, SP::NF>([&](auto jc) {
      constexpr int j = decltype(jc)::v;
      constexpr int c = SP::COL[j];
      xr[j] = c < 0 ? (uint64_t)np : v[c < 0 ? 0 : c][r];
    });
    if (maxnp > 1) {
      const uint32_t rank = __popc(peers & ((1u << lane) - 1u));
      const uint32_t above = lane == 31 ? 0u : (peers & (0xffffffffu << (lane + 1)));
      int sk = above ? __ffs(above) - 1 : -1;  // next member of this lane's group
      for (uint32_t k = 1; k < maxnp; k <<= 1) {
        const int src = sk < 0 ? (int)lane : sk;
        const bool take = sk >= 0 && (rank & (2 * k - 1)) == 0;
        sfor<0, SP::NF>([&](auto jc) {
          constexpr int j = decltype(jc)::v;
          constexpr int c = SP::COL[j], K = SP::KIND[j];
          if constexpr (c >= 0) {
            const uint64_t y = __shfl_sync(0xffffffffu, xr[j], src);
            if (take) xr[j] = combine_vals<K>(xr[j], y);
          }
        });
        const int s2 = __shfl_sync(0xffffffffu, sk, src);
        sk = sk < 0 ? -1 : s2;
      }
      if (rank != 0) continue;  // a non-leader's row is in its leader's combined values
    }
    if (!hr) continue;
    sfor<0, SP::NF>([&](auto jc) {
      constexpr int j = decltype(jc)::v;
      constexpr int KK = SP::COL[j] < 0 ? FK_COUNT : SP::KIND[j];
      s_upd<KK, true>(sm + SP::SOFF[j], fe[r], ST, xr[j]);
    });
  }
}

// Register accumulator of the rank front's hottest key (SP::HOTREG, JIT only): that key's rows are
// combined per thread in registers (encoded like the shared table) and flushed once at the end, so
// the key that most often collides with itself inside a warp costs no shared-memory atomics.
template <class SP, int H>
struct HotAccT {
  __device__ __forceinline__ void init(const uint64_t*) {}
};
template <class SP, int H>
struct HotAccT2 {
  uint64_t key[H];
  uint64_t a[H][SP::NF];
  template <int j>
  static constexpr int kind() { return SP::COL[j] < 0 ? FK_COUNT : SP::KIND[j]; }
  __device__ __forceinline__ void init(const uint64_t* hk) {
#pragma unroll
    for (int h = 0; h < H; ++h) {
      key[h] = hk ? __ldg((const unsigned long long*)hk + h) : kEmpty;
      sfor<0, SP::NF>([&](auto jc) {
        constexpr int j = decltype(jc)::v;
        a[h][j] = identity64(kind<j>());
      });
    }
  }
  template <int h, int NV, int R>
  __device__ __forceinline__ void add(const uint64_t (&v)[NV][R], int r) {
    sfor<0, SP::NF>([&](auto jc) {
      constexpr int j = decltype(jc)::v;
      constexpr int K = kind<j>(), c = SP::COL[j];
      uint64_t& acc = a[h][j];
      if constexpr (c < 0) {
        acc += 1;
      } else {
        const uint64_t x = enc<K, true>(v[c][r]);
        if constexpr (K == FK_COUNT || K == FK_SUMI) acc += x;
        else if constexpr (K == FK_SUMF)
          acc = (uint64_t)__double_as_longlong(__longlong_as_double((long long)acc) + __longlong_as_double((long long)x));
        else if constexpr (K == FK_MINI32) acc = (int)x < (int)acc ? (uint64_t)(int64_t)(int)x : acc;
        else if constexpr (K == FK_MAXI32) acc = (int)x > (int)acc ? (uint64_t)(int64_t)(int)x : acc;
        else if constexpr (K == FK_MINI64 || K == FK_MINF64) acc = (long long)x < (long long)acc ? x : acc;
        else acc = (long long)x > (long long)acc ? x : acc;
      }
    });
  }
  // take the rows of the hot keys out of `valid` (their fields go to registers)
  template <int NV, int R>
  __device__ __forceinline__ void take(const uint64_t (&k)[R], uint32_t& valid, const uint64_t (&v)[NV][R]) {
#pragma unroll
    for (int r = 0; r < R; ++r)
      sfor<0, H>([&](auto hc) {  // h a compile-time index: the partials stay in registers
        constexpr int h = decltype(hc)::v;
        if ((valid >> r & 1) && k[r] == key[h]) {
          add<h>(v, r);
          valid &= ~(1u << r);
        }
      });
  }
  // into the key's rank-front entry, or straight into the dense state if the key is not in the front
  __device__ __forceinline__ void flush(const AggParams& p, uint8_t* sm) {
#pragma unroll
    for (int h = 0; h < H; ++h) {
      const uint64_t kh = key[h];
      if (kh == kEmpty || count(h) == 0) continue;
      const uint64_t x = ((const uint64_t*)(sm + p.key_off))[kh >> 5];
      const uint32_t b = (uint32_t)kh & 31u, bits = (uint32_t)x;
      const bool in_front = bits >> b & 1u;
      const uint32_t e = (uint32_t)(x >> 32) + __popc(bits & ((1u << b) - 1u));
      sfor<0, SP::NF>([&](auto jc) {
        constexpr int j = decltype(jc)::v;
        constexpr int K = kind<j>();
        if (in_front) s_upd<K, false>(sm + p.soff[j], e, p.S, a[h][j]);
        else d_upd<K, false>(dense_addr(p, j, kh), a[h][j]);
      });
    }
  }
  // rank-front entry of hot key h, or ~0u (empty key or not in the front)
  __device__ __forceinline__ uint32_t entry(const AggParams& p, const uint8_t* sm, int h) const {
    const uint64_t kh = key[h];
    if (kh == kEmpty) return ~0u;
    const uint64_t x = ((const uint64_t*)(sm + p.key_off))[kh >> 5];
    const uint32_t b = (uint32_t)kh & 31u, bits = (uint32_t)x;
    return (bits >> b & 1u) ? (uint32_t)(x >> 32) + __popc(bits & ((1u << b) - 1u)) : ~0u;
  }
  __device__ __forceinline__ uint64_t count(int h) const {
    uint64_t c = 0;
    sfor<0, SP::NF>([&](auto jc) {
      constexpr int j = decltype(jc)::v;
      if constexpr (kind<j>() == FK_COUNT) c = a[h][j];
    });
    return c;
  }
};
template <class SP> struct HotAccT<SP, 1> : HotAccT2<SP, 1> {};
template <class SP> struct HotAccT<SP, 2> : HotAccT2<SP, 2> {};
template <class SP>
using HotAcc = HotAccT<SP, SP::HOTREG>;

// One tile's rows after loading: hot-key front (rank image or hash table), then the global table
// (path b: convergent probing; b': direct) for the rows the front did not take.
template <class SP, int NV, int R, bool FRONT, bool DIRECT>
__device__ __forceinline__ void process_rows(const AggParams& p, uint8_t* sm, uint64_t (&key)[R], uint32_t valid,
                                             uint64_t (&v)[NV][R], HotAcc<SP>& ha) {
  if constexpr (FRONT && DIRECT && SP::HOTREG != 0) {  // the hottest key: registers (see HotAccT)
    ha.take(key, valid, v);
  }
  const Layout& L = p.lay;
  const uint32_t S = p.S;
  uint8_t* tb = (uint8_t*)p.table;
  uint32_t miss = valid;
  bool deduped = false;
  if constexpr (FRONT && SP::kStatic) {
    if constexpr (SP::DEDUPE) {  // opt-in (BLU_GBY_DEDUPE=1): pays off only for extreme skew
      if (!p.front_rank_words) {
        front_dedupe_rows<SP, NV, R, DIRECT>(p, sm, key, valid, v);
        miss = 0;
        deduped = true;
      }
    }
  }
  if (FRONT && DIRECT && p.front_rank_words && !deduped) {
    // rank front: a dense key k is hot iff bit k%32 of word k/32 is set; its entry is the word's
    // prefix plus the hot keys below it in the word. Converged, one LDS.64 per row, no probe loop.
    const uint64_t* img = (const uint64_t*)(sm + p.key_off);
    uint32_t fe[R];
    uint32_t hit = 0;
#pragma unroll
    for (int r = 0; r < R; ++r) {
      const uint64_t x = (valid >> r & 1) ? img[key[r] >> 5] : 0ull;
      const uint32_t b = (uint32_t)key[r] & 31u, bits = (uint32_t)x;
      fe[r] = (uint32_t)(x >> 32) + __popc(bits & ((1u << b) - 1u));
      hit |= (bits >> b & 1u) << r;
    }
    bool done = false;
    if constexpr (SP::kStatic) {
      if constexpr (SP::DEDUPE) {  // opt-in (BLU_GBY_DEDUPE=1): warp-level combining of equal entries
        rank_dedupe_apply<SP, NV, R>(p, sm, fe, hit, v);
        done = true;
      }
    }
    if (!done) smem_apply_rows<SP, NV, R, mm_front_on<SP>()>(p, sm, fe, hit, v);
    miss = valid & ~hit;
  } else if (FRONT && !deduped) {
    // hot-key front: small open-addressing table per CTA in shared memory
    uint64_t* fk = (uint64_t*)(sm + p.key_off);
    const bool seeded = p.front_seed != nullptr;
    uint32_t fe[R];
    uint32_t hit = 0;
#pragma unroll
    for (int r = 0; r < R; ++r) {
      fe[r] = 0;
      if (!(valid >> r & 1)) continue;
      uint32_t s = front_home(key[r], S);
      if (seeded) {  // read-only front (load <= 1/2): stop at the key or the first empty slot
#pragma unroll 1
        for (int q = 0; q < 8; ++q) {
          const uint64_t cur = fk[s];
          if (cur == key[r]) { hit |= 1u << r; break; }
          if (cur == kEmpty) break;
          s = (s + 1) & (S - 1);
        }
      } else {
#pragma unroll 1
        for (int q = 0; q < 8; ++q) {
          uint64_t cur = *(volatile uint64_t*)(fk + s);
          if (cur == key[r]) { hit |= 1u << r; break; }
          if (cur == kEmpty) {
            unsigned long long old = atomicCAS((unsigned long long*)(fk + s), (unsigned long long)kEmpty,
                                               (unsigned long long)key[r]);
            if (old == kEmpty || old == key[r]) { hit |= 1u << r; break; }
          }
          s = (s + 1) & (S - 1);
        }
      }
      fe[r] = s;
    }
    __syncwarp();  // reconverge after the data-dependent probe loops (independent thread scheduling)
    smem_apply_rows<SP, NV, R>(p, sm, fe, hit, v);
    miss = valid & ~hit;
  }
  uint64_t slot[R];
  if (DIRECT) {
#pragma unroll
    for (int r = 0; r < R; ++r) slot[r] = key[r];
  } else {
    // Convergent multi-row probe: every pending row of the lane advances one slot per iteration
    // and all their key loads are issued together (memory-level parallelism); the warp stays
    // converged (__any_sync), so the REDs that follow are warp-wide.
    uint64_t cur[R];
#pragma unroll
    for (int r = 0; r < R; ++r) {
      slot[r] = fmix64(key[r]) & p.cap_mask;
      cur[r] = (miss >> r & 1) ? __ldcg((const unsigned long long*)(tb + slot[r] * L.slot_bytes)) : 0ull;
    }
    uint32_t pending = miss;
    for (uint32_t it = 0;; ++it) {
#pragma unroll
      for (int r = 0; r < R; ++r) {
        if (!(pending >> r & 1)) continue;
        if (cur[r] == key[r]) {
          pending &= ~(1u << r);
        } else {
          if (cur[r] == kEmpty) {
            unsigned long long old = atomicCAS((unsigned long long*)(tb + slot[r] * L.slot_bytes),
                                               (unsigned long long)kEmpty, (unsigned long long)key[r]);
            if (old == kEmpty || old == key[r]) {
              pending &= ~(1u << r);
              continue;
            }
          }
          slot[r] = (slot[r] + 1) & p.cap_mask;
        }
      }
      if (!__any_sync(0xffffffffu, pending)) break;
      if (it + 1 >= 4) {
        // long tails (a few rows per warp): finish them one lane at a time, then reconverge
#pragma unroll
        for (int r = 0; r < R; ++r) {
          if (!(pending >> r & 1)) continue;
          uint64_t sl;
          const uint64_t c = __ldcg((const unsigned long long*)(tb + slot[r] * L.slot_bytes));
          if (hash_locate(tb, p.cap_mask, L.slot_bytes, key[r], c, slot[r], p.max_probe, sl)) {
            slot[r] = sl;
          } else {  // the estimate was too small: flag, regrow, rerun
            miss &= ~(1u << r);
            atomicOr(p.flags, FLAG_OVERFLOW);
          }
        }
        break;
      }
#pragma unroll
      for (int r = 0; r < R; ++r)
        if (pending >> r & 1) cur[r] = __ldcg((const unsigned long long*)(tb + slot[r] * L.slot_bytes));
    }
    __syncwarp();  // reconverge before the field reductions so each RED instruction is warp-wide
  }
  if (!DIRECT && L.lock_off) global_apply_rows_locked<SP, NV, R>(p, slot, miss, v);  // kernel 3
  else global_apply_rows<SP, NV, R, DIRECT>(p, slot, miss, v);
}

// MODE 0: rows from columns; 1: records (merge of exchanged partials); 2: segments (pass 2 of the
// partitioned mode: tiles enumerate the buckets in order, so at any moment all CTAs work inside
// one bucket whose slice of the table is L2-resident).
template <class SP, int NV, int R, bool FRONT, bool DIRECT, int MODE>
__device__ __forceinline__ void global_body(const AggParams& p, const RecSrc& rs) {
  extern __shared__ __align__(16) uint8_t sm[];
  constexpr bool RECORDS = MODE == 1;
  // MODE 3: rows from columns, MODE 4: segments, both software-pipelined (JIT only, see RawTile)
  constexpr bool SEG = MODE == 2 || MODE == 4;
  if (p.gate && ((*(volatile const uint32_t*)p.gate != 0) != (p.gate_run_if != 0))) return;
  const Layout& L = p.lay;
  const uint32_t S = p.S;
  __shared__ uint64_t tpre[SEG ? kMaxSegs + 1 : 1];  // the planner keeps n_segs <= kMaxSegs in this mode
  __shared__ uint64_t tend[MODE == 4 ? kMaxSegs : 1];  // MODE 4: end row of each segment
  if constexpr (SEG) {  // warp-tile prefix over the buckets (warp 0)
    if (threadIdx.x < 32) {
      const uint64_t tile = 32ull * R;
      uint64_t carry = 0;
      for (uint32_t b0 = 0; b0 < p.n_segs; b0 += 32) {
        uint32_t b = b0 + threadIdx.x;
        uint64_t x = b < p.n_segs ? (p.seg_count[b] + tile - 1) / tile : 0, inc = x;
        for (int o = 1; o < 32; o <<= 1) {
          uint64_t y = __shfl_up_sync(0xffffffffu, inc, o);
          if ((int)threadIdx.x >= o) inc += y;
        }
        if (b < p.n_segs) tpre[b] = carry + inc - x;
        if (MODE == 4 && b < p.n_segs) tend[b] = (uint64_t)b * p.seg_stride + p.seg_count[b];
        carry += __shfl_sync(0xffffffffu, inc, 31);
      }
      if (threadIdx.x == 0) tpre[p.n_segs] = carry;
    }
    __syncthreads();
  }
  if (FRONT) {
    const uint64_t* seed = p.front_seed;
    for (uint32_t e = threadIdx.x; e < S; e += blockDim.x)
      ((uint64_t*)(sm + p.key_off))[e] = seed ? __ldg((const unsigned long long*)seed + e) : kEmpty;
    for (int j = 0; j < L.n_fields; ++j)
      for (uint32_t e = threadIdx.x; e < S; e += blockDim.x) smem_init_entry(sm + p.soff[j], L.f[j].kind, e, S);
    mm_init<SP, FRONT && DIRECT && mm_front_on<SP>()>();
    __syncthreads();
  }
  HotAcc<SP> ha;
  ha.init(FRONT && DIRECT && p.front_rank_words ? p.hot_key : nullptr);
  // rank front: every warp refreshes the MIN/MAX skip bounds over its slice of the hot entries (the
  // register-held hottest keys' entries excluded: their rows never reach the table before the flush)
  uint32_t mm_it = 0;
  auto mm_front = [&]() {
    if constexpr (FRONT && DIRECT) {
      if constexpr (mm_front_on<SP>()) {
#ifndef BLU_MM_NOREFRESH
        if (p.front_rank_words && ++mm_it % kMMRefresh == 0) {
#else
        if (false) {
#endif
          const uint64_t xl = ((const uint64_t*)(sm + p.key_off))[p.front_rank_words - 1];
          const uint32_t nh = (uint32_t)(xl >> 32) + __popc((uint32_t)xl);
          uint32_t s0 = ~0u, s1 = ~0u;
          if constexpr (SP::HOTREG >= 1) s0 = ha.entry(p, sm, 0);
          if constexpr (SP::HOTREG >= 2) s1 = ha.entry(p, sm, 1);
          mm_refresh<SP>(sm, nh, s0, s1);
        }
      }
    }
  };
  const uint64_t pol = evict_first_policy();
  // SEG: warp tiles (32*R rows) handed out in bucket order by a global counter, so every warp of
  // the grid stays inside the same one or two buckets (their table slices L2-resident); static
  // grid-stride assignment lets CTAs drift several buckets apart and thrash L2.
  const uint64_t tile = SEG ? 32ull * R : (uint64_t)blockDim.x * R;
  const uint64_t ntiles = SEG ? tpre[p.n_segs] : (p.n_rows + tile - 1) / tile;
  const unsigned lane = threadIdx.x & 31;
  uint8_t* tb = (uint8_t*)p.table;
  uint32_t flag_seen = 0;
  // SEG: a warp claims kGrab consecutive warp tiles per atomic (one counter for the whole grid). The
  // rows in flight span (warps x kGrab x tile) rows in bucket order, i.e. that fraction of the table
  // (p.grab, 0 = 16; 1-4 keep C5's table window in L2 but measured no faster)
  const uint32_t kGrab = p.grab ? p.grab : 16u;
  uint64_t t = blockIdx.x, chunk = 0, chunk_next = 0;
  uint32_t k_in = 0;
  const bool dyn = SEG && p.tile_ctr != nullptr;
  if (SEG && !dyn) t = (uint64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);  // static warp tiles
  if (dyn) {
    chunk = lane == 0 ? atomicAdd((unsigned long long*)p.tile_ctr, 1ull) : 0ull;
    chunk = __shfl_sync(0xffffffffu, chunk, 0);
    chunk_next = lane == 0 ? atomicAdd((unsigned long long*)p.tile_ctr, 1ull) : 0ull;  // prefetched
    t = chunk * kGrab;
  }
  // SEG with p.prefetch: lane 0 has the warp's next claimed chunk; its rows (within their bucket)
  // go DRAM -> L2 by the TMA unit while the current chunk is worked on (BLU_GBY_SEG_PF)
  auto seg_prefetch = [&](uint64_t cn) {
    if constexpr (SEG && SP::kStatic) {
      if (p.prefetch && lane == 0 && cn * kGrab < ntiles) {
        const uint64_t tt = cn * kGrab;
        uint32_t lo = 0, hi = p.n_segs - 1;
        while (lo < hi) {
          const uint32_t mid = (lo + hi + 1) >> 1;
          if (tpre[mid] <= tt) lo = mid; else hi = mid - 1;
        }
        const uint64_t a = (uint64_t)lo * p.seg_stride + (tt - tpre[lo]) * tile;
        const uint64_t end = (uint64_t)lo * p.seg_stride + p.seg_count[lo];
        bulk_prefetch_rows_l2<SP>(p, a, a + (uint64_t)kGrab * tile < end ? a + (uint64_t)kGrab * tile : end);
      }
    }
  };
  if (dyn) seg_prefetch(chunk_next);
  if constexpr (MODE == 3) {  // software-pipelined row stream (see RawTile)
    const uint64_t n = p.n_rows;
    const unsigned warp = threadIdx.x >> 5;
    RawTile<SP, R> A, B;
    if (t < ntiles) tile_load<SP, R>(p, lane_base<R>(t * tile, warp, lane), n, pol, A);
    while (t < ntiles) {
      const uint64_t tn = t + gridDim.x;
      const uint32_t fl = *(volatile uint32_t*)p.flags;  // consumed after the tile: off the critical path
      if (tn < ntiles) tile_load<SP, R>(p, lane_base<R>(tn * tile, warp, lane), n, pol, B);
      uint64_t key[R];
      uint64_t v[NV][R];
      const uint32_t valid = tile_unpack<SP, NV, R>(p, A, lane_base<R>(t * tile, warp, lane), n, key, v);
      process_rows<SP, NV, R, FRONT, DIRECT>(p, sm, key, valid, v, ha);
      mm_front();
      if (__any_sync(0xffffffffu, fl)) break;  // warp-uniform abort
      A = B;
      t = tn;
    }
  }
  if constexpr (MODE == 4) {  // segments, software-pipelined: tile coordinates from shared memory
    auto coords = [&](uint64_t tt, uint64_t& lb, uint64_t& nn) {
      uint32_t lo = 0, hi = p.n_segs - 1;
      while (lo < hi) {
        const uint32_t mid = (lo + hi + 1) >> 1;
        if (tpre[mid] <= tt) lo = mid; else hi = mid - 1;
      }
      lb = lane_base<R>((uint64_t)lo * p.seg_stride + (tt - tpre[lo]) * tile, 0, lane);
      nn = tend[lo];
    };
    RawTile<SP, R> A, B;
    uint64_t lbA = 0, nA = 0, lbB = 0, nB = 0;
    if (t < ntiles) {
      coords(t, lbA, nA);
      tile_load<SP, R>(p, lbA, nA, pol, A);
    }
    while (t < ntiles) {
      uint64_t t_next;
      if (!dyn) {
        t_next = t + (uint64_t)gridDim.x * (blockDim.x >> 5);
      } else if (++k_in < kGrab) {
        t_next = t + 1;
      } else {
        k_in = 0;
        chunk = __shfl_sync(0xffffffffu, chunk_next, 0);
        t_next = chunk * kGrab;
        chunk_next = lane == 0 ? atomicAdd((unsigned long long*)p.tile_ctr, 1ull) : 0ull;
        seg_prefetch(chunk_next);
      }
      const uint32_t fl = *(volatile uint32_t*)p.flags;
      if (t_next < ntiles) {
        coords(t_next, lbB, nB);
        tile_load<SP, R>(p, lbB, nB, pol, B);
      }
      uint64_t key[R];
      uint64_t v[NV][R];
      const uint32_t valid = tile_unpack<SP, NV, R>(p, A, lbA, nA, key, v);
      process_rows<SP, NV, R, FRONT, DIRECT>(p, sm, key, valid, v, ha);
      if (__any_sync(0xffffffffu, fl)) break;
      A = B;
      lbA = lbB;
      nA = nB;
      t = t_next;
    }
  }
  while (MODE != 3 && MODE != 4 && t < ntiles) {
    if (flag_seen) break;
    flag_seen = __any_sync(0xffffffffu, *(volatile uint32_t*)p.flags);  // warp-uniform abort
    uint64_t n = p.n_rows, row0 = t * tile, t_next = t + gridDim.x;
    uint64_t row;
    if constexpr (SEG) {  // bucket of warp tile t: largest b with tpre[b] <= t
      if (!dyn) {
        t_next = t + (uint64_t)gridDim.x * (blockDim.x >> 5);
      } else if (++k_in < kGrab) {
        t_next = t + 1;
      } else {
        k_in = 0;
        chunk = __shfl_sync(0xffffffffu, chunk_next, 0);
        t_next = chunk * kGrab;
        chunk_next = lane == 0 ? atomicAdd((unsigned long long*)p.tile_ctr, 1ull) : 0ull;
        seg_prefetch(chunk_next);
      }
      uint32_t lo = 0, hi = p.n_segs - 1;
      while (lo < hi) {
        uint32_t mid = (lo + hi + 1) >> 1;
        if (tpre[mid] <= t) lo = mid; else hi = mid - 1;
      }
      row0 = (uint64_t)lo * p.seg_stride + (t - tpre[lo]) * tile;
      n = (uint64_t)lo * p.seg_stride + p.seg_count[lo];
      row = lane_base<R>(row0, 0, lane);
    } else {
      row = lane_base<R>(row0, threadIdx.x >> 5, lane);
    }
    uint64_t key[R];
    uint64_t v[NV][R];
    uint32_t valid;
    if (RECORDS) {
      valid = 0;
#pragma unroll
      for (int r = 0; r < R; ++r) {
        key[r] = 0;
#pragma unroll
        for (int c = 0; c < NV; ++c) v[c][r] = 0;
        const uint64_t rr = row_of<R>(row, r);
        if (rr >= n) continue;
        const uint64_t* rec = rs.rec + rr * rs.words;
        key[r] = __ldg((const unsigned long long*)rec);
        valid |= 1u << r;
#pragma unroll
        for (int c = 0; c < NV; ++c)
          if (c < L.n_vals) {
            uint64_t w = __ldg((const unsigned long long*)rec + 1 + c);
            v[c][r] = L.val_dtype[c] == BLU_I32 ? (uint64_t)(int64_t)(int32_t)(uint32_t)w : w;
          }
      }
    } else {
      if (!SEG && p.prefetch)  // the warp's next tile: in flight in L2 while this one is worked on
        prefetch_warp_rows_l2<SP>(p, t_next * tile + (uint64_t)(threadIdx.x >> 5) * 32 * R, 32ull * R, n, lane);
      valid = pack_keys<SP, R>(p, row, n, pol, key);
      load_vals<SP, NV, R>(p, row, n, pol, v);
    }
    process_rows<SP, NV, R, FRONT, DIRECT>(p, sm, key, valid, v, ha);
    mm_front();
    t = t_next;
  }
  if constexpr (FRONT && DIRECT && SP::HOTREG != 0) ha.flush(p, sm);
  if (FRONT) {
    // merge the front into the global table
    __syncthreads();
    const uint64_t* fk = (const uint64_t*)(sm + p.key_off);
    const int cf = L.count_field;
    if (DIRECT && p.front_rank_words) {  // rank front: entry prefix + j holds key 32w + (j-th set bit)
      for (uint32_t w = threadIdx.x; w < p.front_rank_words; w += blockDim.x) {
        const uint64_t x = fk[w];
        uint32_t bits = (uint32_t)x, e = (uint32_t)(x >> 32);
        for (; bits; bits &= bits - 1, ++e) {
          if (s_read<FK_COUNT>(sm + p.soff[cf], e, S) == 0) continue;
          const uint64_t g = (uint64_t)w * 32 + (uint64_t)(__ffs(bits) - 1);
          for (int j = 0; j < L.n_fields; ++j) {
            const uint8_t* b = sm + p.soff[j];
            dispatch_kind(L.f[j].kind, [&](auto kc) {
              constexpr int K = decltype(kc)::v;
              d_upd<K, false>(dense_addr(p, j, g), s_read<K>(b, e, S));
            });
          }
        }
      }
      return;
    }
    for (uint32_t e = threadIdx.x; e < S; e += blockDim.x) {
      const uint64_t key = fk[e];
      if (key == kEmpty) continue;
      if (p.front_seed && s_read<FK_COUNT>(sm + p.soff[cf], e, S) == 0) continue;  // seeded, no rows here
      uint64_t s = key;
      if (!DIRECT) {
        uint64_t idx = fmix64(key) & p.cap_mask;
        uint64_t first = __ldcg((const unsigned long long*)(tb + idx * L.slot_bytes));
        if (!hash_locate(tb, p.cap_mask, L.slot_bytes, key, first, idx, p.max_probe, s)) {
          atomicOr(p.flags, FLAG_OVERFLOW);
          continue;
        }
      }
      for (int j = 0; j < L.n_fields; ++j) {
        const uint8_t* b = sm + p.soff[j];
        dispatch_kind(L.f[j].kind, [&](auto kc) {
          constexpr int K = decltype(kc)::v;
          if (DIRECT) d_upd<K, false>(dense_addr(p, j, s), s_read<K>(b, e, S));
          else g_upd<K, false>(tb + s * L.slot_bytes + L.f[j].goff, s_read<K>(b, e, S));
        });
      }
    }
  }
}

// ------------------------------------------------------------------------------------------------
// Partitioned path (b), pass 2 with bucket-local shared-memory tables. After the scatter, the rows
// of bucket b hold exactly the groups whose slot lies in slice b of the global table, and no other
// bucket holds any of them. So a CTA can aggregate a piece of one bucket in an open-addressing table
// of its own shared memory (the paper's shared-memory kernel, applied per bucket instead
// of per query) and merge it into the global table once per piece ("merged"): one CAS + one
// RED per field per GROUP and piece instead of per ROW. Rows whose key finds no room within
// kBucketProbe slots (a bucket with more groups than the table holds) take the global path.
// Work items = (bucket, piece) handed out in bucket order by one global counter. p.S = table
// entries (any multiple of 16), p.lay = the records' layout (packed u64 key, value columns).
// ------------------------------------------------------------------------------------------------
constexpr uint32_t kBucketProbe = 32;

// The table is 4-way bucketed: entries [4h, 4h + 4) form bucket h; a key's home bucket comes from the
// high half of a second hash (independent of the slot bits that chose the partition). One probe step
// reads the bucket's four keys with two 16-byte loads, so at the table's load (<= 0.7) almost every
// row resolves in the first step (linear probing by single entries needed ~14 convergent steps per
// warp tile at load 0.6: the longest of 128 probe sequences).
__device__ __forceinline__ uint32_t bucket_home(uint64_t key, uint32_t nbk) {
  return (uint32_t)(((fmix64(key ^ 0x2545F4914F6CDD1Dull) >> 32) * (uint64_t)nbk) >> 32);
}

__device__ __forceinline__ void lds_v2_volatile(const uint64_t* p, uint64_t& a, uint64_t& b) {
  const uint32_t s = (uint32_t)__cvta_generic_to_shared(p);
  asm volatile("ld.volatile.shared.v2.u64 {%0, %1}, [%2];" : "=l"(a), "=l"(b) : "r"(s));
}

// Merge entry e of the shared table into the global table, then reset it to the mask.
__device__ __forceinline__ void bucket_flush_entry(const AggParams& p, uint8_t* sm, uint32_t e) {
  const Layout& L = p.lay;
  const uint32_t S = p.S;
  uint64_t* fk = (uint64_t*)(sm + p.key_off);
  const uint64_t key = fk[e];
  if (key == kEmpty) return;
  uint8_t* tb = (uint8_t*)p.table;
  const uint64_t idx = fmix64(key) & p.cap_mask;
  uint64_t s;
  const bool ok = hash_locate(tb, p.cap_mask, L.slot_bytes, key, __ldcg((const unsigned long long*)(tb + idx * L.slot_bytes)),
                              idx, p.max_probe, s);
  if (!ok) atomicOr(p.flags, FLAG_OVERFLOW);
  for (int j = 0; j < L.n_fields; ++j) {
    uint8_t* b = sm + p.soff[j];
    const int kind = L.f[j].kind;
    if (ok)
      dispatch_kind(kind, [&](auto kc) {
        constexpr int K = decltype(kc)::v;
        g_upd<K, false>(tb + s * L.slot_bytes + L.f[j].goff, s_read<K>(b, e, S));
      });
    smem_init_entry(b, kind, e, S);
  }
  fk[e] = kEmpty;
}

template <class SP, int NV, int R, bool PIPE = false>
__device__ __forceinline__ void bucket_body(const AggParams& p) {
  extern __shared__ __align__(16) uint8_t sm[];
  if (p.gate && ((*(volatile const uint32_t*)p.gate != 0) != (p.gate_run_if != 0))) return;
  const Layout& L = p.lay;
  const uint32_t S = p.S;
  const uint32_t nb = p.n_segs;
  // piece_rows 0: one work item per bucket, no prefix (aux = 2 scalars); else pieces of piece_rows rows
  // with the buckets' piece prefix (nb + 1 u32) ahead of the 2 scalars
  const bool whole = p.piece_rows == 0;
  uint32_t* ppre = (uint32_t*)(sm + p.aux_off);
  volatile uint32_t* s_item = whole ? ppre : ppre + nb + 1;
  uint64_t* fk = (uint64_t*)(sm + p.key_off);
  const uint64_t piece = whole ? ~0ull : p.piece_rows;
  // piece prefix over the buckets (warp 0) and the table mask (all threads)
  if (!whole && threadIdx.x < 32) {
    uint32_t carry = 0;
    for (uint32_t b0 = 0; b0 < nb; b0 += 32) {
      const uint32_t b = b0 + threadIdx.x;
      const uint32_t x = b < nb ? (uint32_t)((p.seg_count[b] + piece - 1) / piece) : 0u;
      uint32_t inc = x;
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
        if ((int)threadIdx.x >= o) inc += y;
      }
      if (b < nb) ppre[b] = carry + inc - x;
      carry += __shfl_sync(0xffffffffu, inc, 31);
    }
    if (threadIdx.x == 0) ppre[nb] = carry;
  }
  for (uint32_t e = threadIdx.x; e < S; e += blockDim.x) fk[e] = kEmpty;
  for (int j = 0; j < L.n_fields; ++j)
    for (uint32_t e = threadIdx.x; e < S; e += blockDim.x) smem_init_entry(sm + p.soff[j], L.f[j].kind, e, S);
  const uint64_t pol = evict_first_policy();
  const uint64_t tile = (uint64_t)blockDim.x * R;
  const unsigned lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint8_t* tb = (uint8_t*)p.table;
  for (;;) {
    __syncthreads();  // prefix ready / previous piece flushed and the table reset
    if (threadIdx.x == 0) {
      s_item[0] = (uint32_t)atomicAdd((unsigned long long*)p.tile_ctr, 1ull);
      s_item[1] = *(volatile uint32_t*)p.flags;
    }
    __syncthreads();
    const uint32_t item = s_item[0];
    if (item >= (whole ? nb : ppre[nb]) || (s_item[1] & FLAG_OVERFLOW)) break;
    uint32_t lo = whole ? item : 0, hi = whole ? item : nb - 1;  // bucket of the item: largest b with ppre[b] <= item
    while (lo < hi) {
      const uint32_t mid = (lo + hi + 1) >> 1;
      if (ppre[mid] <= item) lo = mid; else hi = mid - 1;
    }
    const uint64_t seg0 = (uint64_t)lo * p.seg_stride;
    const uint64_t cnt = p.seg_count[lo];
    const uint64_t k = whole ? 0 : (uint64_t)(item - ppre[lo]);  // piece of the bucket
    const uint64_t r0 = seg0 + k * (whole ? 0 : piece);
    const uint64_t r1 = whole ? seg0 + cnt : seg0 + (k * piece + piece < cnt ? k * piece + piece : cnt);
#ifdef BLU_DEBUG_BOUNDS
    if (threadIdx.x == 0 && (lo >= nb || r1 > seg0 + p.seg_stride || r0 > r1))
      printf("BOUNDS item %u lo %u nb %u r0 %llu r1 %llu seg0 %llu stride %llu cnt %llu piece %llu\n", item, lo, nb,
             (unsigned long long)r0, (unsigned long long)r1, (unsigned long long)seg0, (unsigned long long)p.seg_stride,
             (unsigned long long)cnt, (unsigned long long)piece);
#endif
    // PIPE (NVRTC kernels): the piece's next tile is loaded into registers before this one is probed
    using Raw = RawTileFor<SP, R, PIPE>;
    Raw A, Bt;
    if constexpr (PIPE)
      if (r0 < r1) tile_load<SP, R>(p, lane_base<R>(r0, warp, lane), r1, pol, A);
    for (uint64_t row0 = r0; row0 < r1; row0 += tile) {
      const uint64_t row = lane_base<R>(row0, warp, lane);
      if constexpr (SP::kStatic) {
        if (p.prefetch && threadIdx.x == 0) {  // the tile p.prefetch tiles ahead: DRAM -> L2 by the TMA unit
          const uint64_t a = row0 + (uint64_t)p.prefetch * tile;
          if (a < r1) {
            const uint64_t m = r1 - a < tile ? r1 - a : tile;
            bulk_prefetch_l2((const uint64_t*)p.key[0] + a, m * 8);
            sfor<0, SP::NV>([&](auto cc) {
              constexpr int c = decltype(cc)::v;
              constexpr uint64_t w = SP::VDT[c] == BLU_I32 ? 4 : 8;
              bulk_prefetch_l2((const uint8_t*)p.val[c] + a * w, m * w);
            });
          }
        }
      }
      uint64_t key[R];
      uint64_t v[NV][R];
      uint32_t valid;
      if constexpr (PIPE) {
        if (row0 + tile < r1) tile_load<SP, R>(p, lane_base<R>(row0 + tile, warp, lane), r1, pol, Bt);
        valid = tile_unpack<SP, NV, R>(p, A, row, r1, key, v);
        A = Bt;
      } else {
        valid = pack_keys<SP, R>(p, row, r1, pol, key);
        load_vals<SP, NV, R>(p, row, r1, pol, v);
      }
      // convergent probe of the shared table: every pending row inspects one 4-entry bucket per step
      const uint32_t nbk = S >> 2;
      uint32_t e[R], h[R];
#pragma unroll
      for (int r = 0; r < R; ++r) {
        h[r] = bucket_home(key[r], nbk);
        e[r] = 0;
      }
      uint32_t pending = valid, hit = 0;
      for (uint32_t it = 0; it < kBucketProbe; ++it) {
#pragma unroll
        for (int r = 0; r < R; ++r) {
          if (!(pending >> r & 1)) continue;
          const uint64_t* q = fk + 4 * h[r];
          uint64_t k0, k1, k2, k3;
          lds_v2_volatile(q, k0, k1);
          lds_v2_volatile(q + 2, k2, k3);
          const uint64_t kk = key[r];
          int m = k0 == kk ? 0 : k1 == kk ? 1 : k2 == kk ? 2 : k3 == kk ? 3 : -1;
          if (m < 0) {
            const int z = k0 == kEmpty ? 0 : k1 == kEmpty ? 1 : k2 == kEmpty ? 2 : k3 == kEmpty ? 3 : -1;
            if (z >= 0) {  // claim the first empty entry; on a lost race re-read this bucket next step
              const unsigned long long old = atomicCAS((unsigned long long*)(q + z), (unsigned long long)kEmpty,
                                                       (unsigned long long)kk);
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
        if (!__any_sync(0xffffffffu, pending)) break;
      }
      __syncwarp();
#ifdef BLU_DEBUG_BOUNDS
      for (int r = 0; r < R; ++r)
        if ((hit >> r & 1) && e[r] >= S) printf("BOUNDS e %u S %u\n", e[r], S);
#endif
      smem_apply_rows<SP, NV, R>(p, sm, e, hit, v);
      if (__any_sync(0xffffffffu, pending)) {  // no room in the shared table: global table (S5b)
        uint64_t slot[R];
        uint32_t miss = pending;
#pragma unroll
        for (int r = 0; r < R; ++r) {
          slot[r] = 0;
          if (!(miss >> r & 1)) continue;
          const uint64_t idx = fmix64(key[r]) & p.cap_mask;
          if (!hash_locate(tb, p.cap_mask, L.slot_bytes, key[r], __ldcg((const unsigned long long*)(tb + idx * L.slot_bytes)),
                           idx, p.max_probe, slot[r])) {
            miss &= ~(1u << r);
            atomicOr(p.flags, FLAG_OVERFLOW);
          }
        }
        __syncwarp();
#ifdef BLU_DEBUG_BOUNDS
        for (int r = 0; r < R; ++r)
          if ((miss >> r & 1) && slot[r] > p.cap_mask) printf("BOUNDS slot %llu mask %llu\n", (unsigned long long)slot[r], (unsigned long long)p.cap_mask);
#endif
        global_apply_rows<SP, NV, R, false>(p, slot, miss, v);
      }
    }
    __syncthreads();  // every row of the piece applied
    for (uint32_t x = threadIdx.x; x < S; x += blockDim.x) bucket_flush_entry(p, sm, x);
  }
}

// ------------------------------------------------------------------------------------------------
// Partitioned path (b), pass 1: radix scatter of rows into B buckets by the top bits of their slot.
// Per tile: shared-memory counting sort by bucket, one global cursor reservation per (tile,
// bucket), then coalesced writes of each bucket's contiguous segment (packed u64 key + values).
// ------------------------------------------------------------------------------------------------
__device__ __forceinline__ void block_excl_scan(uint32_t* a, uint32_t* out, uint32_t B, uint32_t* warp_tot,
                                                uint32_t* total) {
  // exclusive scan of a[0..B) into out (B <= 4 * blockDim.x; blockDim.x a multiple of 32, <= 1024):
  // thread t owns the C consecutive elements [C*t, C*t + C)
  const unsigned t = threadIdx.x, lane = t & 31, w = t >> 5, nw = blockDim.x >> 5;
  const uint32_t C = (B + blockDim.x - 1) / blockDim.x;
  uint32_t x[4], sum = 0;
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const uint32_t k = C * t + i;
    x[i] = (i < (int)C && k < B) ? a[k] : 0u;
    sum += x[i];
  }
  uint32_t inc = sum;
  for (int o = 1; o < 32; o <<= 1) {
    uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
    if ((int)lane >= o) inc += y;
  }
  if (lane == 31) warp_tot[w] = inc;
  __syncthreads();
  if (w == 0) {
    uint32_t v = lane < nw ? warp_tot[lane] : 0, vi = v;
    for (int o = 1; o < 32; o <<= 1) {
      uint32_t y = __shfl_up_sync(0xffffffffu, vi, o);
      if ((int)lane >= o) vi += y;
    }
    if (lane < nw) warp_tot[lane] = vi - v;
    if (lane == 31) *total = vi;
  }
  __syncthreads();
  uint32_t excl = warp_tot[w] + inc - sum;
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const uint32_t k = C * t + i;
    if (i < (int)C && k < B) out[k] = excl;
    excl += x[i];
  }
}

constexpr uint32_t kMaxInSeg = 256;  // first-level buckets of a two-level scatter (32 or 128)

// PIPE (NVRTC kernels only): the next tile's rows are loaded into registers as soon as the current
// tile is staged in shared memory, so those HBM reads are in flight during its write-out phase.
template <class SP, int NV, int R, bool PIPE = false, bool SEGIN = false, bool TMAS = false>
__device__ __forceinline__ void scatter_body(const AggParams& p, const ScatterParams& sp) {
  extern __shared__ __align__(16) uint8_t sm[];
  // second scatter level: skipped once the first level overflowed a bucket (the chunk then takes the
  // gated one-pass fallback; an overflowed bucket's region may hold unwritten rows)
  if (p.gate && ((*(volatile const uint32_t*)p.gate != 0) != (p.gate_run_if != 0))) return;
  const Layout& L = p.lay;
  // histogram bins: the buckets one tile can reach (segmented input: the B2 buckets of its first-level
  // bucket, global index bbase + local bin)
  const uint32_t B = SEGIN ? sp.in_B2 : sp.B;
  const uint32_t TILE = blockDim.x * R;
  // staging stride: TMAS pads every bucket's run to an even length, up to B rows more than the tile
  const uint32_t TS = TMAS ? TILE + ((B + 1u) & ~1u) : TILE;
  uint64_t* skey = (uint64_t*)sm;                       // TS
  uint64_t* sval = skey + TS;                           // NV x TS
  uint64_t* gpos = sval + (size_t)NV * TS;              // B
  uint32_t* histbuf = (uint32_t*)(gpos + B);            // 2 x B: tiles alternate (zeroed one tile ahead)
  uint32_t* lstart = histbuf + 2 * B;                   // B
  uint32_t* wtot = lstart + B;                          // 32
  uint32_t* total = wtot + 32;                          // 1
  uint16_t* sbid = (uint16_t*)(total + 4);              // TILE
  uint32_t* hcnt = (uint32_t*)(sbid + TILE);            // B (TMAS: rows per bucket before padding)
  const uint64_t pol = evict_first_policy();
  const uint64_t n = p.n_rows;
  const uint64_t ntiles = (n + TILE - 1) / TILE;
  // segmented input (second scatter level): rows [s * in_seg, s * in_seg + in_count[s]) of every
  // first-level bucket s; in_seg is a multiple of TILE, so a tile lies in one bucket
  __shared__ uint64_t seg_end[SEGIN ? kMaxInSeg : 1];  // end row of each first-level bucket
  if constexpr (SEGIN) {
    const uint32_t nseg = (uint32_t)((n + sp.in_seg - 1) / sp.in_seg);
    for (uint32_t s0 = threadIdx.x; s0 < nseg && s0 < kMaxInSeg; s0 += blockDim.x) {
      const uint64_t c = sp.in_count[s0];
      seg_end[s0] = s0 * sp.in_seg + (c < sp.in_seg ? c : sp.in_seg);
    }
    __syncthreads();
  }
  auto tile_lim = [&](uint64_t t) -> uint64_t {
    if constexpr (SEGIN) return seg_end[(t * TILE) / sp.in_seg];
    return n;
  };
  for (uint32_t b = threadIdx.x; b < 2 * B; b += blockDim.x) histbuf[b] = 0;
  __syncthreads();
  uint32_t kt = 0;  // tiles processed by this CTA (selects the histogram buffer)
  using Raw = RawTileFor<SP, R, PIPE>;
  Raw T;
  if constexpr (PIPE)
    if (blockIdx.x < ntiles)
      tile_load<SP, R>(p, lane_base<R>(blockIdx.x * TILE, threadIdx.x >> 5, threadIdx.x & 31), tile_lim(blockIdx.x), pol, T);
  for (uint64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
    const uint64_t lim = tile_lim(t);
    if (SEGIN && lim <= t * TILE) {  // past its first-level bucket's rows (the segment's slack)
      if constexpr (PIPE) {
        const uint64_t tn = t + gridDim.x;
        if (tn < ntiles) tile_load<SP, R>(p, lane_base<R>(tn * TILE, threadIdx.x >> 5, threadIdx.x & 31), tile_lim(tn), pol, T);
      }
      continue;
    }
    // No barrier at the top of a tile: the previous tile's readers of the staging, lstart and gpos are
    // ordered before this tile's writers by the barrier after the rank atomics below, and this tile's
    // histogram buffer was zeroed during the previous tile.
    uint32_t* hist = histbuf + (kt & 1u) * B;
    uint32_t* hnext = histbuf + ((kt + 1u) & 1u) * B;
    ++kt;
    const uint64_t row = lane_base<R>(t * TILE, threadIdx.x >> 5, threadIdx.x & 31);
    const uint32_t bbase = SEGIN ? (uint32_t)((t * TILE) / sp.in_seg) * sp.in_B2 : 0u;
    uint64_t key[R];
    uint64_t v[NV][R];
    uint32_t valid;
    if constexpr (PIPE) {
      valid = tile_unpack<SP, NV, R>(p, T, row, lim, key, v);
    } else {
      valid = pack_keys<SP, R>(p, row, lim, pol, key);
      load_vals<SP, NV, R>(p, row, lim, pol, v);
    }
    if (!PIPE && p.prefetch) {  // a later tile of this CTA: in flight during the sort and the writes below
      const uint64_t nt = t + (uint64_t)gridDim.x * p.prefetch;
      prefetch_rows_l2<SP>(p, nt * TILE, nt * TILE + TILE < n ? nt * TILE + TILE : n);
    }
    if (PIPE && p.prefetch > 1 && threadIdx.x == 0) {  // beyond the register-pipelined next tile: TMA L2 prefetch
      const uint64_t nt = t + (uint64_t)gridDim.x * p.prefetch;
      if (nt < ntiles) {
        const uint64_t lim2 = tile_lim(nt);
        bulk_prefetch_rows_l2<SP>(p, nt * TILE, nt * TILE + TILE < lim2 ? nt * TILE + TILE : lim2);
      }
    }
    uint32_t bb[R], pos[R];
#pragma unroll
    for (int r = 0; r < R; ++r) {
      bb[r] = (uint32_t)((fmix64(key[r]) & p.cap_mask) >> sp.shift);
      pos[r] = (valid >> r & 1) ? atomicAdd(&hist[bb[r]], 1u) : 0u;
    }
    __syncthreads();
    if constexpr (TMAS) {  // bulk copies move whole 16-byte units: runs padded to an even row count
      for (uint32_t b = threadIdx.x; b < B; b += blockDim.x) {
        const uint32_t h = hist[b];
        hcnt[b] = h;
        hist[b] = (h + 1u) & ~1u;
      }
      __syncthreads();
    }
    block_excl_scan(hist, lstart, B, wtot, total);
    for (uint32_t b = threadIdx.x; b < B; b += blockDim.x) {
      hnext[b] = 0;  // every thread is past the previous tile (its last reader of this buffer)
      uint32_t h = hist[b];
      if (h) {
        uint64_t g = atomicAdd((unsigned long long*)&sp.cursor[bbase + b], (unsigned long long)h);
        gpos[b] = g;
        if (g + h > sp.seg_cap) atomicExch(sp.gate, 1u);
        if constexpr (TMAS) {
          if (hcnt[b] & 1u) skey[lstart[b] + hcnt[b]] = kEmpty;  // the padding record
        }
      }
    }
    __syncthreads();  // lstart and gpos visible to every thread
#pragma unroll
    for (int r = 0; r < R; ++r)
      if (valid >> r & 1) {
        uint32_t e = lstart[bb[r]] + pos[r];
        skey[e] = key[r];
        sbid[e] = (uint16_t)bb[r];
#pragma unroll
        for (int c = 0; c < NV; ++c) sval[(size_t)c * TS + e] = v[c][r];
      }
    if constexpr (PIPE) {  // this tile is in shared memory: the next one's loads go out now
      const uint64_t tn = t + gridDim.x;
      if (tn < ntiles) tile_load<SP, R>(p, lane_base<R>(tn * TILE, threadIdx.x >> 5, threadIdx.x & 31), tile_lim(tn), pol, T);
    }
    if constexpr (TMAS) {
      // every bucket's run of every column leaves shared memory in one bulk copy (TMA engine; no
      // per-element loads and stores): thread t copies column t / B of bucket t % B
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // staged writes -> async proxy
      __syncthreads();
      for (uint32_t t2 = threadIdx.x; t2 < B * (1u + (uint32_t)NV); t2 += blockDim.x) {
        const uint32_t col = t2 / B, b = t2 - col * B;
        const uint32_t hp = hist[b];
        if (!hp || (col > 0 && (int)col > L.n_vals) || gpos[b] + hp > sp.seg_cap) continue;
        const uint64_t row = (uint64_t)(bbase + b) * sp.seg_stride + gpos[b];
        const uint64_t* src = (col == 0 ? skey : sval + (size_t)(col - 1) * TS) + lstart[b];
        uint64_t* dst = (col == 0 ? sp.out_key : (uint64_t*)sp.out_val[col - 1]) + row;
        asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst),
                     "r"((uint32_t)__cvta_generic_to_shared(src)), "r"(hp * 8u)
                     : "memory");
      }
      asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");  // sources read: staging reusable
      continue;
    }
    __syncthreads();
    const uint32_t tot = *total;
    for (uint32_t e = threadIdx.x; e < tot; e += blockDim.x) {
      const uint32_t b = sbid[e];
      const uint64_t g = gpos[b] + (e - lstart[b]);
      if (g >= sp.seg_cap) continue;
      const uint64_t idx = (uint64_t)(bbase + b) * sp.seg_stride + g;
      sp.out_key[idx] = skey[e];
      if constexpr (SP::kStatic) {  // JIT: the value columns and their widths are compile-time
        sfor<0, SP::NV>([&](auto cc) {
          constexpr int c = decltype(cc)::v;
          const uint64_t x = sval[(size_t)c * TS + e];
          if constexpr (SP::VDT[c] == BLU_I32) ((int32_t*)sp.out_val[c])[idx] = (int32_t)(uint32_t)x;
          else ((uint64_t*)sp.out_val[c])[idx] = x;
        });
      } else {
#pragma unroll
        for (int c = 0; c < NV; ++c)
          if (c < L.n_vals) {
            const uint64_t x = sval[(size_t)c * TS + e];
            if (L.val_dtype[c] == BLU_I32) ((int32_t*)sp.out_val[c])[idx] = (int32_t)(uint32_t)x;
            else ((uint64_t*)sp.out_val[c])[idx] = x;
          }
      }
    }
  }
  if constexpr (TMAS) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");  // bulk writes complete
}


}  // namespace blu
