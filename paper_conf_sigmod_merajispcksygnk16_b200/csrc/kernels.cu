// kernels.cu — the sm_100a kernels of libblugby.
//
//   k_init_slots / k_init_dense   S4  hash-table mask copied by parallel threads (Table 1)
//   k_agg_dense_smem<NV,R>        S5a path (a): per-CTA shared-memory dense tables, CTA -> global
//                                     merge with native 64-bit REDs (§4.3.2)
//   k_agg_global<NV,R,FRONT,DIRECT>
//                                 S5b path (b): global open-addressing table, read-before-CAS
//                                     linear probing on the 64-bit key, REDs on the aggregate
//                                     fields (§4.3.1; §4.4 atomics);
//                                     DIRECT = path (b'): direct-mapped dense domain;
//                                     FRONT = shared-memory hot-key front (P:168 spill/merge)
//   k_compact_count/scan/emit     S8  path (c): occupancy -> block counts -> exclusive scan ->
//                                     dense output, key unpack, AVG = SUM / COUNT
//   k_partition_*                 S10 owner bucketing of partial states for the all-to-all
//
// Column streams are read with 128-bit non-coherent loads that bypass L1 allocation and carry an
// L2 evict-first policy, so the fact-table stream does not evict an L2-resident hash table.
// No tensor cores: nothing here is a contraction.
#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>
#include <atomic>
#include <mutex>
#include <unordered_map>

#include "blu_internal.h"
#include "blu_device.cuh"

#include <stdio.h>
#include <string.h>
#include <string>
#include <chrono>

namespace blu {

static std::atomic<uint64_t> g_launches{0};
thread_local char t_last_kernel[64] = "";
static void note_kernel(const char* k) {
  strncpy(t_last_kernel, k, sizeof t_last_kernel - 1);
  t_last_kernel[sizeof t_last_kernel - 1] = 0;
}
void count_launch(uint64_t n) { g_launches.fetch_add(n, std::memory_order_relaxed); }
uint64_t launches_total() { return g_launches.load(); }

// R (rows per thread) for a given number of value columns; identical for AOT and JIT kernels.
static int rows_per_thread(int nv) { return nv <= 4 ? 4 : nv <= 8 ? 2 : 1; }
// JIT-only tuning knobs (benchmarks): rows per thread of the dense kernel, min CTAs per SM.
static int jit_env(const char* k, int def) {
  const char* v = benv(k);
  return v && *v ? atoi(v) : def;
}

// Launch the NVRTC-specialised kernel for this plan's layout, if the JIT is enabled and succeeds.
static bool launch_jit(const char* body, const char* entry_decl, const AggParams& p, void** args, cudaStream_t st,
                       uint32_t grid, uint32_t block, uint32_t smem, const char* entry, int min_blocks = 1) {
  static const bool hdbg = benv("BLU_GBY_DEBUG_HOST") != nullptr;
  auto hnow = [] { return std::chrono::steady_clock::now(); };
  const auto h0 = hnow();
  if (!p.jit_ok || !jit_enabled()) return false;
  // 1024-thread CTAs (one per SM, wide hot-key front) keep the same 64-register budget
  // (a 768-thread CTA gets 80 registers: __launch_bounds__(768, 1))
  const int maxt = block > 512 ? (int)block : 512, minb = block > 512 ? 1 : jit_env("BLU_GBY_JIT_MINB", min_blocks);
  // Launch-path cache: (layout, entry, launch bounds, shared-table shape, device, experiment knobs)
  // -> kernel handle, so repeated executes of a plan skip building the kernel and spec sources and
  // the source-keyed lookup (host time the GPU would otherwise sit idle for). The key is a POD
  // hashed a word at a time and compared whole on a hit.
  struct Key {
    Layout lay;
    char entry[64];
    char body[256];
    char defs[128];
    int32_t maxt, minb, dev, hot;
    uint32_t S, soff[kMaxFields];
  };
  struct Fast {
    Key key;
    const void* k;
    uint32_t smem_ok;
  };
  static std::mutex fmu;
  static std::unordered_map<uint64_t, Fast> fast;
  const bool probe = jit_probe_active();
  thread_local Key key;  // ~2 KB: not on the stack of every launch
  memset(&key, 0, sizeof key);
  memcpy(&key.lay, &p.lay, sizeof key.lay);
  strncpy(key.entry, entry, sizeof key.entry - 1);
  strncpy(key.body, body, sizeof key.body - 1);
  if (const char* defs = benv("BLU_GBY_JIT_DEFS")) strncpy(key.defs, defs, sizeof key.defs - 1);
  key.maxt = maxt;
  key.minb = minb;
  if (!probe) cudaGetDevice(&key.dev);
  key.hot = jit_hot_reg();
  key.S = p.S;
  for (int j = 0; j < p.lay.n_fields; ++j) key.soff[j] = p.soff[j];
  uint64_t h = 1469598103934665603ull;
  {
    static_assert(sizeof(Key) % 8 == 0, "key hashed by 8-byte words");
    const uint64_t* w = (const uint64_t*)&key;
    for (size_t i = 0; i < sizeof(Key) / 8; ++i) h = (h ^ w[i]) * 1099511628211ull;
  }
  const auto h1 = hnow();
  const void* k = nullptr;
  uint32_t smem_ok = 0;
  if (!probe) {
    std::lock_guard<std::mutex> lk(fmu);
    auto it = fast.find(h);
    if (it != fast.end() && memcmp(&it->second.key, &key, sizeof key) == 0) {
      k = it->second.k;
      smem_ok = it->second.smem_ok;
    }
  }
  if (!k) {
    std::string src = "extern \"C\" __global__ void __launch_bounds__(" + std::to_string(maxt) + ", " +
                      std::to_string(minb) + ") ";
    src += entry_decl;
    src += " { ";
    src += body;
    src += " }\n";
    k = jit_kernel(jit_spec("JitSpec", p.lay, p.S, p.soff), src, entry);
    if (probe) return true;  // compile-only probe: nothing is launched
    if (!k) return false;
  }
  if (smem > 48 * 1024 && smem > smem_ok) {
    if (cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess) {
      cudaGetLastError();
      return false;
    }
    smem_ok = smem;
  }
  {
    std::lock_guard<std::mutex> lk(fmu);
    Fast& f = fast[h];
    if (f.k != k || f.smem_ok < smem_ok || memcmp(&f.key, &key, sizeof key) != 0) f = Fast{key, k, smem_ok};
  }
  const auto h2 = hnow();
  if (cudaLaunchKernel(k, dim3(grid), dim3(block), args, smem, st) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  if (hdbg) {
    const auto h3 = hnow();
    auto us = [](std::chrono::steady_clock::time_point a, std::chrono::steady_clock::time_point b) {
      return std::chrono::duration<double, std::micro>(b - a).count();
    };
    fprintf(stderr, "[blugby host] launch_jit us: key %.1f | lookup %.1f | cudaLaunchKernel %.1f\n", us(h0, h1),
            us(h1, h2), us(h2, h3));
  }
  count_launch(1);
  if (strncmp(entry, "blu_jit_scatter", 15) != 0) note_kernel(entry);
  return true;
}


// ------------------------------------------------------------------------------------------------
// S4: table initialisation — the mask row copied by parallel threads with 16-byte stores
// ------------------------------------------------------------------------------------------------
struct SlotTemplate {
  uint64_t w[32];  // up to 256-byte slots
  uint32_t words;  // slot_bytes / 8
};

__global__ void __launch_bounds__(256) k_init_slots(SlotTemplate t, uint64_t* table, uint64_t n_words2, uint64_t* zero,
                                                   uint32_t n_zero) {
  // n_words2 = number of 16-byte chunks; slot_bytes is a multiple of 16; zero: optional u64 block set to 0
  uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  if (zero && blockIdx.x == 0 && threadIdx.x < n_zero) zero[threadIdx.x] = 0;
  uint32_t pairs = t.words / 2;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n_words2; i += stride) {
    uint32_t w = (uint32_t)(i % pairs) * 2;
    ulonglong2 v = make_ulonglong2(t.w[w], t.w[w + 1]);
    reinterpret_cast<ulonglong2*>(table)[i] = v;
  }
}

__global__ void __launch_bounds__(256) k_fill_u64(uint64_t* a, uint64_t n, uint64_t v) {
  uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) a[i] = v;
}

// ------------------------------------------------------------------------------------------------
// AOT kernels (GenericSpec): the schema-generic versions of the bodies in blu_device.cuh
// ------------------------------------------------------------------------------------------------
template <int NV, int R, bool FUSE>
__global__ void __launch_bounds__(512, 2) k_agg_dense_smem(AggParams p, FinalParams fp) {
  dense_body<GenericSpec, NV, R, FUSE>(p, fp);
}

template <int NV, int R, bool FRONT, bool DIRECT, int MODE>
__global__ void __launch_bounds__(512, 2) k_agg_global(AggParams p, RecSrc rs) {
  global_body<GenericSpec, NV, R, FRONT, DIRECT, MODE>(p, rs);
}

template <int NV, int R, bool SEGIN>
__global__ void __launch_bounds__(512, 2) k_scatter(AggParams p, ScatterParams sp) {
  scatter_body<GenericSpec, NV, R, false, SEGIN>(p, sp);
}

// wide fan-out (B > 512): one 1024-thread CTA per SM, a tile twice as long (more rows per bucket
// per cursor reservation)
template <int NV, int R, bool SEGIN>
__global__ void __launch_bounds__(1024, 1) k_scatter_wide(AggParams p, ScatterParams sp) {
  scatter_body<GenericSpec, NV, R, false, SEGIN>(p, sp);
}

uint32_t scatter_block(uint32_t B) { return B > 512 ? 1024u : 512u; }
uint32_t scatter_grid(uint32_t sms, uint32_t B) { return B > 512 ? sms : 2 * sms; }  // resident CTAs

size_t scatter_smem(int nv, uint32_t B, bool tma) {
  const int R = rows_per_thread(nv);
  const size_t NV = nv <= 1 ? 1 : nv <= 2 ? 2 : nv <= 4 ? 4 : nv <= 8 ? 8 : 16;
  const size_t TILE = (size_t)scatter_block(B) * R;
  // the TMA write-out pads every bucket's run to an even length: staging rows TILE + B
  const size_t TS = tma ? TILE + ((B + 1) & ~1u) : TILE;
  return TS * 8 * (1 + NV) + (size_t)B * 20 + 36 * 4 + 16 + TILE * 2 + (size_t)B * 4;  // hist x 2
}

template <int NV, int R>
static int launch_scatter_nv(const AggParams& p, const ScatterParams& sp, cudaStream_t st, uint32_t grid) {
  const uint32_t bins = sp.in_seg ? sp.in_B2 : sp.B;  // histogram bins of one tile
  const uint32_t block = scatter_block(bins);
  const size_t smem = scatter_smem(p.lay.n_vals, bins, sp.tma != 0);
  if (p.jit_ok && jit_env("BLU_GBY_JIT_SCATTER", 1)) {
    char body[160], decl[160], name[64];
    // register-pipelined tile loads instead of the L2 prefetch (C3 scatter 10.07 -> 9.48 ms)
    const int pipe = jit_env("BLU_GBY_SCATTER_PIPE", 1);
    const bool seg = sp.in_seg != 0, tma = sp.tma != 0;
    snprintf(name, sizeof name, "blu_jit_scatter_%d_%d%s%s%s", NV, R, pipe ? "_p" : "", seg ? "_s" : "", tma ? "_t" : "");
    snprintf(decl, sizeof decl, "%s(blu::AggParams p, blu::ScatterParams sp)", name);
    snprintf(body, sizeof body, "blu::scatter_body<blu::JitSpec, %d, %d, %s, %s, %s>(p, sp);", NV, R,
             pipe ? "true" : "false", seg ? "true" : "false", tma ? "true" : "false");
    AggParams pc = p;
    ScatterParams sc = sp;
    void* args[] = {&pc, &sc};
    if (launch_jit(body, decl, p, args, st, grid, block, (uint32_t)smem, name, 2)) return 0;
  }
  auto k = sp.in_seg ? (block > 512 ? k_scatter_wide<NV, R, true> : k_scatter<NV, R, true>)
                     : (block > 512 ? k_scatter_wide<NV, R, false> : k_scatter<NV, R, false>);
  cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e) return (int)e;
  k<<<grid, block, smem, st>>>(p, sp);
  count_launch(1);
  return (int)cudaGetLastError();
}

int launch_scatter(const AggParams& p, const ScatterParams& sp, void* stream, uint32_t grid) {
  cudaStream_t st = (cudaStream_t)stream;
  int nv = p.lay.n_vals;
  if (nv <= 1) return launch_scatter_nv<1, 4>(p, sp, st, grid);
  if (nv <= 2) return launch_scatter_nv<2, 4>(p, sp, st, grid);
  if (nv <= 4) return launch_scatter_nv<4, 4>(p, sp, st, grid);
  if (nv <= 8) return launch_scatter_nv<8, 2>(p, sp, st, grid);
  return launch_scatter_nv<16, 1>(p, sp, st, grid);
}

// ------------------------------------------------------------------------------------------------
// Partitioned pass 2 with bucket-local shared-memory tables (bucket_body): one 1024-thread CTA per SM
// ------------------------------------------------------------------------------------------------
template <int NV, int R>
__global__ void __launch_bounds__(1024, 1) k_agg_bucket(AggParams p) {
  bucket_body<GenericSpec, NV, R>(p);
}

template <int NV, int R>
static int launch_bucket_nv(const AggParams& p, cudaStream_t st, uint32_t grid, uint32_t smem) {
  if (p.jit_ok) {
    char body[160], decl[160], name[64];
    // BLU_GBY_BUCKET_PIPE=1: 768 threads x 80 registers with the tile loads double-buffered
    const int pipe = jit_env("BLU_GBY_BUCKET_PIPE", 0) && R % 2 == 0;
    const uint32_t threads = pipe ? (uint32_t)jit_env("BLU_GBY_BUCKET_THREADS", 768) : 1024u;
    snprintf(name, sizeof name, "blu_jit_bucket_%d_%d%s", NV, R, pipe ? "_p" : "");
    snprintf(decl, sizeof decl, "%s(blu::AggParams p)", name);
    snprintf(body, sizeof body, "blu::bucket_body<blu::JitSpec, %d, %d, %s>(p);", NV, R, pipe ? "true" : "false");
    AggParams pc = p;
    void* args[] = {&pc};
    if (launch_jit(body, decl, p, args, st, grid, threads, smem, name, 1)) return 0;
  }
  auto k = k_agg_bucket<NV, R>;
  cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e) return (int)e;
  if (!p.gate || p.gate_run_if == 0) note_kernel("k_agg_bucket (generic)");
  k<<<grid, 1024, smem, st>>>(p);
  count_launch(1);
  return (int)cudaGetLastError();
}

int launch_bucket(const AggParams& p, void* stream, uint32_t grid, uint32_t smem) {
  cudaStream_t st = (cudaStream_t)stream;
  int nv = p.lay.n_vals;
  if (nv <= 1) return launch_bucket_nv<1, 4>(p, st, grid, smem);
  if (nv <= 2) return launch_bucket_nv<2, 4>(p, st, grid, smem);
  if (nv <= 4) return launch_bucket_nv<4, 4>(p, st, grid, smem);
  if (nv <= 8) return launch_bucket_nv<8, 2>(p, st, grid, smem);
  return launch_bucket_nv<16, 1>(p, st, grid, smem);
}

__device__ __forceinline__ uint64_t hash128(uint64_t w0, uint64_t w1) { return fmix64(w0 ^ fmix64(w1 ^ 0x9E3779B97F4A7C15ull)); }

// ------------------------------------------------------------------------------------------------
// Wide keys (> 64 bits; "If the key size is larger than 64 bit, we can not use CUDA atomic
// operations any more so we try to acquire a lock ... Murmur hashing"). On sm_100a a 16-byte CAS is
// native (ATOMG.E.CAS.128), so the 128-bit packed key is claimed exactly like the 64-bit one: read
// both words, compare, CAS EMPTY -> key. Hash: Murmur3 finalizer over both words. Path (b) only.
// MODE 0: columns; 1: records [w0, w1, states...].
// ------------------------------------------------------------------------------------------------
__device__ __forceinline__ void cas128(unsigned long long* a, unsigned long long cl, unsigned long long ch,
                                       unsigned long long nl, unsigned long long nh, unsigned long long& ol,
                                       unsigned long long& oh) {
  asm volatile("{\n\t.reg .b128 d, c, n;\n\tmov.b128 c, {%2, %3};\n\tmov.b128 n, {%4, %5};\n\t"
               "atom.global.cas.b128 d, [%6], c, n;\n\tmov.b128 {%0, %1}, d;\n\t}"
               : "=l"(ol), "=l"(oh)
               : "l"(cl), "l"(ch), "l"(nl), "l"(nh), "l"(a)
               : "memory");
}

__device__ __forceinline__ bool hash_locate128(uint8_t* table, uint64_t mask, uint32_t sb, uint64_t k0, uint64_t k1,
                                               uint32_t max_probe, uint64_t& out) {
  uint64_t idx = hash128(k0, k1) & mask;
  for (uint32_t q = 0; q < max_probe; ++q) {
    unsigned long long* kp = (unsigned long long*)(table + idx * sb);
    const ulonglong2 cur = __ldcg((const ulonglong2*)kp);
    if (cur.x == k0 && cur.y == k1) { out = idx; return true; }
    if (cur.x == kEmpty && cur.y == kEmpty) {
      unsigned long long ol, oh;
      cas128(kp, kEmpty, kEmpty, k0, k1, ol, oh);
      if ((ol == kEmpty && oh == kEmpty) || (ol == k0 && oh == k1)) { out = idx; return true; }
    }
    idx = (idx + 1) & mask;
  }
  return false;
}

template <int NV, int R, int MODE>
__global__ void __launch_bounds__(256) k_agg_wide(AggParams p, RecSrc rs) {
  const Layout& L = p.lay;
  const uint64_t pol = evict_first_policy();
  const uint64_t n = p.n_rows;
  const uint64_t tile = (uint64_t)blockDim.x * R;
  const uint64_t ntiles = (n + tile - 1) / tile;
  uint8_t* tb = (uint8_t*)p.table;
  uint32_t flag_seen = 0;
  for (uint64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
    if (flag_seen) break;
    flag_seen = __any_sync(0xffffffffu, *(volatile uint32_t*)p.flags);
    const uint64_t row = lane_base<R>(t * tile, threadIdx.x >> 5, threadIdx.x & 31);
    uint64_t w0[R], w1[R], v[NV][R];
    uint32_t valid = 0;
#pragma unroll
    for (int r = 0; r < R; ++r) {
      w0[r] = w1[r] = 0;
#pragma unroll
      for (int c = 0; c < NV; ++c) v[c][r] = 0;
      if (row_of<R>(row, r) < n) valid |= 1u << r;
    }
    if (MODE == 1) {
#pragma unroll
      for (int r = 0; r < R; ++r) {
        const uint64_t rr = row_of<R>(row, r);
        if (rr >= n) continue;
        const unsigned long long* rec = (const unsigned long long*)rs.rec + rr * rs.words;
        w0[r] = __ldg(rec);
        w1[r] = __ldg(rec + 1);
#pragma unroll
        for (int c = 0; c < NV; ++c)
          if (c < L.n_vals) {
            const uint64_t x = __ldg(rec + 2 + c);
            v[c][r] = L.val_dtype[c] == BLU_I32 ? (uint64_t)(int64_t)(int32_t)(uint32_t)x : x;
          }
      }
    } else {
      uint32_t bad = 0;
      for (int k = 0; k < L.n_keys; ++k) {
        uint64_t c[R];
        load_rows<R>(p.key[k], L.key_dtype[k], row, n, p.vec_ok, pol, c);
        const uint64_t d = L.dict[k], st = L.stride[k];
        const int wd = L.kword[k];
#pragma unroll
        for (int r = 0; r < R; ++r) {
          if (d ? c[r] >= d : (int64_t)c[r] < 0) bad |= 1u << r;
          const uint64_t x = d ? c[r] * st : c[r];
          if (wd) w1[r] += x;
          else w0[r] += x;
        }
      }
      bad &= valid;
      if (bad) atomicOr(p.flags, FLAG_KEY_RANGE);
      valid &= ~bad;
      load_vals<GenericSpec, NV, R>(p, row, n, pol, v);
    }
    uint64_t slot[R];
    uint32_t ok = valid;
#pragma unroll
    for (int r = 0; r < R; ++r) {
      slot[r] = 0;
      if (!(valid >> r & 1)) continue;
      uint64_t sl;
      if (hash_locate128(tb, p.cap_mask, L.slot_bytes, w0[r], w1[r], p.max_probe, sl)) {
        slot[r] = sl;
      } else {
        ok &= ~(1u << r);
        atomicOr(p.flags, FLAG_OVERFLOW);
      }
    }
    __syncwarp();
    global_apply_rows<GenericSpec, NV, R, false>(p, slot, ok, v);
  }
}
// ------------------------------------------------------------------------------------------------
// 128-bit integer payloads ("the 128bit Integer or Decimal data type" aggregated with
// atomicCAS). Path (b), one pass, generic kernel. SUM mod 2^128: the low word is added atomically
// and the carry it produced is added with the high word — addition mod 2^128 is associative and each
// low-word wrap is seen by exactly one adder, so the high word ends at sum(hi) + #wraps. MIN/MAX: a
// 16-byte CAS loop (atom.global.cas.b128); a value that looks no better than the field is confirmed
// with a CAS that writes back what it read, so a torn 16-byte read can never skip an update.
// ------------------------------------------------------------------------------------------------
__device__ __forceinline__ bool lt128(uint64_t al, uint64_t ah, uint64_t bl, uint64_t bh) {
  return (int64_t)ah < (int64_t)bh || (ah == bh && al < bl);
}

__device__ __forceinline__ void q_add(uint8_t* a, uint64_t lo, uint64_t hi) {
  const unsigned long long old = atomicAdd((unsigned long long*)a, (unsigned long long)lo);
  const uint64_t h = hi + (old + lo < old ? 1ull : 0ull);
  if (h) atomicAdd((unsigned long long*)(a + 8), (unsigned long long)h);
}

template <bool MIN>
__device__ __forceinline__ void q_minmax(uint8_t* a, uint64_t lo, uint64_t hi) {
  unsigned long long* w = (unsigned long long*)a;
  const ulonglong2 c0 = __ldcg((const ulonglong2*)a);
  unsigned long long cl = c0.x, ch = c0.y;
  for (;;) {
    const bool better = MIN ? lt128(lo, hi, cl, ch) : lt128(cl, ch, lo, hi);
    unsigned long long ol, oh;
    if (better) cas128(w, cl, ch, lo, hi, ol, oh);
    else cas128(w, cl, ch, cl, ch, ol, oh);  // confirm the value compared against
    if (ol == cl && oh == ch) return;
    cl = ol;
    ch = oh;
  }
}

__device__ __forceinline__ void ld_q(const void* base, uint64_t row, uint64_t pol, uint64_t& lo, uint64_t& hi) {
  const uint8_t* q = (const uint8_t*)base + row * 16;
  if (((uintptr_t)base & 15) == 0) {
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.u64 {%0,%1}, [%2], %3;" : "=l"(lo), "=l"(hi) : "l"(q), "l"(pol));
  } else {
    lo = ld_stream_u64(q, pol);
    hi = ld_stream_u64(q + 8, pol);
  }
}

template <int NV>
__global__ void __launch_bounds__(256) k_agg_q(AggParams p) {
  constexpr int R = 2;
  const Layout& L = p.lay;
  const uint64_t pol = evict_first_policy();
  const uint64_t n = p.n_rows, tile = (uint64_t)blockDim.x * R;
  uint8_t* tb = (uint8_t*)p.table;
  for (uint64_t t = blockIdx.x; t * tile < n; t += gridDim.x) {
    if (*(volatile uint32_t*)p.flags & FLAG_OVERFLOW) break;
    const uint64_t row = lane_base<R>(t * tile, threadIdx.x >> 5, threadIdx.x & 31);
    uint64_t key[R];
    const uint32_t valid = pack_keys<GenericSpec, R>(p, row, n, pol, key);
    uint64_t vlo[NV][R], vhi[NV][R];
#pragma unroll
    for (int c = 0; c < NV; ++c) {
#pragma unroll
      for (int r = 0; r < R; ++r) vlo[c][r] = vhi[c][r] = 0;
      if (c >= L.n_vals) continue;
      if (L.val_dtype[c] == BLU_I128) {
#pragma unroll
        for (int r = 0; r < R; ++r)
          if (row_of<R>(row, r) < n) ld_q(p.val[c], row_of<R>(row, r), pol, vlo[c][r], vhi[c][r]);
      } else {
        load_rows<R>(p.val[c], L.val_dtype[c], row, n, p.vec_ok, pol, vlo[c]);
      }
    }
    uint64_t slot[R];
    uint32_t ok = valid;
#pragma unroll
    for (int r = 0; r < R; ++r) {
      slot[r] = 0;
      if (!(valid >> r & 1)) continue;
      const uint64_t idx = fmix64(key[r]) & p.cap_mask;
      if (!hash_locate(tb, p.cap_mask, L.slot_bytes, key[r], __ldcg((const unsigned long long*)(tb + idx * L.slot_bytes)),
                       idx, p.max_probe, slot[r])) {
        ok &= ~(1u << r);
        atomicOr(p.flags, FLAG_OVERFLOW);
      }
    }
#pragma unroll
    for (int r = 0; r < R; ++r) {
      if (!(ok >> r & 1)) continue;
      uint8_t* sl = tb + slot[r] * L.slot_bytes;
      for (uint32_t m = p.cntmask; m; m &= m - 1) g_upd<FK_COUNT, true>(sl + L.f[__ffs(m) - 1].goff, 1ull);
#pragma unroll
      for (int c = 0; c < NV; ++c) {
        if (c >= L.n_vals) break;
        for (uint32_t m = p.colmask[c]; m; m &= m - 1) {
          const Field& f = L.f[__ffs(m) - 1];
          uint8_t* a = sl + f.goff;
          if (f.kind == FK_SUMQ) {
            // a 64-bit column summed into a 128-bit field (merges of COUNT never land here)
            q_add(a, vlo[c][r], L.val_dtype[c] == BLU_I128 ? vhi[c][r] : (uint64_t)((int64_t)vlo[c][r] >> 63));
          } else if (f.kind == FK_MINQ) {
            q_minmax<true>(a, vlo[c][r], vhi[c][r]);
          } else if (f.kind == FK_MAXQ) {
            q_minmax<false>(a, vlo[c][r], vhi[c][r]);
          } else {
            dispatch_kind(f.kind, [&](auto kc) {
              constexpr int K = decltype(kc)::v;
              g_upd<K, true>(a, vlo[c][r]);
            });
          }
        }
      }
    }
  }
}

// Correctly rounded (round-to-nearest-even) conversion of a two's-complement 128-bit integer to f64:
// the top 64 significant bits are converted with the sticky OR of the rest folded into bit 0 (below
// the 11 bits __ull2double_rn drops), then scaled by an exact power of two.
__device__ __forceinline__ double i128_to_f64(uint64_t lo, uint64_t hi) {
  const bool neg = (int64_t)hi < 0;
  if (neg) {
    lo = ~lo + 1ull;
    hi = ~hi + (lo == 0 ? 1ull : 0ull);
  }
  double r;
  if (hi == 0) {
    r = __ull2double_rn(lo);
  } else {
    const int z = __clzll((long long)hi);  // 0..63
    const uint64_t top = z ? (hi << z) | (lo >> (64 - z)) : hi;
    const uint64_t rest = z ? lo << z : lo;
    r = __ull2double_rn(top | (rest != 0 ? 1ull : 0ull));
    r *= __longlong_as_double((long long)(1023 + 64 - z) << 52);  // 2^(64 - z), exact
  }
  return neg ? -r : r;
}

// ------------------------------------------------------------------------------------------------
// S8: compaction (path (c))
// ------------------------------------------------------------------------------------------------
constexpr int kCT = 256;        // threads
constexpr int kCRounds = 16;    // entries per thread
constexpr uint64_t kCB = (uint64_t)kCT * kCRounds;

__device__ __forceinline__ bool occupied(const CompactParams& p, uint64_t e) {
  if (p.source == 0)
    return __ldg((const unsigned long long*)((const uint8_t*)p.table + e * p.lay.slot_bytes)) != kEmpty;
  const Field& cf = p.lay.f[p.lay.count_field];
  return __ldg((const long long*)p.dense[cf.sgroup] + (uint64_t)cf.sidx * p.n_entries + e) > 0;
}

// field j of entry e as the encoded 64-bit value
__device__ __forceinline__ uint64_t read_field(const CompactParams& p, int j, uint64_t e) {
  const Field& f = p.lay.f[j];
  if (p.source == 0) {
    const uint8_t* a = (const uint8_t*)p.table + e * p.lay.slot_bytes + f.goff;
    if (f.gsize == 4) return (uint64_t)(int64_t)__ldg((const int*)a);
    return __ldg((const unsigned long long*)a);
  }
  return __ldg((const unsigned long long*)p.dense[f.sgroup] + (uint64_t)f.sidx * p.n_entries + e);
}

__device__ __forceinline__ void store_as(void* out, uint64_t pos, int dtype, uint64_t bits) {
  if (dtype == BLU_I32) ((int32_t*)out)[pos] = (int32_t)(uint32_t)bits;
  else ((uint64_t*)out)[pos] = bits;
}

// high word of a 16-byte field (hash table only)
__device__ __forceinline__ uint64_t read_field_hi(const CompactParams& p, int j, uint64_t e) {
  const uint8_t* a = (const uint8_t*)p.table + e * p.lay.slot_bytes + p.lay.f[j].goff + 8;
  return __ldg((const unsigned long long*)a);
}

__device__ __forceinline__ void store_q(void* out, uint64_t pos, uint64_t lo, uint64_t hi) {
  ((uint64_t*)out)[2 * pos] = lo;
  ((uint64_t*)out)[2 * pos + 1] = hi;
}

__global__ void __launch_bounds__(kCT) k_compact_count(CompactParams p) {
  uint64_t base = (uint64_t)blockIdx.x * kCB;
  uint32_t c = 0;
  for (int i = 0; i < kCRounds; ++i) {
    uint64_t e = base + (uint64_t)i * kCT + threadIdx.x;
    if (e < p.n_entries && occupied(p, e)) ++c;
  }
  __shared__ uint32_t ws[kCT / 32];
  for (int o = 16; o; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
  if ((threadIdx.x & 31) == 0) ws[threadIdx.x >> 5] = c;
  __syncthreads();
  if (threadIdx.x == 0) {
    uint64_t t = 0;
    for (int w = 0; w < kCT / 32; ++w) t += ws[w];
    p.block_counts[blockIdx.x] = t;
  }
}

__global__ void __launch_bounds__(1024) k_compact_scan(uint64_t* counts, uint64_t* offsets, uint64_t nb, uint64_t* total) {
  __shared__ uint64_t ws[32];
  __shared__ uint64_t carry;
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  for (uint64_t base = 0; base < nb; base += 1024) {
    uint64_t i = base + threadIdx.x;
    uint64_t x = i < nb ? counts[i] : 0;
    uint64_t inc = x;
    for (int o = 1; o < 32; o <<= 1) {
      uint64_t y = __shfl_up_sync(0xffffffffu, inc, o);
      if ((threadIdx.x & 31) >= (unsigned)o) inc += y;
    }
    if ((threadIdx.x & 31) == 31) ws[threadIdx.x >> 5] = inc;
    __syncthreads();
    if (threadIdx.x < 32) {
      uint64_t w = ws[threadIdx.x], wi = w;
      for (int o = 1; o < 32; o <<= 1) {
        uint64_t y = __shfl_up_sync(0xffffffffu, wi, o);
        if (threadIdx.x >= (unsigned)o) wi += y;
      }
      ws[threadIdx.x] = wi - w;  // exclusive warp offsets
    }
    __syncthreads();
    uint64_t excl = carry + ws[threadIdx.x >> 5] + inc - x;
    if (i < nb) offsets[i] = excl;
    __syncthreads();
    if (threadIdx.x == 1023) carry = excl + x;
    __syncthreads();
  }
  if (threadIdx.x == 0) *total = carry;
}

// SINGLE: one CTA of T = 1024 threads covers all n_entries (<= kCB) and publishes n_groups itself
// (no count/scan launches; a 1024-entry dense domain is one round of loads instead of four).
template <bool SINGLE, int T = (SINGLE ? 1024 : kCT)>
__global__ void __launch_bounds__(T) k_compact_emit(CompactParams p) {
  __shared__ uint32_t ws[T / 32];
  const uint64_t base = (uint64_t)blockIdx.x * kCB;
  uint64_t out_pos = SINGLE ? 0 : p.block_offsets[blockIdx.x];
  const Layout& L = p.lay;
  const unsigned lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (int i = 0; i < (int)(kCB / T) && base + (uint64_t)i * T < p.n_entries; ++i) {
    uint64_t e = base + (uint64_t)i * T + threadIdx.x;
    bool occ = e < p.n_entries && occupied(p, e);
    unsigned bal = __ballot_sync(0xffffffffu, occ);
    if (lane == 0) ws[warp] = __popc(bal);
    __syncthreads();
    uint32_t before = 0, tot = 0;
    for (unsigned w = 0; w < T / 32; ++w) {
      if (w < warp) before += ws[w];
      tot += ws[w];
    }
    before += __popc(bal & ((1u << lane) - 1u));
    if (occ) {
      uint64_t pos = out_pos + before;
      const unsigned long long* kp = (const unsigned long long*)((const uint8_t*)p.table + e * L.slot_bytes);
      uint64_t key = p.source == 0 ? __ldg(kp) : e;
      if (L.key_words == 2) {  // wide keys: per-word mixed radix (a sparse code is its whole word)
        const uint64_t w[2] = {key, __ldg(kp + 1)};
        for (int k = 0; k < L.n_keys; ++k) {
          const uint64_t x = w[L.kword[k]];
          store_as(p.out_keys[k], pos, L.key_dtype[k], L.dict[k] ? (x / L.stride[k]) % L.dict[k] : x);
        }
      } else {
        const bool narrow = key >> 32 == 0 && L.domain >> 32 == 0;  // 32-bit division suffices
        for (int k = 0; k < L.n_keys; ++k) {
          uint64_t code = L.sparse ? key
                          : narrow ? (uint64_t)(((uint32_t)key / (uint32_t)L.stride[k]) % (uint32_t)L.dict[k])
                                   : (key / L.stride[k]) % L.dict[k];
          store_as(p.out_keys[k], pos, L.key_dtype[k], code);
        }
      }
      if (p.partial) {
        for (int j = 0; j < L.n_fields; ++j) {
          uint64_t x = read_field(p, j, e);
          int k = L.f[j].kind;
          if (L.f[j].gsize == 16) {
            store_q(p.out_vals[j], pos, x, read_field_hi(p, j, e));
            continue;
          }
          if (k == FK_MINF64 || k == FK_MAXF64) x = unord_f64((int64_t)x);
          int dt = (k == FK_MINI32 || k == FK_MAXI32) ? BLU_I32 : BLU_I64;
          store_as(p.out_vals[j], pos, dt, x);
        }
      } else {
        for (int o = 0; o < p.n_out; ++o) {
          int j = p.out_field[o];
          uint64_t x = read_field(p, j, e);
          int k = L.f[j].kind;
          if (p.out_kind[o] == 1) {  // AVG = (double)SUM / (double)COUNT (reading A12)
            uint64_t cnt = read_field(p, p.out_field2[o], e);
            double s = k == FK_SUMF ? __longlong_as_double((long long)x)
                       : k == FK_SUMQ ? i128_to_f64(x, read_field_hi(p, j, e)) : (double)(long long)x;
            double a = s / (double)(long long)cnt;
            x = (uint64_t)__double_as_longlong(a);
          } else if (L.f[j].gsize == 16) {
            store_q(p.out_vals[o], pos, x, read_field_hi(p, j, e));
            continue;
          } else if (k == FK_MINF64 || k == FK_MAXF64) {
            x = unord_f64((int64_t)x);
          }
          store_as(p.out_vals[o], pos, p.out_dtype[o], x);
        }
      }
    }
    __syncthreads();
    out_pos += tot;
  }
  if (SINGLE && threadIdx.x == 0) *p.n_groups = out_pos;
}

// ------------------------------------------------------------------------------------------------
// S10: owner partition of partial states for the all-to-all
// ------------------------------------------------------------------------------------------------
struct PartParams {
  Layout lay;  // merge layout (state columns)
  const void* key[kMaxKeys];
  const void* st[kMaxFields];
  uint64_t n;
  int32_t n_parts;
  uint64_t chunk;     // rows per CTA (contiguous range [blockIdx.x * chunk, ...))
  uint32_t ctas;      // grid size of the count and scatter kernels
  uint64_t* totals;   // n_parts: records per owner (the send counts)
  uint64_t* cnt;      // n_parts x ctas, owner-major: CTA c's records for owner o at [o * ctas + c]
  uint64_t* out;
  uint32_t words;
  uint32_t* flags;    // rows mode: FLAG_KEY_RANGE if a key code is outside its dictionary (else NULL)
};

// rows mode: a key code outside [0, dict) (or a negative sparse code) would pack into another key
__device__ __forceinline__ bool row_keys_bad(const PartParams& p, uint64_t i) {
  const Layout& L = p.lay;
  for (int k = 0; k < L.n_keys; ++k) {
    const int64_t c = L.key_dtype[k] == BLU_I32 ? (int64_t)((const int32_t*)p.key[k])[i] : ((const int64_t*)p.key[k])[i];
    if (c < 0 || (L.dict[k] && (uint64_t)c >= L.dict[k])) return true;
  }
  return false;
}

__device__ __forceinline__ void pack_row_wide(const PartParams& p, uint64_t i, uint64_t& w0, uint64_t& w1) {
  const Layout& L = p.lay;
  w0 = w1 = 0;
  for (int k = 0; k < L.n_keys; ++k) {
    uint64_t c = L.key_dtype[k] == BLU_I32 ? (uint64_t)(int64_t)((const int32_t*)p.key[k])[i] : ((const uint64_t*)p.key[k])[i];
    uint64_t x = L.dict[k] ? c * L.stride[k] : c;
    if (L.kword[k]) w1 += x;
    else w0 += x;
  }
}

__device__ __forceinline__ uint64_t pack_row(const PartParams& p, uint64_t i) {
  const Layout& L = p.lay;
  if (L.sparse) {
    return L.key_dtype[0] == BLU_I32 ? (uint64_t)(int64_t)((const int32_t*)p.key[0])[i] : ((const uint64_t*)p.key[0])[i];
  }
  uint64_t key = 0;
  for (int k = 0; k < L.n_keys; ++k) {
    uint64_t c = L.key_dtype[k] == BLU_I32 ? (uint64_t)(int64_t)((const int32_t*)p.key[k])[i] : ((const uint64_t*)p.key[k])[i];
    key += c * L.stride[k];
  }
  return key;
}

__device__ __forceinline__ uint32_t owner_of(uint64_t key, int32_t P) { return (uint32_t)__umul64hi(fmix64(key), (uint64_t)P); }

// S10 owner partition, three launches and no host round trip between them (the send counts are
// read back once at the end). Each CTA owns a contiguous row range: (1) it counts its rows per owner
// in shared memory (warp-aggregated: lanes with the same owner add once), no global atomics; (2) one
// CTA scans the owner-major count matrix into each (owner, CTA) output offset and the per-owner
// totals; (3) each CTA replays its range and writes every record at its owner's next position
// (shared cursors, warp-aggregated). Records of one owner keep the CTA order; within a CTA's range
// their order follows the warp aggregation (any order merges to the same result).
__device__ __forceinline__ bool part_owner(const PartParams& p, uint64_t i, uint32_t& o, uint64_t& key, uint64_t& key1) {
  if (p.flags && row_keys_bad(p, i)) return false;
  key1 = 0;
  if (p.lay.key_words == 2) {
    pack_row_wide(p, i, key, key1);
    o = (uint32_t)__umul64hi(hash128(key, key1), (uint64_t)p.n_parts);
  } else {
    key = pack_row(p, i);
    o = owner_of(key, p.n_parts);
  }
  return true;
}

__global__ void __launch_bounds__(256) k_partition_count(PartParams p) {
  __shared__ uint32_t hist[1024];
  for (int o = threadIdx.x; o < p.n_parts; o += blockDim.x) hist[o] = 0;
  __syncthreads();
  const uint64_t r0 = (uint64_t)blockIdx.x * p.chunk, r1 = min(p.n, r0 + p.chunk);
  for (uint64_t b = r0; b < r1; b += blockDim.x) {
    const uint64_t i = b + threadIdx.x;
    uint32_t o = 0xFFFFFFFFu;
    uint64_t k0, k1;
    if (i < r1 && !part_owner(p, i, o, k0, k1)) {
      atomicOr(p.flags, FLAG_KEY_RANGE);
      o = 0xFFFFFFFFu;
    }
    const unsigned peers = __match_any_sync(0xffffffffu, o);
    if (o != 0xFFFFFFFFu && (threadIdx.x & 31) == (unsigned)(__ffs(peers) - 1)) atomicAdd(&hist[o], (uint32_t)__popc(peers));
  }
  __syncthreads();
  for (int o = threadIdx.x; o < p.n_parts; o += blockDim.x) p.cnt[(uint64_t)o * p.ctas + blockIdx.x] = hist[o];
}

// one CTA: thread o (< n_parts <= 1024) sums owner o's row of the matrix, a block scan gives the
// owner bases, then the row is rewritten as exclusive offsets
__global__ void __launch_bounds__(1024) k_partition_scan(PartParams p) {
  __shared__ uint64_t tot[1024];
  const int o = threadIdx.x;
  uint64_t t = 0;
  if (o < p.n_parts)
    for (uint32_t c = 0; c < p.ctas; ++c) t += p.cnt[(uint64_t)o * p.ctas + c];
  tot[o] = t;
  __syncthreads();
  for (int d = 1; d < 1024; d <<= 1) {  // inclusive Hillis-Steele scan over the owners
    const uint64_t x = o >= d ? tot[o - d] : 0;
    __syncthreads();
    tot[o] += x;
    __syncthreads();
  }
  if (o < p.n_parts) {
    p.totals[o] = t;
    uint64_t run = tot[o] - t;
    for (uint32_t c = 0; c < p.ctas; ++c) {
      uint64_t* q = p.cnt + (uint64_t)o * p.ctas + c;
      const uint64_t x = *q;
      *q = run;
      run += x;
    }
  }
}

__global__ void __launch_bounds__(256) k_partition_scatter(PartParams p) {
  __shared__ unsigned long long cur[1024];
  for (int o = threadIdx.x; o < p.n_parts; o += blockDim.x) cur[o] = p.cnt[(uint64_t)o * p.ctas + blockIdx.x];
  __syncthreads();
  const int kw = p.lay.key_words == 2 ? 2 : 1;
  const unsigned lane = threadIdx.x & 31;
  const uint64_t r0 = (uint64_t)blockIdx.x * p.chunk, r1 = min(p.n, r0 + p.chunk);
  for (uint64_t b = r0; b < r1; b += blockDim.x) {
    const uint64_t i = b + threadIdx.x;
    uint32_t o = 0xFFFFFFFFu;
    uint64_t key = 0, key1 = 0;
    if (i < r1 && !part_owner(p, i, o, key, key1)) o = 0xFFFFFFFFu;
    const unsigned peers = __match_any_sync(0xffffffffu, o);
    const int leader = __ffs(peers) - 1;
    unsigned long long base = 0;
    if (o != 0xFFFFFFFFu && (int)lane == leader) base = atomicAdd(&cur[o], (unsigned long long)__popc(peers));
    base = __shfl_sync(0xffffffffu, base, leader);
    if (o == 0xFFFFFFFFu) continue;
    const uint64_t pos = base + __popc(peers & ((1u << lane) - 1u));
    uint64_t* rec = p.out + pos * p.words;
    rec[0] = key;
    if (kw == 2) rec[1] = key1;
    for (int j = 0; j < p.lay.n_vals; ++j) {
      uint64_t w = p.lay.val_dtype[j] == BLU_I32 ? (uint64_t)(int64_t)((const int32_t*)p.st[j])[i] : ((const uint64_t*)p.st[j])[i];
      rec[kw + j] = w;
    }
  }
}

// ------------------------------------------------------------------------------------------------
// Seeded hot-key front: heavy hitters of a row sample (the heavy-hitter aggregation of [20],
// P:38 / P:316). 1) count the packed keys of ~2^20 sampled rows in a global sample table;
// 2) histogram their counts; 3) pick the count threshold that keeps <= K keys; 4) lay those keys
// out as the front's open-addressing image (load <= 1/2) that every CTA copies into shared memory.
// ------------------------------------------------------------------------------------------------
static int grid_for(uint64_t n, int threads, int max_blocks);

struct HHParams {
  uint64_t* skey;       // sample table keys (cap_s, kEmpty = free)
  uint32_t* scnt;       // sample table counts
  uint64_t cap_s;       // power of two
  uint32_t* hist;       // kHHBins counts-of-counts
  uint32_t* ctl;        // [0] threshold, [1] keys placed
  uint64_t* front;      // S-slot front image
  uint32_t S, K;
  uint64_t blocks, block_rows, block_stride;  // sample = `blocks` runs of block_rows rows
};
constexpr uint32_t kHHBins = 4096;

__global__ void __launch_bounds__(512) k_hh_count(AggParams p, HHParams h) {
  constexpr int R = 4;
  const uint64_t pol = evict_first_policy();
  const uint64_t tiles_per_block = (h.block_rows + 512 * R - 1) / (512 * R);
  for (uint64_t w = blockIdx.x; w < h.blocks * tiles_per_block; w += gridDim.x) {
    const uint64_t b = w / tiles_per_block, t = w % tiles_per_block;
    const uint64_t r0 = b * h.block_stride + t * 512 * R;
    const uint64_t n = std::min<uint64_t>(p.n_rows, b * h.block_stride + h.block_rows);
    const uint64_t row = lane_base<R>(r0, threadIdx.x >> 5, threadIdx.x & 31);
    uint64_t key[R];
    const uint32_t valid = pack_keys<GenericSpec, R>(p, row, n, pol, key);
#pragma unroll
    for (int r = 0; r < R; ++r) {
      if (!(valid >> r & 1)) continue;
      uint64_t s = fmix64(key[r] ^ 0x68686868ull) & (h.cap_s - 1);
      for (int q = 0; q < 64; ++q) {
        uint64_t cur = __ldcg((const unsigned long long*)h.skey + s);
        if (cur == kEmpty) {
          cur = atomicCAS((unsigned long long*)h.skey + s, (unsigned long long)kEmpty, (unsigned long long)key[r]);
          if (cur == kEmpty) cur = key[r];
        }
        if (cur == key[r]) {
          atomicAdd(h.scnt + s, 1u);
          break;
        }
        s = (s + 1) & (h.cap_s - 1);
      }
    }
  }
}

__global__ void __launch_bounds__(256) k_hh_hist(HHParams h) {
  __shared__ uint32_t sh[kHHBins];
  for (uint32_t i = threadIdx.x; i < kHHBins; i += blockDim.x) sh[i] = 0;
  __syncthreads();
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < h.cap_s; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t c = h.scnt[i];
    if (c) atomicAdd(&sh[std::min<uint32_t>(c, kHHBins - 1)], 1u);
  }
  __syncthreads();
  for (uint32_t i = threadIdx.x; i < kHHBins; i += blockDim.x)
    if (sh[i]) atomicAdd(&h.hist[i], sh[i]);
}

// smallest threshold t >= 2 with #(keys with count >= t) <= K (one warp, bins scanned from the top)
__global__ void k_hh_pick(HHParams h) {
  if (threadIdx.x != 0) return;
  uint64_t acc = 0;
  uint32_t t = kHHBins;
  for (int b = kHHBins - 1; b >= 2; --b) {
    if (acc + h.hist[b] > h.K) break;
    acc += h.hist[b];
    t = b;
  }
  if (t == kHHBins) t = kHHBins - 1;  // even the top bin overflows K: take its keys first come
  h.ctl[0] = t;
}

__global__ void __launch_bounds__(256) k_hh_build(HHParams h) {
  const uint32_t t = h.ctl[0];
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < h.cap_s; i += (uint64_t)gridDim.x * blockDim.x) {
    if (h.scnt[i] < t) continue;
    if (atomicAdd(&h.ctl[1], 1u) >= h.K) continue;
    const uint64_t key = h.skey[i];
    uint32_t s = front_home(key, h.S);
    for (uint32_t q = 0; q < h.S; ++q) {  // load <= 1/2: always finds a free slot
      if (atomicCAS((unsigned long long*)h.front + s, (unsigned long long)kEmpty, (unsigned long long)key) == kEmpty) break;
      s = (s + 1) & (h.S - 1);
    }
  }
}

// Rank front (path b'): the hot keys' bits in the low halves of the image words (bit k%32 of word
// k/32), then one CTA writes each word's prefix count of hot keys into its high half.
__global__ void __launch_bounds__(256) k_hh_build_rank(HHParams h) {
  const uint32_t t = h.ctl[0];
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < h.cap_s; i += (uint64_t)gridDim.x * blockDim.x) {
    if (h.scnt[i] < t) continue;
    if (atomicAdd(&h.ctl[1], 1u) >= h.K) continue;
    const uint64_t key = h.skey[i];  // a valid dense code: < D <= 32 * rank_words
    atomicOr((uint32_t*)(h.front + (key >> 5)), 1u << (key & 31));  // low half (little endian)
  }
}

__global__ void __launch_bounds__(1024) k_hh_rank_scan(HHParams h, uint32_t words) {
  __shared__ uint32_t wsum[32];
  __shared__ uint32_t carry;
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  const unsigned lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (uint32_t w0 = 0; w0 < words; w0 += blockDim.x) {
    const uint32_t w = w0 + threadIdx.x;
    const uint32_t c = w < words ? (uint32_t)__popc((uint32_t)h.front[w]) : 0u;
    uint32_t inc = c;
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
      if ((int)lane >= o) inc += y;
    }
    if (lane == 31) wsum[warp] = inc;
    __syncthreads();
    uint32_t before = carry;
    for (unsigned q = 0; q < warp; ++q) before += wsum[q];
    if (w < words) h.front[w] = (uint64_t)(uint32_t)h.front[w] | ((uint64_t)(before + inc - c) << 32);
    __syncthreads();
    if (threadIdx.x == blockDim.x - 1) carry = before + inc;
    __syncthreads();
  }
}

// the sample's `top` most frequent keys -> (uint64_t*)(ctl + 2)[0..top) (~0 where the sample has
// fewer keys); one CTA, one argmax pass per key
__global__ void __launch_bounds__(1024) k_hh_top(HHParams h, int top) {
  __shared__ unsigned long long wbest[32];
  __shared__ unsigned long long taken[4];
  uint64_t* out = (uint64_t*)(h.ctl + 2);
  for (int q = 0; q < top; ++q) {
    unsigned long long best = 0;  // (count << 32) | slot
    for (uint64_t i = threadIdx.x; i < h.cap_s; i += blockDim.x) {
      bool skip = false;
      for (int u = 0; u < q; ++u) skip |= taken[u] == i;
      const unsigned long long c = skip ? 0ull : ((unsigned long long)h.scnt[i] << 32) | (unsigned long long)i;
      best = c > best ? c : best;
    }
    for (int o = 16; o; o >>= 1) {
      const unsigned long long y = __shfl_xor_sync(0xffffffffu, best, o);
      best = y > best ? y : best;
    }
    if ((threadIdx.x & 31) == 0) wbest[threadIdx.x >> 5] = best;
    __syncthreads();
    if (threadIdx.x == 0) {
      for (unsigned w = 0; w < (blockDim.x >> 5); ++w) best = wbest[w] > best ? wbest[w] : best;
      taken[q] = (best >> 32) ? (best & 0xffffffffull) : ~0ull;
      out[q] = (best >> 32) ? h.skey[best & 0xffffffffull] : kEmpty;
    }
    __syncthreads();
  }
}

size_t front_seed_bytes(uint32_t S) { return (size_t)S * 8 + ((size_t)1 << 18) * 12 + kHHBins * 4 + 64; }

int launch_front_seed(const AggParams& base, uint64_t n, uint32_t S, uint32_t rank_words, void* ws, void* stream,
                      int sms, const uint64_t** front_out, const uint64_t** hot_out) {
  cudaStream_t st = (cudaStream_t)stream;
  HHParams h{};
  h.S = S;
  h.K = rank_words ? S : S / 2;  // the rank front has no load-factor slack
  h.cap_s = (uint64_t)1 << 18;
  uint8_t* w = (uint8_t*)ws;
  h.front = (uint64_t*)w;
  h.skey = (uint64_t*)(w + (size_t)S * 8);
  h.scnt = (uint32_t*)(h.skey + h.cap_s);
  h.hist = h.scnt + h.cap_s;
  h.ctl = h.hist + kHHBins;
  // sample: up to 256 evenly spaced runs of 4096 rows (2^20 rows; all rows if fewer)
  h.block_rows = 4096;
  h.blocks = std::min<uint64_t>(256, (n + h.block_rows - 1) / h.block_rows);
  h.block_stride = h.blocks > 1 ? (n - h.block_rows) / (h.blocks - 1) / 4 * 4 : 0;
  if (h.blocks <= 1) h.block_rows = n;
  k_fill_u64<<<grid_for((uint64_t)S + h.cap_s, 256, sms * 8), 256, 0, st>>>(h.front, (uint64_t)S + h.cap_s, kEmpty);
  cudaMemsetAsync(h.scnt, 0, h.cap_s * 4 + kHHBins * 4 + 64, st);
  if (rank_words) cudaMemsetAsync(h.front, 0, (size_t)S * 8, st);  // empty bitmap, zero prefixes
  AggParams p = base;
  p.n_rows = n;
  k_hh_count<<<sms * 2, 512, 0, st>>>(p, h);
  k_hh_hist<<<sms, 256, 0, st>>>(h);
  k_hh_pick<<<1, 32, 0, st>>>(h);
  if (rank_words) {
    k_hh_build_rank<<<sms, 256, 0, st>>>(h);
    k_hh_rank_scan<<<1, 1024, 0, st>>>(h, rank_words);
    count_launch(6);
    if (hot_out) {
      k_hh_top<<<1, 1024, 0, st>>>(h, jit_hot_reg());
      count_launch(1);
      *hot_out = (const uint64_t*)(h.ctl + 2);
    }
  } else {
    k_hh_build<<<sms, 256, 0, st>>>(h);
    count_launch(5);
  }
  *front_out = h.front;
  return (int)cudaGetLastError();
}

// ------------------------------------------------------------------------------------------------
// read-only roofline (measurement helper): stream every column once, XOR-fold, one RED per CTA
// ------------------------------------------------------------------------------------------------
struct ReadCols {
  const int4* c[kMaxKeys + kMaxVals];
  uint64_t n16[kMaxKeys + kMaxVals];  // 16-byte chunks per column
  int n;
  unsigned long long* out;
};

__global__ void __launch_bounds__(512, 2) k_read_roofline(ReadCols rc) {
  const uint64_t pol = evict_first_policy();
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  uint64_t acc = 0;
  for (int j = 0; j < rc.n; ++j) {
    const int4* p = rc.c[j];
    const uint64_t n = rc.n16[j];
    uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    for (; i + 3 * stride < n; i += 4 * stride) {  // 4 independent loads in flight per thread
      const int4 a = ld_stream_v4(p + i, pol), b = ld_stream_v4(p + i + stride, pol);
      const int4 c = ld_stream_v4(p + i + 2 * stride, pol), d = ld_stream_v4(p + i + 3 * stride, pol);
      acc ^= (uint64_t)(uint32_t)(a.x ^ b.x ^ c.x ^ d.x) | (uint64_t)(uint32_t)(a.y ^ b.y ^ c.y ^ d.y) << 32;
      acc ^= (uint64_t)(uint32_t)(a.z ^ b.z ^ c.z ^ d.z) | (uint64_t)(uint32_t)(a.w ^ b.w ^ c.w ^ d.w) << 32;
    }
    for (; i < n; i += stride) {
      const int4 a = ld_stream_v4(p + i, pol);
      acc ^= (uint64_t)(uint32_t)a.x | (uint64_t)(uint32_t)a.y << 32;
      acc ^= (uint64_t)(uint32_t)a.z | (uint64_t)(uint32_t)a.w << 32;
    }
  }
  for (int o = 16; o; o >>= 1) acc ^= __shfl_xor_sync(0xffffffffu, acc, o);
  if ((threadIdx.x & 31) == 0) atomicXor(rc.out, (unsigned long long)acc);
}

int launch_read_roofline(const void* const* cols, const uint64_t* bytes, int n_cols, void* stream, uint64_t* out,
                         int sms) {
  ReadCols rc{};
  rc.n = n_cols;
  rc.out = (unsigned long long*)out;
  for (int j = 0; j < n_cols; ++j) {
    rc.c[j] = (const int4*)cols[j];
    rc.n16[j] = bytes[j] / 16;
  }
  k_read_roofline<<<2 * sms, 512, 0, (cudaStream_t)stream>>>(rc);
  count_launch(1);
  return (int)cudaGetLastError();
}

// ------------------------------------------------------------------------------------------------
// launchers
// ------------------------------------------------------------------------------------------------
static int grid_for(uint64_t n, int threads, int max_blocks) {
  uint64_t b = (n + threads - 1) / threads;
  if (b > (uint64_t)max_blocks) b = max_blocks;
  return (int)(b ? b : 1);
}

int launch_init_slots(const Layout& lay, void* table, uint64_t n_slots, void* stream, uint64_t* zero, uint32_t n_zero) {
  if (!n_slots && !zero) return 0;
  SlotTemplate t{};
  uint8_t buf[256];
  build_slot_template(lay, buf);
  memcpy(t.w, buf, lay.slot_bytes);
  t.words = lay.slot_bytes / 8;
  uint64_t chunks = n_slots * (lay.slot_bytes / 16);
  if (!chunks && !zero) return 0;
  k_init_slots<<<grid_for(std::max<uint64_t>(chunks, 1), 256, 148 * 16), 256, 0, (cudaStream_t)stream>>>(
      t, (uint64_t*)table, chunks, zero, zero ? n_zero : 0);
  count_launch(1);
  return (int)cudaGetLastError();
}

static uint64_t identity_host(int k) {
  switch (k) {
    case FK_MINI32: return (uint64_t)(int64_t)INT32_MAX;
    case FK_MAXI32: return (uint64_t)(int64_t)INT32_MIN;
    case FK_MINI64: case FK_MINF64: return (uint64_t)INT64_MAX;
    case FK_MAXI64: case FK_MAXF64: return (uint64_t)INT64_MIN;
    default: return 0ull;
  }
}

struct DenseInit {
  uint64_t* a[4];
  uint64_t n[4];
  uint64_t* zero;  // optional block of n_zero u64 words set to 0 (the execute's flag/counter block)
  uint32_t n_zero;
};

__global__ void __launch_bounds__(256) k_init_dense_all(DenseInit d) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x, t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (d.zero && t < d.n_zero) d.zero[t] = 0;
#pragma unroll
  for (int g = 0; g < 4; ++g) {
    const uint64_t v = g == SG_MIN ? (uint64_t)INT64_MAX : g == SG_MAX ? (uint64_t)INT64_MIN : 0ull;
    for (uint64_t i = t; i < d.n[g]; i += stride) d.a[g][i] = v;
  }
}

int launch_init_dense(const Layout& lay, void* const dense[4], uint64_t D, void* stream, uint64_t* zero,
                      uint32_t n_zero) {
  // Dense state groups: ISUM/FSUM -> 0; MIN -> INT64_MAX (covers widened i32 and ordered f64);
  // MAX -> INT64_MIN. Each group is one contiguous array; one launch initialises all of them.
  DenseInit d{};
  uint64_t tot = n_zero;
  for (int g = 0; g < 4; ++g) {
    d.a[g] = (uint64_t*)dense[g];
    d.n[g] = (uint64_t)lay.n_group[g] * D;
    tot = std::max<uint64_t>(tot, d.n[g]);
  }
  d.zero = zero;
  d.n_zero = zero ? n_zero : 0;
  if (!tot) return 0;
  k_init_dense_all<<<grid_for(tot, 256, 148 * 16), 256, 0, (cudaStream_t)stream>>>(d);
  count_launch(1);
  (void)identity_host;
  return (int)cudaGetLastError();
}

template <int NV, int R>
static int launch_agg_nv(const blu_gby_plan_s* P, int path, const AggParams& p, const RecSrc& rs, bool records,
                         void* stream, uint32_t grid, uint32_t block, uint32_t smem, const FinalParams* fin) {
  cudaStream_t st = (cudaStream_t)stream;
  cudaError_t e = cudaSuccess;
  if (p.lay.has_q) {  // 128-bit payloads: path (b), columns, generic kernel
    if (records || path != BLU_PATH_HASH_GLOBAL || p.lay.key_words == 2) return (int)cudaErrorInvalidValue;
    note_kernel("k_agg_q (generic)");
    k_agg_q<NV><<<grid, 256, 0, st>>>(p);
    count_launch(1);
    return (int)cudaGetLastError();
  }
  if (!records && p.jit_ok && p.lay.key_words != 2) {
    const int nv = p.lay.n_vals < 1 ? 1 : p.lay.n_vals;
    int r = rows_per_thread(p.lay.n_vals);
    char body[256], decl[160], name[64];
    AggParams pc = p;
    RecSrc rc = rs;
    if (path == BLU_PATH_DENSE_SMEM) {
      r = jit_env("BLU_GBY_JIT_R", r);
      const int fuse = fin && fin->enabled;
      snprintf(name, sizeof name, "blu_jit_dense_%d_%d%s", nv, r, fuse ? "_fused" : "");
      snprintf(decl, sizeof decl, "%s(blu::AggParams p, blu::FinalParams fp)", name);
      const int pairmap = r == 4 && jit_env("BLU_GBY_DENSE_PAIR", 0);
      // software-pipelined stream (BLU_GBY_DENSE_PIPE=0/1, rows per thread BLU_GBY_DENSE_PIPE_R)
      // default on for the large-input kernel (C2: 0.704 -> 0.603 ms); the fused small-input kernel
      // is launch-bound and measured slightly slower with it (C1: 18 -> 20 us)
      const int pipe = !pairmap && jit_env("BLU_GBY_DENSE_PIPE", fuse ? 0 : 1);
      if (pipe) {
        r = jit_env("BLU_GBY_DENSE_PIPE_R", 2) >= 4 ? 4 : 2;
        snprintf(name, sizeof name, "blu_jit_dense_%d_%d%s_p", nv, r, fuse ? "_fused" : "");
        snprintf(decl, sizeof decl, "%s(blu::AggParams p, blu::FinalParams fp)", name);
      }
      snprintf(body, sizeof body, "blu::dense_body<blu::JitSpec, %d, %d, %s, %s, %s>(p, fp);", nv, r, fuse ? "true" : "false",
               pairmap ? "true" : "false", pipe ? "true" : "false");
      FinalParams fpc = fin ? *fin : FinalParams{};
      void* args[] = {&pc, &fpc};
      // 2 CTAs x 512 threads per SM: <= 64 registers (one resident wave, see plan.cpp)
      if (launch_jit(body, decl, p, args, st, grid, block, smem, name, 2)) return 0;
    } else {
      const int front = p.front_slots > 0, direct = path == BLU_PATH_DIRECT_GLOBAL;
      // MODE 3: one-pass row stream with the next tile's loads issued before the current tile's
      // work (BLU_GBY_PIPE=0/1, rows per thread BLU_GBY_PIPE_R, even)
      // (default on: C4 14.2 -> 10.1 ms)
      // MODE 4: the same for pass 2 of the partitioned path (BLU_GBY_SEG_PIPE=0/1)
      const int pipe = p.seg_stride ? jit_env("BLU_GBY_SEG_PIPE", 0) : jit_env("BLU_GBY_PIPE", 1);
      const int mode = p.seg_stride ? (pipe ? 4 : 2) : pipe ? 3 : 0;
      // rows per thread double-buffered: 4 when the CTA has 513..768 threads (>= 80 registers), else 2
      if (pipe) r = jit_env("BLU_GBY_PIPE_R", block > 512 && block <= 768 ? 4 : 2) >= 4 ? 4 : 2;
      snprintf(name, sizeof name, "blu_jit_global_%d_%d_%d_%d_%d", nv, r, front, direct, mode);
      snprintf(decl, sizeof decl, "%s(blu::AggParams p, blu::RecSrc rs)", name);
      snprintf(body, sizeof body, "blu::global_body<blu::JitSpec, %d, %d, %s, %s, %d>(p, rs);", nv, r,
               front ? "true" : "false", direct ? "true" : "false", mode);
      void* args[] = {&pc, &rc};
      // <= 64 registers: 2 CTAs of 512 (front) or 4 of 256 threads per SM stay resident
      if (launch_jit(body, decl, p, args, st, grid, block, smem, name, 2)) return 0;
    }
  }
  if (path == BLU_PATH_DENSE_SMEM) {
    if constexpr (NV > 16) {
      return (int)cudaErrorInvalidValue;
    } else {
      note_kernel("k_agg_dense_smem (generic)");
      auto k = (fin && fin->enabled) ? k_agg_dense_smem<NV, R, true> : k_agg_dense_smem<NV, R, false>;
      if (smem > 48 * 1024) e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
      if (e) return (int)e;
      k<<<grid, block, smem, st>>>(p, fin ? *fin : FinalParams{});
    }
  } else {
    void (*k)(AggParams, RecSrc);
    bool front = p.front_slots > 0;
    bool direct = path == BLU_PATH_DIRECT_GLOBAL;
    if (p.lay.key_words == 2) {  // wide keys: 16-byte key CAS (hash path only)
      if constexpr (NV <= 16) {
        k = records ? k_agg_wide<NV, R, 1> : k_agg_wide<NV, R, 0>;
        note_kernel("k_agg_wide (generic)");
        k<<<grid, block < 256 ? block : 256, 0, st>>>(p, rs);
        count_launch(1);
        return (int)cudaGetLastError();
      } else {
        return (int)cudaErrorInvalidValue;
      }
    }
    if constexpr (NV > 16) {  // merges of wide states: no front, no records
      if (records || front || direct) return (int)cudaErrorInvalidValue;
      k = k_agg_global<NV, R, false, false, 0>;
    } else {
      if (records) k = k_agg_global<NV, R, false, false, 1>;
      else if (p.seg_stride) k = k_agg_global<NV, R, false, false, 2>;
      else if (direct) k = front ? k_agg_global<NV, R, true, true, 0> : k_agg_global<NV, R, false, true, 0>;
      else k = front ? k_agg_global<NV, R, true, false, 0> : k_agg_global<NV, R, false, false, 0>;
    }
    if (smem > 48 * 1024) e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e) return (int)e;
    if (!p.gate || p.gate_run_if == 0) note_kernel("k_agg_global (generic)");
    k<<<grid, block > 512 ? 512 : block, smem, st>>>(p, rs);  // generic kernels: <= 512 threads
  }
  count_launch(1);
  return (int)cudaGetLastError();
}

int launch_aggregate_impl(const blu_gby_plan_s* P, int path, const AggParams& p, const RecSrc& rs, bool records,
                          void* stream, uint32_t grid, uint32_t block, uint32_t smem, const FinalParams* fin) {
  int nv = p.lay.n_vals;
  if (nv <= 1) return launch_agg_nv<1, 4>(P, path, p, rs, records, stream, grid, block, smem, fin);
  if (nv <= 2) return launch_agg_nv<2, 4>(P, path, p, rs, records, stream, grid, block, smem, fin);
  if (nv <= 4) return launch_agg_nv<4, 4>(P, path, p, rs, records, stream, grid, block, smem, fin);
  if (nv <= 8) return launch_agg_nv<8, 2>(P, path, p, rs, records, stream, grid, block, smem, fin);
  if (nv <= 16) return launch_agg_nv<16, 1>(P, path, p, rs, records, stream, grid, block, smem, fin);
  return launch_agg_nv<24, 1>(P, path, p, rs, records, stream, grid, block, smem, fin);
}

int launch_compact(const CompactParams& p, void* stream, uint32_t* launches) {
  cudaStream_t st = (cudaStream_t)stream;
  uint64_t nb = (p.n_entries + kCB - 1) / kCB;
  if (nb == 0) {
    cudaMemsetAsync(p.n_groups, 0, 8, st);
    return (int)cudaGetLastError();
  }
  if (nb == 1) {  // small table / dense domain: one CTA, one launch
    k_compact_emit<true><<<1, 1024, 0, st>>>(p);
    count_launch(1);
    if (launches) *launches += 1;
    return (int)cudaGetLastError();
  }
  k_compact_count<<<(unsigned)nb, kCT, 0, st>>>(p);
  k_compact_scan<<<1, 1024, 0, st>>>(p.block_counts, p.block_offsets, nb, p.n_groups);
  k_compact_emit<false><<<(unsigned)nb, kCT, 0, st>>>(p);
  count_launch(3);
  if (launches) *launches += 3;
  return (int)cudaGetLastError();
}

uint64_t partition_scratch_bytes(uint64_t n, int32_t n_parts) {
  return (uint64_t)n_parts * partition_ctas(n) * 8 + 64;
}

uint32_t partition_ctas(uint64_t n) {
  const uint64_t by_rows = (n + 4095) / 4096;  // >= 4096 rows per CTA
  // per-CTA shared counts are 32-bit: at most 2^31 rows per CTA
  const uint64_t min_ctas = (n >> 31) + 1;
  return (uint32_t)std::max<uint64_t>(min_ctas, std::max<uint64_t>(1, std::min<uint64_t>(by_rows, 148 * 8)));
}

int launch_partition(const Layout& lay, const void* const* key_cols, const void* const* state_cols, uint64_t n,
                     int32_t n_parts, void* send_buf, uint64_t* d_totals, void* scratch, void* stream,
                     uint32_t* d_flags) {
  cudaStream_t st = (cudaStream_t)stream;
  PartParams p{};
  p.lay = lay;
  for (int k = 0; k < lay.n_keys; ++k) p.key[k] = key_cols[k];
  for (int j = 0; j < lay.n_vals; ++j) p.st[j] = state_cols[j];
  p.n = n;
  p.n_parts = n_parts;
  p.ctas = partition_ctas(n);
  p.chunk = (n + p.ctas - 1) / p.ctas;
  p.totals = d_totals;
  p.cnt = (uint64_t*)scratch;
  p.out = (uint64_t*)send_buf;
  p.words = (lay.key_words == 2 ? 2 : 1) + lay.n_vals;
  p.flags = d_flags;
  k_partition_count<<<p.ctas, 256, 0, st>>>(p);
  k_partition_scan<<<1, 1024, 0, st>>>(p);
  k_partition_scatter<<<p.ctas, 256, 0, st>>>(p);
  count_launch(3);
  return (int)cudaGetLastError();
}

}  // namespace blu
