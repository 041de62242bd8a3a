// api.cu — the execute / merge / exchange entry points of libblugby (C ABI, include/blu_gby.h).
//
// One execute is stream-ordered: S4 init -> S5 aggregate (one launch per input batch) -> S8
// compaction into upper-bound-sized outputs -> ONE synchronisation that reads {flags, n_groups}.
// If the flags report that a probe exceeded its bound (the estimate was too small, "error
// detection code-path ... we could still process the query"), the table is regrown 4x and the
// query rerun; a key outside its dictionary returns BLU_E_KEY_RANGE with no result.
#include <cuda_runtime.h>
#include <stdarg.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <chrono>
#include <functional>
#include <mutex>
#include <vector>

#include "blu_internal.h"

namespace blu {


extern thread_local char t_last_kernel[64];  // kernels.cu
static thread_local bool t_timing = false;
static thread_local blu_gby_timing_t t_last{};

struct Events {
  cudaEvent_t e[8];
  bool ok = false;
  void make() {
    if (ok) return;
    for (auto& x : e) cudaEventCreate(&x);
    ok = true;
  }
};
static thread_local Events t_ev;

// Partitioned path (b): three events per chunk (before the scatter, between the passes, after pass 2),
// read by run_core after its synchronisation.
struct PartEvents {
  std::vector<cudaEvent_t> ev;
  size_t used = 0;
  uint32_t* gates = nullptr;  // pinned: per chunk, 1 if a bucket overflowed (fallback ran)
  uint32_t* gate_slot(size_t chunk) {
    if (!gates && cudaMallocHost((void**)&gates, 4 * 256) != cudaSuccess) {
      cudaGetLastError();
      gates = nullptr;
    }
    return gates && chunk < 256 ? gates + chunk : nullptr;
  }
  cudaEvent_t next() {
    if (used == ev.size()) {
      cudaEvent_t e;
      cudaEventCreate(&e);
      ev.push_back(e);
    }
    return ev[used++];
  }
};
static thread_local PartEvents t_pev;

static uint64_t* pinned_scratch() {
  static thread_local uint64_t* p = nullptr;
  if (!p) {
    if (cudaMallocHost((void**)&p, 256) != cudaSuccess) {
      cudaGetLastError();
      p = nullptr;
    }
  }
  return p;
}

void setup_pool() {
  static std::once_flag once;
  std::call_once(once, [] {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaMemPool_t pool;
    if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) {
      uint64_t thr = UINT64_MAX;
      cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
    }
    // L2 fetch granularity for the random slot traffic of path (b) (a hint; 0 keeps the default)
    if (const char* g = benv("BLU_GBY_L2_FETCH")) {
      int v = atoi(g);
      if (v > 0) cudaDeviceSetLimit(cudaLimitMaxL2FetchGranularity, (size_t)v);
    }
    cudaGetLastError();
  });
}

static blu_status_t cuda_fail(cudaError_t e, const char* what) {
  if (e == cudaErrorMemoryAllocation) return fail(BLU_E_OOM, "%s: %s", what, cudaGetErrorString(e));
  return fail(BLU_E_CUDA, "%s: %s", what, cudaGetErrorString(e));
}

#define CK(call, what)                              \
  do {                                              \
    cudaError_t _e = (cudaError_t)(call);           \
    if (_e != cudaSuccess) {                        \
      cudaGetLastError();                           \
      return cuda_fail(_e, what);                   \
    }                                               \
  } while (0)

// Owner record behind blu_gby_result_t::_owner.
struct Owner {
  std::vector<void*> dev;
  std::vector<void*> host;  // pinned blocks of the host-result cache (released with host_put)
};

// Pinned host blocks for host results (blu_gby_execute_host), kept and reused across queries — the
// paper's "single large memory segment" pinned once and reused: results are copied at the
// pinned D2H rate with no page-locking, page faults or bounce copy per query. A block returns to the
// cache when its result is freed.
struct HostBlock {
  void* p;
  size_t bytes;
  bool busy;
};
static std::mutex g_hcache_mu;
static std::vector<HostBlock> g_hcache;

static void* host_get(size_t bytes) {
  bytes = std::max<size_t>((bytes + 4095) & ~(size_t)4095, 4096);
  {
    std::lock_guard<std::mutex> lk(g_hcache_mu);
    int best = -1;
    for (int i = 0; i < (int)g_hcache.size(); ++i) {
      const HostBlock& b = g_hcache[i];
      if (b.busy || b.bytes < bytes || b.bytes > 2 * bytes + (16u << 20)) continue;
      if (best < 0 || b.bytes < g_hcache[best].bytes) best = i;
    }
    if (best >= 0) {
      g_hcache[best].busy = true;
      return g_hcache[best].p;
    }
  }
  void* p = nullptr;
  if (cudaMallocHost(&p, bytes) != cudaSuccess) {
    cudaGetLastError();
    return nullptr;
  }
  std::lock_guard<std::mutex> lk(g_hcache_mu);
  g_hcache.push_back(HostBlock{p, bytes, true});
  return p;
}

static void host_put(void* p) {
  std::lock_guard<std::mutex> lk(g_hcache_mu);
  for (auto& b : g_hcache)
    if (b.p == p) b.busy = false;
}

static size_t dtype_bytes(int dt) { return dt == BLU_I32 ? 4 : dt == BLU_I128 ? 16 : 8; }

// Workspace cache (per process, per device): the hash table, dense state and partition buffers of
// an execute come from blocks that are cudaMalloc'd once and reused by later executes — the B200
// counterpart of the paper's "single large memory segment" registered up front and sub-allocated
// per call. Re-mapping tens of GB of stream-ordered pool memory per query stalls the GPU.
// A block is handed back only after the stream that used it has been synchronised (every entry
// point synchronises before returning).
struct CacheBlock {
  void* p;
  size_t bytes;
  int dev;
  bool busy;
};
static std::mutex g_cache_mu;
static std::vector<CacheBlock> g_cache;

cudaError_t cache_get(void** out, size_t bytes) {
  int dev = 0;
  cudaGetDevice(&dev);
  bytes = (bytes + (2u << 20) - 1) & ~(size_t)((2u << 20) - 1);
  std::lock_guard<std::mutex> lk(g_cache_mu);
  int best = -1;
  for (int i = 0; i < (int)g_cache.size(); ++i) {
    const CacheBlock& b = g_cache[i];
    if (b.busy || b.dev != dev || b.bytes < bytes || b.bytes > 2 * bytes + (64u << 20)) continue;
    if (best < 0 || b.bytes < g_cache[best].bytes) best = i;
  }
  if (best >= 0) {
    g_cache[best].busy = true;
    *out = g_cache[best].p;
    return cudaSuccess;
  }
  void* p = nullptr;
  cudaError_t e = cudaMalloc(&p, bytes);
  if (e == cudaErrorMemoryAllocation) {  // give idle cached blocks back and retry once
    cudaGetLastError();
    for (auto it = g_cache.begin(); it != g_cache.end();) {
      if (!it->busy && it->dev == dev) {
        cudaFree(it->p);
        it = g_cache.erase(it);
      } else {
        ++it;
      }
    }
    e = cudaMalloc(&p, bytes);
  }
  if (e != cudaSuccess) return e;
  g_cache.push_back(CacheBlock{p, bytes, dev, true});
  *out = p;
  return cudaSuccess;
}

static size_t cache_idle_bytes() {
  int dev = 0;
  cudaGetDevice(&dev);
  std::lock_guard<std::mutex> lk(g_cache_mu);
  size_t t = 0;
  for (auto& b : g_cache)
    if (!b.busy && b.dev == dev) t += b.bytes;
  return t;
}

void cache_put(void* p) {
  std::lock_guard<std::mutex> lk(g_cache_mu);
  for (auto& b : g_cache)
    if (b.p == p) b.busy = false;
}

// Scratch of one execute; released (to the cache) when destroyed. A block may only go back once
// the kernels queued on `st` that use it have finished: the success paths synchronise `st` and call
// drained(); on an early error return the destructor synchronises `st` itself before releasing.
struct Work {
  cudaStream_t st;
  std::vector<void*> ptrs;
  bool synced = false;
  explicit Work(cudaStream_t s) : st(s) {}
  void drained() { synced = true; }
  cudaError_t alloc(void** p, size_t bytes) {
    *p = nullptr;
    if (!bytes) return cudaSuccess;
    cudaError_t e = cache_get(p, bytes);
    if (e == cudaSuccess) ptrs.push_back(*p);
    return e;
  }
  ~Work() {
    if (!ptrs.empty() && !synced) {
      cudaStreamSynchronize(st);  // error path: queued kernels may still write these blocks
      cudaGetLastError();
    }
    for (void* p : ptrs) cache_put(p);
  }
};

// What the compaction emits.
struct OutSpec {
  bool partial;
  int n_out;
  int out_kind[kMaxFields], out_field[kMaxFields], out_field2[kMaxFields], out_dtype[kMaxFields];
};

static OutSpec make_outspec(const blu_gby_plan_s* P, const Layout& lay, bool partial) {
  OutSpec o{};
  o.partial = partial;
  if (partial) {
    o.n_out = lay.n_fields;
    for (int j = 0; j < lay.n_fields; ++j) {
      int k = lay.f[j].kind;
      o.out_dtype[j] = (k == FK_MINI32 || k == FK_MAXI32) ? BLU_I32
                       : (k == FK_SUMF || k == FK_MINF64 || k == FK_MAXF64) ? BLU_F64
                       : (k == FK_SUMQ || k == FK_MINQ || k == FK_MAXQ) ? BLU_I128 : BLU_I64;
    }
  } else {
    o.n_out = (int)P->amap.size();
    for (int a = 0; a < o.n_out; ++a) {
      const AggMap& m = P->amap[a];
      o.out_kind[a] = m.op == BLU_AVG ? 1 : 0;
      o.out_field[a] = m.field;
      o.out_field2[a] = m.field2;
      o.out_dtype[a] = m.out_dtype;
    }
  }
  return o;
}

// Feeds every input batch to the aggregation kernel for one attempt. `base` carries the targets.
using Feeder = std::function<cudaError_t(AggParams& base, uint32_t* launches, Work& w, const FinalParams* fin)>;

static bool ptr_aligned(const void* p) { return ((uintptr_t)p & 15) == 0; }
static uint32_t prefetch_enabled() {  // scatter prefetch distance in tiles (BLU_GBY_PREFETCH, default 1)
  static const uint32_t d = benv("BLU_GBY_PREFETCH") ? (uint32_t)atoi(benv("BLU_GBY_PREFETCH")) : 1u;
  return d;
}

// Launch the aggregation for rows [0, n) of one batch, chunked so per-CTA 32-bit shared counters
// cannot overflow.
static cudaError_t agg_batch(const blu_gby_plan_s* P, int path, AggParams p, const void* const* keys,
                             const void* const* vals, uint64_t n, const RecSrc* rs, cudaStream_t st,
                             uint32_t grid, uint32_t block, uint32_t smem, uint32_t* launches,
                             const FinalParams* fin = nullptr) {
  const Layout& L = p.lay;
  uint64_t max_rows = ((uint64_t)grid * (1ull << 30)) & ~3ull;
  for (uint64_t r0 = 0; r0 < n; r0 += max_rows) {
    uint64_t m = std::min(max_rows, n - r0);
    bool vec = true;
    if (!rs) {
      for (int k = 0; k < L.n_keys; ++k) {
        p.key[k] = (const uint8_t*)keys[k] + r0 * dtype_bytes(L.key_dtype[k]);
        vec = vec && ptr_aligned(p.key[k]);
      }
      for (int c = 0; c < L.n_vals; ++c) {
        p.val[c] = (const uint8_t*)vals[c] + r0 * dtype_bytes(L.val_dtype[c]);
        vec = vec && ptr_aligned(p.val[c]);
      }
    }
    p.vec_ok = vec ? 1 : 0;
    if (vec) {
      bool v32 = true;
      for (int k = 0; k < L.n_keys; ++k) v32 = v32 && ((uintptr_t)p.key[k] & 31) == 0;
      for (int c = 0; c < L.n_vals; ++c) v32 = v32 && ((uintptr_t)p.val[c] & 31) == 0;
      if (v32) p.vec_ok |= 2;
    }
    p.n_rows = m;
    RecSrc r{nullptr, 0};
    if (rs) r = RecSrc{rs->rec + r0 * rs->words, rs->words};
    int e = launch_aggregate_impl(P, path, p, r, rs != nullptr, st, grid, block, smem, fin);
    if (e) return (cudaError_t)e;
    if (launches) ++*launches;
  }
  return cudaSuccess;
}

// The core: init -> feed -> compact -> one sync -> regrow on overflow.
static blu_status_t run_core(const blu_gby_plan_s* P, const Layout& lay, int path, bool front, uint64_t cap0,
                             uint64_t total_rows, const Feeder& feed, bool partial, cudaStream_t st,
                             blu_gby_result_t* out, bool host_out, float* h2d_ms_acc, bool fuse_req = false) {
  static const bool hprof = benv("BLU_GBY_DEBUG_HOST") != nullptr;  // host-time breakdown per execute
  auto hnow = [] { return std::chrono::steady_clock::now(); };
  const auto h_entry = hnow();
  std::chrono::steady_clock::time_point h_init{}, h_feed{}, h_alloc{}, h_compact{}, h_sync{};
  setup_pool();
  memset(out, 0, sizeof *out);
  const bool dense = path != BLU_PATH_HASH_GLOBAL;
  const uint64_t D = lay.domain;
  uint64_t cap = dense ? D : cap0;
  uint32_t retries = 0;
  blu_gby_timing_t tm{};
  if (t_timing) t_ev.make();
  OutSpec os = make_outspec(P, lay, partial);

  for (;;) {
    Work w(st);
    void* table = nullptr;
    void* dense_g[4] = {nullptr, nullptr, nullptr, nullptr};
    if (t_timing) cudaEventRecord(t_ev.e[0], st);
    // path (a) with a small domain: init (S4) and compaction (S8) fused into the aggregation kernel
    const bool fuse = fuse_req && path == BLU_PATH_DENSE_SMEM && D <= 65536 && !partial && !host_out &&
                      !benv("BLU_GBY_NO_FUSE");
    const uint64_t n_entries = dense ? D : cap;
    const uint64_t nb = (n_entries + 4095) / 4096;
    void* small = nullptr;
    CK(w.alloc(&small, 64 + 16 * std::max<uint64_t>(nb, 1)), "workspace alloc");
    uint32_t* d_flags = (uint32_t*)small;
    uint64_t* d_ngroups = (uint64_t*)((uint8_t*)small + 8);
    uint64_t* d_bcounts = (uint64_t*)((uint8_t*)small + 64);
    uint64_t* d_boffs = d_bcounts + std::max<uint64_t>(nb, 1);
    if (dense) {
      for (int g = 0; g < 4; ++g) CK(w.alloc(&dense_g[g], (size_t)lay.n_group[g] * D * 8), "dense state alloc");
      if (!fuse) CK(launch_init_dense(lay, dense_g, D, st, (uint64_t*)small, 8), "init dense");  // + flags
      else CK(cudaMemsetAsync(small, 0, 64, st), "memset flags");
    } else {
      CK(w.alloc(&table, (size_t)cap * lay.slot_bytes), "hash table alloc");
      CK(launch_init_slots(lay, table, cap, st, (uint64_t*)small, 8), "init slots");  // + flags
    }
    if (t_timing) cudaEventRecord(t_ev.e[1], st);
    if (hprof) h_init = hnow();

    AggParams base{};
    base.lay = lay;
    base.table = table;
    base.cap_mask = dense ? 0 : cap - 1;
    base.max_probe = (uint32_t)std::min<uint64_t>(cap, 4096);
    for (int g = 0; g < 4; ++g) base.dense[g] = dense_g[g];
    base.front_slots = front ? P->front_slots : 0;
    base.flags = d_flags;
    fill_smem_layout(base, path == BLU_PATH_DENSE_SMEM ? (uint32_t)D : base.front_slots, base.front_slots > 0);
    uint32_t launches = 0;
    // outputs, sized by the upper bound min(entries, rows)
    const uint64_t U = std::min<uint64_t>(n_entries, total_rows);
    Owner* own = new Owner();
    std::vector<void*> okeys(lay.n_keys, nullptr), ovals(os.n_out, nullptr);
    auto free_owner = [&]() {
      for (void* p : own->dev) cudaFreeAsync(p, st);
      delete own;
    };
    // Output allocation (stream-ordered). The fused kernel needs the pointers at launch; otherwise
    // they are allocated after the aggregation launch, so this host work overlaps the kernel.
    auto alloc_outputs = [&]() -> cudaError_t {
      cudaError_t ae = cudaSuccess;
      for (int k = 0; k < lay.n_keys && ae == cudaSuccess; ++k) {
        ae = U ? cudaMallocAsync(&okeys[k], U * dtype_bytes(lay.key_dtype[k]), st) : cudaSuccess;
        if (okeys[k]) own->dev.push_back(okeys[k]);
      }
      for (int o = 0; o < os.n_out && ae == cudaSuccess; ++o) {
        ae = U ? cudaMallocAsync(&ovals[o], U * dtype_bytes(os.out_dtype[o]), st) : cudaSuccess;
        if (ovals[o]) own->dev.push_back(ovals[o]);
      }
      if (ae != cudaSuccess) cudaGetLastError();
      return ae;
    };
    if (fuse) {
      cudaError_t ae = alloc_outputs();
      if (ae != cudaSuccess) {
        free_owner();
        return cuda_fail(ae, "output alloc");
      }
    }
    FinalParams fp{};
    if (fuse) {
      base.fuse_init = 1;
      base.sync = (uint32_t*)((uint8_t*)small + 16);
      fp.enabled = 1;
      fp.n_out = os.n_out;
      for (int o = 0; o < os.n_out; ++o) {
        fp.out_kind[o] = os.out_kind[o];
        fp.out_field[o] = os.out_field[o];
        fp.out_field2[o] = os.out_field2[o];
        fp.out_dtype[o] = os.out_dtype[o];
        fp.out_vals[o] = ovals[o];
      }
      for (int k = 0; k < lay.n_keys; ++k) fp.out_keys[k] = okeys[k];
      fp.n_groups = d_ngroups;
    }
    {
      cudaError_t fe = feed(base, &launches, w, fuse ? &fp : nullptr);
      if (fe != cudaSuccess) {
        cudaGetLastError();
        free_owner();
        return cuda_fail(fe, "aggregate launch");
      }
    }
    if (t_timing) cudaEventRecord(t_ev.e[2], st);
    if (hprof) h_feed = hnow();
    if (!fuse) {
      cudaError_t ae = alloc_outputs();
      if (ae != cudaSuccess) {
        free_owner();
        return cuda_fail(ae, "output alloc");
      }
    }

    if (hprof) h_alloc = hnow();
    if (U && !fuse) {
      CompactParams cp{};
      cp.lay = lay;
      cp.source = dense ? 1 : 0;
      cp.table = table;
      for (int g = 0; g < 4; ++g) cp.dense[g] = dense_g[g];
      cp.n_entries = n_entries;
      cp.partial = partial ? 1 : 0;
      cp.n_out = os.n_out;
      for (int o = 0; o < os.n_out; ++o) {
        cp.out_kind[o] = os.out_kind[o];
        cp.out_field[o] = os.out_field[o];
        cp.out_field2[o] = os.out_field2[o];
        cp.out_dtype[o] = os.out_dtype[o];
        cp.out_vals[o] = ovals[o];
      }
      for (int k = 0; k < lay.n_keys; ++k) cp.out_keys[k] = okeys[k];
      cp.block_counts = d_bcounts;
      cp.block_offsets = d_boffs;
      cp.n_groups = d_ngroups;
      int ce = launch_compact(cp, st, nullptr);
      if (ce) {
        free_owner();
        return cuda_fail((cudaError_t)ce, "compaction launch");
      }
    }
    if (t_timing) cudaEventRecord(t_ev.e[3], st);
    if (hprof) h_compact = hnow();
    uint64_t* hs = pinned_scratch();
    uint64_t hbuf[2] = {0, 0};
    uint64_t* dst = hs ? hs : hbuf;
    cudaError_t ce = cudaMemcpyAsync(dst, small, 16, cudaMemcpyDeviceToHost, st);
    if (ce == cudaSuccess) ce = cudaStreamSynchronize(st);
    if (ce == cudaSuccess) w.drained();
    if (ce != cudaSuccess) {
      cudaGetLastError();
      free_owner();
      return cuda_fail(ce, "execute");
    }
    uint32_t flags = (uint32_t)dst[0];
    uint64_t ng = dst[1];
    if (hprof) {
      h_sync = hnow();
      auto us = [](std::chrono::steady_clock::time_point a, std::chrono::steady_clock::time_point b) {
        return std::chrono::duration<double, std::micro>(b - a).count();
      };
      fprintf(stderr, "[blugby host] us: init %.1f | feed %.1f | out-alloc %.1f | compact %.1f | sync-wait %.1f\n",
              us(h_entry, h_init), us(h_init, h_feed), us(h_feed, h_alloc), us(h_alloc, h_compact), us(h_compact, h_sync));
    }
    if (t_timing) {
      float a = 0, b = 0, c = 0;
      cudaEventElapsedTime(&a, t_ev.e[0], t_ev.e[1]);
      cudaEventElapsedTime(&b, t_ev.e[1], t_ev.e[2]);
      cudaEventElapsedTime(&c, t_ev.e[2], t_ev.e[3]);
      tm.init_ms += a;
      tm.aggregate_ms += b;
      tm.compact_ms += c;
      tm.aggregate_launches += launches;
      for (size_t i = 0; i + 3 <= t_pev.used; i += 3) {
        float x = 0, y = 0;
        cudaEventElapsedTime(&x, t_pev.ev[i], t_pev.ev[i + 1]);
        cudaEventElapsedTime(&y, t_pev.ev[i + 1], t_pev.ev[i + 2]);
        tm.scatter_ms += x;
        tm.pass2_ms += y;
        tm.part_chunks += 1;
        if (t_pev.gates && i / 3 < 256) tm.part_fallbacks += t_pev.gates[i / 3];
      }
      t_pev.used = 0;
    }
    if (flags & FLAG_KEY_RANGE) {
      free_owner();
      return fail(BLU_E_KEY_RANGE, "a key code is outside [0, dict_size) or a sparse code is negative");
    }
    if ((flags & FLAG_OVERFLOW) && !dense) {
      free_owner();
      cap *= 4;
      ++retries;
      if (cap > (1ull << 40)) return fail(BLU_E_OOM, "hash table regrow beyond 2^40 slots");
      continue;
    }
    // success
    P->retries_last.store(retries);
    out->n_groups = ng;
    out->n_keys = lay.n_keys;
    out->is_partial = partial ? 1 : 0;
    out->is_host = host_out ? 1 : 0;
    void** kc = (void**)calloc(std::max(1, lay.n_keys), sizeof(void*));
    void** vc = (void**)calloc(std::max(1, os.n_out), sizeof(void*));
    for (int k = 0; k < lay.n_keys; ++k) kc[k] = okeys[k];
    for (int o = 0; o < os.n_out; ++o) vc[o] = ovals[o];
    if (host_out) {
      // copy to host (pageable memory owned by the result) through two pinned bounce buffers, so the
      // D2H runs at the pinned rate and overlaps the host-side copies; release the device outputs
      Owner* hown = new Owner();
      cudaError_t se = cudaSuccess;
      auto take = [&](const void* dsrc, size_t b) -> void* {
        void* h = host_get(b);
        if (!h) {
          se = cudaErrorMemoryAllocation;
          return nullptr;
        }
        hown->host.push_back(h);
        if (b && se == cudaSuccess) se = cudaMemcpyAsync(h, dsrc, b, cudaMemcpyDeviceToHost, st);
        return h;
      };
      for (int k = 0; k < lay.n_keys; ++k) kc[k] = take(okeys[k], ng * dtype_bytes(lay.key_dtype[k]));
      for (int o = 0; o < os.n_out; ++o) vc[o] = take(ovals[o], ng * dtype_bytes(os.out_dtype[o]));
      if (se == cudaSuccess) se = cudaStreamSynchronize(st);
      free_owner();
      own = hown;
      if (se != cudaSuccess) {
        for (void* h : hown->host) host_put(h);
        delete hown;
        free(kc);
        free(vc);
        return cuda_fail(se, "result D2H");
      }
    }
    if (partial) {
      out->n_states = os.n_out;
      out->state_cols = vc;
      out->agg_cols = nullptr;
    } else {
      out->n_aggs = os.n_out;
      out->agg_cols = vc;
      out->state_cols = nullptr;
    }
    out->key_cols = kc;
    out->_owner = own;
    if (t_timing) {
      tm.retries = retries;
      if (h2d_ms_acc) tm.h2d_ms = *h2d_ms_acc;
      tm.total_ms = tm.init_ms + tm.aggregate_ms + tm.compact_ms;
      memcpy(tm.kernel, t_last_kernel, sizeof tm.kernel);
      t_last = tm;
    }
    return BLU_OK;
  }
}

static bool nonnull_cols(const void* const* cols, int n) {
  if (n == 0) return true;
  if (!cols) return false;
  for (int i = 0; i < n; ++i)
    if (!cols[i]) return false;
  return true;
}

// Partitioned path (b): per chunk of rows, pass 1 scatters rows into P->parts buckets (partition
// buffers in HBM), pass 2 aggregates bucket by bucket (one persistent launch). If any bucket
// overflows its capacity (heavily skewed keys), a device-side gate skips pass 2 and runs the
// one-pass kernel over the chunk's original rows instead. No host synchronisation.
static cudaError_t partitioned_feed(const blu_gby_plan_s* P, AggParams& base, const void* const* keys,
                                    const void* const* vals, uint64_t n, cudaStream_t st, uint32_t* launches,
                                    Work& w) {
  static const bool hdbg = benv("BLU_GBY_DEBUG_HOST") != nullptr;
  auto now = [] { return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now().time_since_epoch()).count(); };
  const double h0 = now();
  const Layout& L = P->lay;
  const uint32_t B = P->parts;
  if (!P->part_smem && B > kMaxSegs) return cudaErrorInvalidConfiguration;  // the planner clamps to kMaxSegs
  size_t row_bytes = 8;
  for (int c = 0; c < L.n_vals; ++c) row_bytes += dtype_bytes(L.val_dtype[c]);
  // Chunk rows: decided once per plan from the free memory (cudaMemGetInfo and the pool queries are
  // host-side calls that would otherwise sit between this query's launches every time).
  uint64_t M = P->part_chunk.load();
  if (M == 0) {
    size_t free_b = 0, total_b = 0;
    cudaMemGetInfo(&free_b, &total_b);
    {  // memory cached by the stream-ordered pool (reserved, not in use) is available too
      int dev = 0;
      cudaGetDevice(&dev);
      cudaMemPool_t pool;
      uint64_t reserved = 0, used = 0;
      if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess &&
          cudaMemPoolGetAttribute(pool, cudaMemPoolAttrReservedMemCurrent, &reserved) == cudaSuccess &&
          cudaMemPoolGetAttribute(pool, cudaMemPoolAttrUsedMemCurrent, &used) == cudaSuccess && reserved > used)
        free_b += (size_t)(reserved - used);
      cudaGetLastError();
    }
    free_b += cache_idle_bytes();  // idle workspace blocks are reusable
    uint64_t budget_rows = (uint64_t)((double)free_b * 0.6 / (double)row_bytes / 1.1);
    M = std::max<uint64_t>(budget_rows, 1ull << 22);
    P->part_chunk.store(M);
  }
  // two-level scatter (bucket tables with >= 256 buckets; BLU_GBY_PART_2LEVEL=0 disables): B1 first-level buckets, each split
  // into B / B1 second-level buckets by a second scatter, instead of one B-way scatter (a 2048-way
  // scatter writes ~2 rows per bucket per tile); needs a second set of partition buffers
  const char* tl = benv("BLU_GBY_PART_2LEVEL");
  uint32_t B1 = (P->part_smem && !(tl && tl[0] == '0') && B >= 256) ? two_level_b1(B) : 0u;
  if (const char* b1 = benv("BLU_GBY_PART_B1"))  // experiment: first-level fan-out (power of two < B)
    if (B1 && atoi(b1) >= 2 && (uint32_t)atoi(b1) < B && !((uint32_t)atoi(b1) & ((uint32_t)atoi(b1) - 1))) B1 = (uint32_t)atoi(b1);
  if (B1) M = std::max<uint64_t>(M / 2, 1ull << 22);
  M = std::min<uint64_t>(n, M);
  if (const char* cr = benv("BLU_GBY_PART_CHUNK")) M = std::min<uint64_t>(n, std::max<uint64_t>(1024, strtoull(cr, 0, 10)));
  // bucket capacity: the mean plus slack for the spread of the number of GROUPS per bucket (keys
  // hash uniformly: relative sd 1/sqrt(est/B); 6 sd) and of rows per group; heavier skew overflows a
  // bucket and takes the gated one-pass fallback
  // TMA bulk write-out of the staged runs (every value column 8 bytes; BLU_GBY_SCATTER_TMA=0 turns it
  // off): each (tile, bucket) run is padded to an even row count with an empty-key record the readers
  // skip. C3 scatter 19.4 -> 18.2 ms, C5 22.1 -> 20.0 ms per chunk
  bool tma = true;
  {
    const char* tm = benv("BLU_GBY_SCATTER_TMA");
    if (tm && tm[0] == '0') tma = false;
    for (int c = 0; c < L.n_vals; ++c) tma = tma && dtype_bytes(L.val_dtype[c]) == 8;
    // the padded staging must fit the scatter's shared memory at the widest histogram of this plan
    const uint32_t bins = B1 ? std::max<uint32_t>(B1, B / B1) : B;
    tma = tma && scatter_smem(L.n_vals, bins, true) <= 232448;
  }
  const double gpb = std::max(1.0, (double)P->est_groups / (double)B);
  // padding: at most one row per (tile, bucket) run, i.e. a fraction ~ bins / (2 x tile rows) of a
  // bucket's rows; reserve twice that (tiles hold >= 2048 rows)
  const double pad = tma ? (double)(B1 ? B / B1 : B) / 2048.0 : 0.0;
  const double slack = 1.03 + std::min(1.0, 6.0 / std::sqrt(gpb)) + pad;
  uint64_t seg_cap = ((uint64_t)((double)((M + B - 1) / B) * slack) + 4096 + 63) & ~63ull;
  uint64_t rows_alloc = seg_cap * B;
  void* kbuf = nullptr;
  void* vbuf[kMaxVals] = {};
  void* meta = nullptr;
  cudaError_t e = w.alloc(&kbuf, rows_alloc * 8);
  for (int c = 0; c < L.n_vals && e == cudaSuccess; ++c) e = w.alloc(&vbuf[c], rows_alloc * dtype_bytes(L.val_dtype[c]));
  if (e == cudaSuccess) e = w.alloc(&meta, (size_t)B * 16 + 64);
  // first-level buffers of the two-level scatter
  uint64_t seg_cap1 = 0;
  void* kbuf1 = nullptr;
  void* vbuf1[kMaxVals] = {};
  uint64_t* d_cursor1 = nullptr;
  if (B1 && e == cudaSuccess) {
    const double gpb1 = std::max(1.0, (double)P->est_groups / (double)B1);
    const double slack1 = 1.03 + std::min(1.0, 6.0 / std::sqrt(gpb1)) + (tma ? (double)B1 / 2048.0 : 0.0);  // as above
    // a multiple of the second-level scatter's tile (1024 threads x up to 4 rows): every tile of the
    // one-launch second level lies inside one first-level bucket
    seg_cap1 = ((uint64_t)((double)((M + B1 - 1) / B1) * slack1) + 4096 + 4095) & ~4095ull;
    e = w.alloc(&kbuf1, seg_cap1 * B1 * 8);
    for (int c = 0; c < L.n_vals && e == cudaSuccess; ++c) e = w.alloc(&vbuf1[c], seg_cap1 * B1 * dtype_bytes(L.val_dtype[c]));
    void* m1 = nullptr;
    if (e == cudaSuccess) e = w.alloc(&m1, (size_t)B1 * 8 + 64);
    d_cursor1 = (uint64_t*)m1;
  }
  if (e != cudaSuccess) return e;
  const double h1 = now();
  uint64_t* d_cursor = (uint64_t*)meta;  // B cursors, gate, tile counter
  uint32_t* d_gate = (uint32_t*)(d_cursor + B);
  const uint32_t sgrid = scatter_grid((uint32_t)P->sms, B);
  Layout L2 = L;  // pass 2 reads the packed u64 key as a single sparse key column
  L2.n_keys = 1;
  L2.sparse = 1;
  L2.key_dtype[0] = BLU_I64;
  L2.pad_keys = 1;  // records: empty-key padding rows (TMA write-out) are skipped
  for (uint64_t r0 = 0; r0 < n; r0 += M) {
    const uint64_t m = std::min(M, n - r0);
    if ((e = cudaMemsetAsync(d_cursor, 0, (size_t)B * 8 + 16, st))) return e;
    AggParams p1 = base;
    bool vec = true;
    for (int k = 0; k < L.n_keys; ++k) {
      p1.key[k] = (const uint8_t*)keys[k] + r0 * dtype_bytes(L.key_dtype[k]);
      vec = vec && ptr_aligned(p1.key[k]);
    }
    for (int c = 0; c < L.n_vals; ++c) {
      p1.val[c] = (const uint8_t*)vals[c] + r0 * dtype_bytes(L.val_dtype[c]);
      vec = vec && ptr_aligned(p1.val[c]);
    }
    p1.vec_ok = vec;
    if (vec) {  // 256-bit loads when every column is 32-byte aligned
      bool v32 = true;
      for (int k = 0; k < L.n_keys; ++k) v32 = v32 && ((uintptr_t)p1.key[k] & 31) == 0;
      for (int c = 0; c < L.n_vals; ++c) v32 = v32 && ((uintptr_t)p1.val[c] & 31) == 0;
      if (v32) p1.vec_ok |= 2;
    }
    p1.prefetch = prefetch_enabled();
    p1.n_rows = m;
    ScatterParams sp{};
    sp.B = B;
    {  // bucket = top log2(B) bits of the slot index of the CURRENT table (it may have regrown)
      uint32_t lc = (uint32_t)__builtin_popcountll(base.cap_mask), lb = 0;
      while ((1u << lb) < B) ++lb;
      sp.shift = lc > lb ? lc - lb : 0;
    }
    sp.seg_stride = seg_cap;
    sp.cursor = d_cursor;
    sp.seg_cap = seg_cap;
    sp.out_key = (uint64_t*)kbuf;
    for (int c = 0; c < L.n_vals; ++c) sp.out_val[c] = vbuf[c];
    sp.gate = d_gate;
    sp.tma = tma ? 1u : 0u;
    static const bool dbg = benv("BLU_GBY_DEBUG_PART") != nullptr;
    cudaEvent_t ev[4];
    if (dbg) {
      for (auto& x : ev) cudaEventCreate(&x);
      cudaEventRecord(ev[0], st);
    }
    cudaEvent_t tev[3] = {nullptr, nullptr, nullptr};
    if (t_timing) {
      for (auto& x : tev) x = t_pev.next();
      cudaEventRecord(tev[0], st);
    }
    int le = 0;
    if (!B1) {
      le = launch_scatter(p1, sp, st, sgrid);
      if (le) return (cudaError_t)le;
    } else {
      uint32_t lc = (uint32_t)__builtin_popcountll(base.cap_mask), lb1 = 0, lb2 = 0;
      while ((1u << lb1) < B1) ++lb1;
      while ((1u << lb2) < B / B1) ++lb2;
      const uint32_t shift1 = lc > lb1 ? lc - lb1 : 0;
      if ((e = cudaMemsetAsync(d_cursor1, 0, (size_t)B1 * 8, st))) return e;
      ScatterParams s1 = sp;
      s1.B = B1;
      s1.shift = shift1;
      s1.seg_stride = seg_cap1;
      s1.seg_cap = seg_cap1;
      s1.cursor = d_cursor1;
      s1.out_key = (uint64_t*)kbuf1;
      for (int c = 0; c < L.n_vals; ++c) s1.out_val[c] = vbuf1[c];
      le = launch_scatter(p1, s1, st, scatter_grid((uint32_t)P->sms, B1));
      if (le) return (cudaError_t)le;
      const uint32_t B2 = B / B1;
      // (the segmented kernel keeps the first-level bucket ends in a 256-entry shared array, kMaxInSeg)
      const bool one_launch = benv("BLU_GBY_2LEVEL_ONE") && atoi(benv("BLU_GBY_2LEVEL_ONE")) == 1 && B1 <= 256;
      if (one_launch) {
        // second level as ONE launch over every first-level bucket (segmented input; the first-level
        // counts stay on the device, no host round trip): bucket b1's rows go to [b1 * B2, b1 * B2 + B2).
        // Measured 21.1 vs 19.4 ms for C3 against the per-bucket launches below, so opt-in.
        AggParams q = base;
        q.lay = L2;
        q.gate = d_gate;  // skipped if the first level overflowed
        q.gate_run_if = 0;
        q.key[0] = kbuf1;
        for (int c = 0; c < L.n_vals; ++c) q.val[c] = vbuf1[c];
        q.vec_ok = 3;  // segments start at multiples of 4096 rows (>= the second level's tile)
        q.n_rows = (uint64_t)B1 * seg_cap1;
        q.prefetch = 0;
        q.cap_mask = shift1 >= 64 ? ~0ull : ((1ull << shift1) - 1);  // the slot bits below the first level's
        ScatterParams s2 = sp;
        s2.B = B;
        s2.shift = shift1 > lb2 ? shift1 - lb2 : 0;
        s2.in_seg = seg_cap1;
        s2.in_count = d_cursor1;
        s2.in_B2 = B2;
        le = launch_scatter(q, s2, st, scatter_grid((uint32_t)P->sms, B2));
        if (le) return (cudaError_t)le;
      } else {
        // second level per first-level bucket: one host read of the B1 counts, then B1 launches
        uint64_t* hc = B1 <= 32 ? pinned_scratch() : nullptr;  // 256 pinned bytes (else pageable)
        std::vector<uint64_t> cnt1(B1);
        if ((e = cudaMemcpyAsync(hc ? (void*)hc : (void*)cnt1.data(), d_cursor1, (size_t)B1 * 8, cudaMemcpyDeviceToHost,
                                 st)))
          return e;
        if ((e = cudaStreamSynchronize(st))) return e;
        if (hc) memcpy(cnt1.data(), hc, (size_t)B1 * 8);
        // the B1 launches round-robin over ns streams (BLU_GBY_2LEVEL_STREAMS, default 2) so one
        // launch's ramp and tail overlap another's (C3 29.9 -> 29.3 ms, C5 forced tables 59.1 -> 57.1 ms
        // per 1.6e9 rows; 3 streams: the same); the host sync above orders them after the first level,
        // and st waits for every auxiliary stream before pass 2
        int ns = benv("BLU_GBY_2LEVEL_STREAMS") ? std::max(1, std::min(4, atoi(benv("BLU_GBY_2LEVEL_STREAMS")))) : 2;
        // per thread and device (streams and events belong to the device current at creation)
        thread_local cudaStream_t aux_all[16][3] = {};
        thread_local cudaEvent_t aux_ev_all[16][3] = {};
        int dev_now = 0;
        cudaGetDevice(&dev_now);
        if (dev_now < 0 || dev_now >= 16) ns = 1;
        cudaStream_t* aux = aux_all[dev_now & 15];
        cudaEvent_t* aux_ev = aux_ev_all[dev_now & 15];
        for (int i = 0; i + 1 < ns; ++i)
          if (!aux[i] && (cudaStreamCreateWithFlags(&aux[i], cudaStreamNonBlocking) != cudaSuccess ||
                          cudaEventCreateWithFlags(&aux_ev[i], cudaEventDisableTiming) != cudaSuccess)) {
            cudaGetLastError();
            ns = i + 1;
            break;
          }
        for (uint32_t b1 = 0; b1 < B1; ++b1) {
          const cudaStream_t sb = b1 % ns == 0 ? st : aux[b1 % ns - 1];
          const uint64_t c1 = std::min(cnt1[b1], seg_cap1);  // an overflowed bucket set the gate: fallback
          if (!c1) continue;
          AggParams q = base;
          q.lay = L2;
          q.gate = d_gate;  // skipped if the first level overflowed
          q.gate_run_if = 0;
          q.key[0] = (const uint8_t*)kbuf1 + b1 * seg_cap1 * 8;
          for (int c = 0; c < L.n_vals; ++c)
            q.val[c] = (const uint8_t*)vbuf1[c] + b1 * seg_cap1 * dtype_bytes(L.val_dtype[c]);
          q.vec_ok = 3;  // segments start at multiples of 4096 rows
          q.n_rows = c1;
          q.prefetch = 0;
          q.cap_mask = shift1 >= 64 ? ~0ull : ((1ull << shift1) - 1);  // the slot bits below the first level's
          ScatterParams s2 = sp;
          s2.B = B2;
          s2.shift = shift1 > lb2 ? shift1 - lb2 : 0;
          s2.cursor = d_cursor + (size_t)b1 * B2;
          s2.out_key = (uint64_t*)kbuf + (size_t)b1 * B2 * seg_cap;
          for (int c = 0; c < L.n_vals; ++c)
            s2.out_val[c] = (uint8_t*)vbuf[c] + (size_t)b1 * B2 * seg_cap * dtype_bytes(L.val_dtype[c]);
          le = launch_scatter(q, s2, sb, scatter_grid((uint32_t)P->sms, B2));
          if (le) return (cudaError_t)le;
        }
        for (int i = 0; i + 1 < ns; ++i) {
          if ((e = cudaEventRecord(aux_ev[i], aux[i]))) return e;
          if ((e = cudaStreamWaitEvent(st, aux_ev[i], 0))) return e;
        }
      }
    }
    if (dbg) cudaEventRecord(ev[1], st);
    if (t_timing) cudaEventRecord(tev[1], st);
    // pass 2 (runs if no bucket overflowed)
    AggParams p2 = base;
    p2.lay = L2;
    if (P->part_smem) fill_smem_layout(p2, P->bucket_S, true);
    p2.key[0] = kbuf;
    for (int c = 0; c < L.n_vals; ++c) p2.val[c] = vbuf[c];
    p2.vec_ok = 1;
    p2.n_rows = 0;
    p2.seg_stride = seg_cap;
    p2.seg_count = d_cursor;
    p2.n_segs = B;
    p2.tile_ctr = benv("BLU_GBY_DYN") && atoi(benv("BLU_GBY_DYN")) == 0 ? nullptr : (uint64_t*)(d_cursor + B + 1);
    // bucket tables: TMA bulk L2 prefetch of the piece's tile this many tiles ahead (0 = off)
    p2.prefetch = P->part_smem ? (benv("BLU_GBY_BUCKET_PF") ? (uint32_t)atoi(benv("BLU_GBY_BUCKET_PF")) : 1u)
                               : (benv("BLU_GBY_SEG_PF") ? (uint32_t)atoi(benv("BLU_GBY_SEG_PF")) : 0u);
    if (const char* g = benv("BLU_GBY_GRAB")) p2.grab = (uint32_t)atoi(g);
    p2.gate = d_gate;
    p2.gate_run_if = 0;
    p2.front_slots = 0;
    if (P->part_smem) {
      // bucket-local shared-memory tables: pieces of ~1/div of the mean bucket, whole 4096-row tiles
      // (div 1, one piece per mean bucket: one flush of each group into the global table instead of
      // two; C3 30.4 vs 31.1 ms for div 2, 32.5 for div 4)
      // piece_rows 0: one work item per bucket (the plan's default, no piece prefix in shared memory)
      const uint64_t div = benv("BLU_GBY_PIECE_DIV") ? std::max(1, atoi(benv("BLU_GBY_PIECE_DIV"))) : 1;
      const uint64_t mean = (m + B - 1) / B;
      uint64_t piece = ((mean + div - 1) / div + 4095) / 4096 * 4096;
      piece = std::min<uint64_t>(std::max<uint64_t>(piece, 4096), 1ull << 30);
      p2.piece_rows = P->bucket_whole ? 0 : piece;
      p2.aux_off = bucket_table_bytes(L2, P->bucket_S);
      p2.tile_ctr = (uint64_t*)(d_cursor + B + 1);
      p2.vec_ok = 3;  // segments start at multiples of 64 rows of 8-byte-aligned buffers
      le = launch_bucket(p2, st, (uint32_t)P->sms, P->bucket_smem);
    } else {
      le = launch_aggregate_impl(P, BLU_PATH_HASH_GLOBAL, p2, RecSrc{nullptr, 0}, false, st, P->grid, P->block, 0);
    }
    if (le) return (cudaError_t)le;
    if (t_timing) {
      cudaEventRecord(tev[2], st);
      if (uint32_t* g = t_pev.gate_slot(t_pev.used / 3 - 1)) cudaMemcpyAsync(g, d_gate, 4, cudaMemcpyDeviceToHost, st);
    }
    // fallback one-pass over the chunk's rows (runs only if a bucket overflowed)
    AggParams p3 = p1;
    p3.jit_ok = 0;  // gated fallback, normally a no-op: keep the precompiled kernel
    p3.gate = d_gate;
    p3.gate_run_if = 1;
    if (dbg) cudaEventRecord(ev[2], st);
    le = launch_aggregate_impl(P, BLU_PATH_HASH_GLOBAL, p3, RecSrc{nullptr, 0}, false, st, P->grid, P->block,
                               P->smem_bytes);
    if (le) return (cudaError_t)le;
    if (dbg) {
      cudaEventRecord(ev[3], st);
      cudaEventSynchronize(ev[3]);
      float a = 0, b = 0, c = 0;
      cudaEventElapsedTime(&a, ev[0], ev[1]);
      cudaEventElapsedTime(&b, ev[1], ev[2]);
      cudaEventElapsedTime(&c, ev[2], ev[3]);
      uint32_t gate = 0;
      cudaMemcpy(&gate, d_gate, 4, cudaMemcpyDeviceToHost);
      fprintf(stderr, "[blugby part] chunk rows %llu B %u seg_cap %llu: scatter %.2f ms pass2 %.2f ms fallback %.2f ms gate %u\n",
              (unsigned long long)m, B, (unsigned long long)seg_cap, a, b, c, gate);
      for (auto& x : ev) cudaEventDestroy(x);
    }
    if (launches) *launches += 3;
  }
  if (hdbg) fprintf(stderr, "[blugby host] feed: alloc %.3f ms, launches %.3f ms\n", h1 - h0, now() - h1);
  return cudaSuccess;
}

// Schema column pointers -> kernel columns (the layout's value columns are the schema's).
static blu_status_t execute_device(const blu_gby_plan_s* P, const void* const* keys, const void* const* vals,
                                   uint64_t n, cudaStream_t st, bool partial, blu_gby_result_t* out,
                                   bool host_out = false) {
  if (!P || !out) return fail(BLU_E_INVALID, "NULL plan or out");
  if (n && (!nonnull_cols(keys, P->lay.n_keys) || !nonnull_cols(vals, P->lay.n_vals)))
    return fail(BLU_E_INVALID, "NULL column pointer");
  const Layout& L = P->lay;
  // fused init + compaction needs exactly one aggregation launch
  const bool single = n <= (((uint64_t)P->grid * (1ull << 30)) & ~3ull);
  Feeder feed = [&](AggParams& base, uint32_t* launches, Work& w, const FinalParams* fin) -> cudaError_t {
    base.jit_ok = L.key_words == 2 ? 0 : 1;
    // path (b)/(b') one pass: each warp L2-prefetches its next tile (BLU_GBY_AGG_PREFETCH=0/1)
    const char* ap = benv("BLU_GBY_AGG_PREFETCH");
    base.prefetch = ap ? (uint32_t)atoi(ap) : 0u;
    // hot-key front seeded with the heavy hitters of a row sample (needs a COUNT field to tell
    // seeded keys that received rows from those that did not)
    static const bool no_seed = benv("BLU_GBY_NO_SEED") != nullptr;
    if (base.front_slots > 0 && L.count_field >= 0 && !no_seed && n >= (1u << 16)) {
      void* ws = nullptr;
      cudaError_t e = w.alloc(&ws, front_seed_bytes(base.front_slots));
      if (e) return e;
      AggParams pk = base;
      uint32_t vec = 1;
      for (int k = 0; k < L.n_keys; ++k) {
        pk.key[k] = keys[k];
        if (((uintptr_t)keys[k] & 15) != 0) vec = 0;
      }
      pk.vec_ok = (int32_t)vec;
      // path (b'): a rank image when the bitmap of the domain fits the front's key region
      const bool no_rank = benv("BLU_GBY_NO_RANK_FRONT") != nullptr;
      const uint64_t W = (L.domain + 31) / 32;
      const uint32_t rank_words =
          P->path == BLU_PATH_DIRECT_GLOBAL && !no_rank && L.domain > 0 && W <= base.front_slots ? (uint32_t)W : 0u;
      const uint64_t* front = nullptr;
      const uint64_t* hot = nullptr;
      int rc = launch_front_seed(pk, n, base.front_slots, rank_words, ws, st, (int)P->sms, &front,
                                 rank_words && jit_hot_reg() ? &hot : nullptr);
      if (rc) return (cudaError_t)rc;
      base.hot_key = hot;
      base.front_seed = front;
      base.front_rank_words = rank_words;
    }
    if (P->path == BLU_PATH_HASH_GLOBAL && P->parts > 1 && n >= 4096 * (uint64_t)P->parts)
      return partitioned_feed(P, base, keys, vals, n, st, launches, w);
    return agg_batch(P, P->path, base, keys, vals, n, nullptr, st, P->grid, P->block, P->smem_bytes, launches, fin);
  };
  // fusion only pays where launch latency dominates (<= 16M rows)
  return run_core(P, L, P->path, P->hot_front != 0, P->cap, n, feed, partial, st, out, host_out, nullptr,
                  single && n > 0 && n <= (16ull << 20));
}

}  // namespace blu

using namespace blu;

extern "C" {

void blu_gby_set_timing(int32_t enable) { t_timing = enable != 0; }

blu_status_t blu_gby_last_timing(blu_gby_timing_t* out) {
  if (!out) return fail(BLU_E_INVALID, "NULL out");
  *out = t_last;
  return BLU_OK;
}

uint64_t blu_gby_launch_count(void) { return launches_total(); }

blu_status_t blu_gby_release_workspace(uint64_t* freed) {
  int dev = 0;
  cudaGetDevice(&dev);
  cudaError_t se = cudaDeviceSynchronize();
  if (se != cudaSuccess) {
    cudaGetLastError();
    return fail(BLU_E_CUDA, "release workspace: %s", cudaGetErrorString(se));
  }
  uint64_t t = 0;
  {
    std::lock_guard<std::mutex> lk(g_cache_mu);
    for (auto it = g_cache.begin(); it != g_cache.end();) {
      if (!it->busy && it->dev == dev) {
        t += it->bytes;
        cudaFree(it->p);
        it = g_cache.erase(it);
      } else {
        ++it;
      }
    }
  }
  {  // idle pinned host-result blocks too
    std::lock_guard<std::mutex> lk(g_hcache_mu);
    for (auto it = g_hcache.begin(); it != g_hcache.end();) {
      if (!it->busy) {
        t += it->bytes;
        cudaFreeHost(it->p);
        it = g_hcache.erase(it);
      } else {
        ++it;
      }
    }
  }
  if (freed) *freed = t;
  return BLU_OK;
}

blu_status_t blu_gby_jit_probe(blu_gby_plan_t P, char* log, uint32_t log_cap, int32_t* n_programs) {
  env_snapshot();
  if (!P) return fail(BLU_E_INVALID, "NULL plan");
  if (log && log_cap) log[0] = 0;
  if (n_programs) *n_programs = 0;
  if (!jit_enabled() || P->lay.key_words == 2 || P->lay.has_q) return fail(BLU_E_UNSUPPORTED, "no JIT kernels for this plan");
  JitProbe pr;
  jit_probe_begin(&pr);
  AggParams p{};
  p.lay = P->lay;
  p.jit_ok = 1;
  p.n_rows = 1;
  p.front_slots = P->hot_front ? P->front_slots : 0;
  fill_smem_layout(p, P->path == BLU_PATH_DENSE_SMEM ? (uint32_t)P->lay.domain : p.front_slots, p.front_slots > 0);
  int rc = launch_aggregate_impl(P, P->path, p, RecSrc{nullptr, 0}, false, nullptr, P->grid, P->block, P->smem_bytes);
  if (P->path == BLU_PATH_HASH_GLOBAL && P->parts > 1) {  // partitioned mode: scatter + segment pass
    ScatterParams sp{};
    sp.B = P->parts;
    if (!rc) rc = launch_scatter(p, sp, nullptr, P->grid);
    bool wide8 = true;  // the TMA write-out variant (8-byte value columns)
    for (int c = 0; c < P->lay.n_vals; ++c) wide8 = wide8 && dtype_bytes(P->lay.val_dtype[c]) == 8;
    if (wide8) {
      sp.tma = 1;
      if (!rc) rc = launch_scatter(p, sp, nullptr, P->grid);
    }
    AggParams p2 = p;
    p2.lay.n_keys = 1;
    p2.lay.sparse = 1;
    p2.lay.key_dtype[0] = BLU_I64;
    if (P->part_smem) {
      fill_smem_layout(p2, P->bucket_S, true);
      if (!rc) rc = launch_bucket(p2, nullptr, (uint32_t)P->sms, P->bucket_smem);
    } else {
      p2.seg_stride = 1;
      if (!rc) rc = launch_aggregate_impl(P, P->path, p2, RecSrc{nullptr, 0}, false, nullptr, P->grid, P->block, P->smem_bytes);
    }
  }
  jit_probe_end();
  if (n_programs) *n_programs = pr.programs;
  if (log && log_cap) {
    strncpy(log, pr.log.c_str(), log_cap - 1);
    log[log_cap - 1] = 0;
  }
  if (rc || pr.failed || !pr.programs)
    return fail(BLU_E_UNSUPPORTED, "JIT probe: %d of %d programs failed", pr.failed, pr.programs);
  return BLU_OK;
}

blu_status_t blu_gby_read_roofline(const void* const* cols, const uint64_t* bytes, int32_t n_cols, void* stream,
                                   uint64_t* dev_out) {
  env_snapshot();
  if (n_cols < 1 || n_cols > kMaxKeys + kMaxVals || !cols || !bytes || !dev_out)
    return fail(BLU_E_INVALID, "bad read_roofline arguments");
  for (int j = 0; j < n_cols; ++j)
    if (!cols[j] || ((uintptr_t)cols[j] & 15) || (bytes[j] & 15)) return fail(BLU_E_INVALID, "column %d: not 16-byte aligned", j);
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  CK(launch_read_roofline(cols, bytes, n_cols, stream, dev_out, sms), "read roofline");
  return BLU_OK;
}

blu_status_t blu_gby_execute(blu_gby_plan_t P, const void* const* key_cols, const void* const* val_cols, uint64_t n_rows,
                             void* stream, blu_gby_result_t* out) {
  env_snapshot();
  return execute_device(P, key_cols, val_cols, n_rows, (cudaStream_t)stream, false, out);
}

blu_status_t blu_gby_execute_partial(blu_gby_plan_t P, const void* const* key_cols, const void* const* val_cols,
                                     uint64_t n_rows, void* stream, blu_gby_result_t* out) {
  env_snapshot();
  return execute_device(P, key_cols, val_cols, n_rows, (cudaStream_t)stream, true, out);
}

blu_status_t blu_gby_execute_host(blu_gby_plan_t P, const void* const* hkeys, const void* const* hvals, uint64_t n,
                                  void* stream, blu_gby_result_t* out) {
  env_snapshot();
  if (!P || !out) return fail(BLU_E_INVALID, "NULL plan or out");
  if (n && (!nonnull_cols(hkeys, P->lay.n_keys) || !nonnull_cols(hvals, P->lay.n_vals)))
    return fail(BLU_E_INVALID, "NULL column pointer");
  cudaStream_t st = (cudaStream_t)stream;
  const Layout& L = P->lay;
  size_t row_bytes = 0;
  for (int k = 0; k < L.n_keys; ++k) row_bytes += dtype_bytes(L.key_dtype[k]);
  for (int c = 0; c < L.n_vals; ++c) row_bytes += dtype_bytes(L.val_dtype[c]);
  // Partitioned hash plans (tables larger than L2): a streamed one-pass aggregation would update a
  // DRAM-resident table at random, so when the columns fit in a quarter of the free device memory they
  // are copied whole (pinned-rate H2D) and the query runs as on device columns (scatter + pass 2).
  if (n && P->path == BLU_PATH_HASH_GLOBAL && P->parts > 1 && !L.has_q && L.key_words == 1) {
    size_t free_b = 0, total_b = 0;
    cudaMemGetInfo(&free_b, &total_b);
    cudaGetLastError();
    if ((double)n * (double)row_bytes < 0.25 * (double)(free_b + cache_idle_bytes())) {
      setup_pool();
      std::vector<void*> dk(L.n_keys, nullptr), dv(L.n_vals, nullptr);
      auto release = [&]() {
        for (void* q : dk) if (q) cudaFreeAsync(q, st);
        for (void* q : dv) if (q) cudaFreeAsync(q, st);
      };
      cudaError_t e = cudaSuccess;
      for (int k = 0; k < L.n_keys && !e; ++k) {
        const size_t b = n * dtype_bytes(L.key_dtype[k]);
        e = cudaMallocAsync(&dk[k], b, st);
        if (!e) e = cudaMemcpyAsync(dk[k], hkeys[k], b, cudaMemcpyHostToDevice, st);
      }
      for (int c = 0; c < L.n_vals && !e; ++c) {
        const size_t b = n * dtype_bytes(L.val_dtype[c]);
        e = cudaMallocAsync(&dv[c], b, st);
        if (!e) e = cudaMemcpyAsync(dv[c], hvals[c], b, cudaMemcpyHostToDevice, st);
      }
      if (e) {
        cudaGetLastError();
        release();
        cudaStreamSynchronize(st);
        return cuda_fail(e, "host columns to device");
      }
      blu_status_t s = execute_device(P, dk.data(), dv.data(), n, st, false, out, true);
      release();
      return s;
    }
  }
  // otherwise: chunks of ~256 MB of rows through two staging buffers, a multiple of 4 rows
  uint64_t chunk = std::max<uint64_t>(4, ((256ull << 20) / std::max<size_t>(row_bytes, 1)) & ~3ull);
  if (chunk > n) chunk = (n + 3) & ~3ull;
  const int ncols = L.n_keys + L.n_vals;
  setup_pool();
  void* stage[2] = {nullptr, nullptr};
  cudaStream_t cs = nullptr;
  cudaEvent_t ready[2] = {nullptr, nullptr}, freed[2] = {nullptr, nullptr}, t0 = nullptr, t1 = nullptr;
  auto cleanup = [&]() {
    if (cs) cudaStreamSynchronize(cs);  // H2D copies still queued on cs must land before the frees
    for (int b = 0; b < 2; ++b) {
      if (stage[b]) cudaFreeAsync(stage[b], st);
      if (ready[b]) cudaEventDestroy(ready[b]);
      if (freed[b]) cudaEventDestroy(freed[b]);
    }
    if (t0) cudaEventDestroy(t0);
    if (t1) cudaEventDestroy(t1);
    if (cs) {
      cudaStreamSynchronize(cs);
      cudaStreamDestroy(cs);
    }
  };
  if (n) {
    for (int b = 0; b < 2; ++b) {
      if (cudaMallocAsync(&stage[b], chunk * row_bytes + 16 * ncols, st) != cudaSuccess) {
        cudaGetLastError();
        cleanup();
        return fail(BLU_E_OOM, "staging buffers");
      }
      cudaEventCreateWithFlags(&ready[b], cudaEventDisableTiming);
      cudaEventCreateWithFlags(&freed[b], cudaEventDisableTiming);
    }
    cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking);
    cudaEventCreate(&t0);
    cudaEventCreate(&t1);
  }
  float h2d_ms = 0.f;
  Feeder feed = [&](AggParams& base, uint32_t* launches, Work&, const FinalParams*) -> cudaError_t {
    if (!n) return cudaSuccess;
    base.jit_ok = L.key_words == 2 ? 0 : 1;
    cudaEventRecord(t0, st);
    cudaStreamWaitEvent(cs, t0, 0);  // staging buffers are allocated on st
    uint64_t nchunks = (n + chunk - 1) / chunk;
    for (uint64_t i = 0; i < nchunks; ++i) {
      int b = (int)(i & 1);
      uint64_t r0 = i * chunk, m = std::min(chunk, n - r0);
      if (i >= 2) cudaStreamWaitEvent(cs, freed[b], 0);
      const void* dk[kMaxKeys];
      const void* dv[kMaxVals];
      uint8_t* ptr = (uint8_t*)stage[b];
      for (int k = 0; k < L.n_keys; ++k) {
        size_t eb = dtype_bytes(L.key_dtype[k]);
        cudaMemcpyAsync(ptr, (const uint8_t*)hkeys[k] + r0 * eb, m * eb, cudaMemcpyHostToDevice, cs);
        dk[k] = ptr;
        ptr += (chunk * eb + 15) / 16 * 16;
      }
      for (int c = 0; c < L.n_vals; ++c) {
        size_t eb = dtype_bytes(L.val_dtype[c]);
        cudaMemcpyAsync(ptr, (const uint8_t*)hvals[c] + r0 * eb, m * eb, cudaMemcpyHostToDevice, cs);
        dv[c] = ptr;
        ptr += (chunk * eb + 15) / 16 * 16;
      }
      cudaEventRecord(ready[b], cs);
      cudaStreamWaitEvent(st, ready[b], 0);
      cudaError_t e = agg_batch(P, P->path, base, dk, dv, m, nullptr, st, P->grid, P->block, P->smem_bytes, launches);
      if (e) return e;
      cudaEventRecord(freed[b], st);
    }
    cudaEventRecord(t1, st);
    return cudaGetLastError();
  };
  blu_status_t s = run_core(P, L, P->path, P->hot_front != 0, P->cap, n, feed, false, st, out, true, nullptr);
  if (s == BLU_OK && n && t_timing) {
    cudaEventElapsedTime(&h2d_ms, t0, t1);  // copy+aggregate pipeline span
    t_last.h2d_ms = h2d_ms;
  }
  cleanup();
  return s;
}

static blu_status_t merge_impl(blu_gby_plan_t P, const blu_gby_result_t* parts, int32_t np, void* stream, bool partial_out,
                               blu_gby_result_t* out) {
  if (!P || !out || (np > 0 && !parts) || np < 0) return fail(BLU_E_INVALID, "bad merge arguments");
  cudaStream_t st = (cudaStream_t)stream;
  const Layout& M = P->merge_lay;
  uint64_t total = 0;
  for (int i = 0; i < np; ++i) {
    if (!parts[i].is_partial || parts[i].is_host) return fail(BLU_E_INVALID, "partial %d: not a device partial result", i);
    if (parts[i].n_states != M.n_vals || parts[i].n_keys != M.n_keys) return fail(BLU_E_INVALID, "partial %d: schema mismatch", i);
    total += parts[i].n_groups;
  }
  uint64_t est = std::max<uint64_t>(1, std::min<uint64_t>(total, std::max<uint64_t>(P->est_groups, 1)));
  uint64_t cap = 1024;
  while ((double)cap * 0.7 < (double)est) cap <<= 1;
  uint32_t grid = (uint32_t)P->sms * 8, block = 256;
  Feeder feed = [&](AggParams& base, uint32_t* launches, Work&, const FinalParams*) -> cudaError_t {
    for (int i = 0; i < np; ++i) {
      if (!parts[i].n_groups) continue;
      cudaError_t e = agg_batch(P, BLU_PATH_HASH_GLOBAL, base, (const void* const*)parts[i].key_cols,
                                (const void* const*)parts[i].state_cols, parts[i].n_groups, nullptr, st, grid, block, 0,
                                launches);
      if (e) return e;
    }
    return cudaSuccess;
  };
  return run_core(P, M, BLU_PATH_HASH_GLOBAL, false, cap, total, feed, partial_out, st, out, false, nullptr);
}

blu_status_t blu_gby_merge(blu_gby_plan_t P, const blu_gby_result_t* parts, int32_t np, void* stream, blu_gby_result_t* out) {
  env_snapshot();
  return merge_impl(P, parts, np, stream, false, out);
}

blu_status_t blu_gby_merge_partial(blu_gby_plan_t P, const blu_gby_result_t* parts, int32_t np, void* stream,
                                   blu_gby_result_t* out) {
  env_snapshot();
  return merge_impl(P, parts, np, stream, true, out);
}

blu_status_t blu_gby_merge_records(blu_gby_plan_t P, const void* records, uint64_t n, void* stream, int32_t partial_out,
                                   blu_gby_result_t* out) {
  env_snapshot();
  if (!P || !out || (n && !records)) return fail(BLU_E_INVALID, "bad merge_records arguments");
  if (P->lay.has_q) return fail(BLU_E_UNSUPPORTED, "merge_records: 128-bit payloads have no record format");
  cudaStream_t st = (cudaStream_t)stream;
  const Layout& M = P->merge_lay;
  uint64_t est = std::max<uint64_t>(1, std::min<uint64_t>(n, std::max<uint64_t>(P->est_groups, 1)));
  uint64_t cap = 1024;
  while ((double)cap * 0.7 < (double)est) cap <<= 1;
  uint32_t grid = (uint32_t)P->sms * 8, block = 256;
  RecSrc rs{(const uint64_t*)records, (uint32_t)((M.key_words == 2 ? 2 : 1) + M.n_vals)};
  Feeder feed = [&](AggParams& base, uint32_t* launches, Work&, const FinalParams*) -> cudaError_t {
    if (!n) return cudaSuccess;
    return agg_batch(P, BLU_PATH_HASH_GLOBAL, base, nullptr, nullptr, n, &rs, st, grid, block, 0, launches);
  };
  return run_core(P, M, BLU_PATH_HASH_GLOBAL, false, cap, n, feed, partial_out != 0, st, out, false, nullptr);
}

blu_status_t blu_gby_execute_dense_state(blu_gby_plan_t P, const void* const* keys, const void* const* vals, uint64_t n,
                                         void* stream, void* const* state_arrays, int32_t init) {
  env_snapshot();
  if (!P || !state_arrays) return fail(BLU_E_INVALID, "NULL plan or state arrays");
  if (P->path == BLU_PATH_HASH_GLOBAL) return fail(BLU_E_UNSUPPORTED, "dense state needs path a or b'");
  if (n && (!nonnull_cols(keys, P->lay.n_keys) || !nonnull_cols(vals, P->lay.n_vals)))
    return fail(BLU_E_INVALID, "NULL column pointer");
  setup_pool();
  cudaStream_t st = (cudaStream_t)stream;
  const Layout& L = P->lay;
  void* dg[4];
  for (int g = 0; g < 4; ++g) {
    dg[g] = state_arrays[g];
    if (L.n_group[g] && !dg[g]) return fail(BLU_E_INVALID, "state array %d is NULL", g);
  }
  if (init) CK(launch_init_dense(L, dg, L.domain, st), "init dense");
  Work w(st);
  void* small = nullptr;
  CK(w.alloc(&small, 64), "flags alloc");
  CK(cudaMemsetAsync(small, 0, 64, st), "memset flags");
  AggParams base{};
  base.lay = L;
  for (int g = 0; g < 4; ++g) base.dense[g] = dg[g];
  base.front_slots = P->hot_front ? P->front_slots : 0;
  base.flags = (uint32_t*)small;
  fill_smem_layout(base, P->path == BLU_PATH_DENSE_SMEM ? (uint32_t)L.domain : base.front_slots, base.front_slots > 0);
  base.jit_ok = L.key_words == 2 ? 0 : 1;
  uint32_t launches = 0;
  if (t_timing) {
    t_ev.make();
    cudaEventRecord(t_ev.e[1], st);
  }
  CK(agg_batch(P, P->path, base, keys, vals, n, nullptr, st, P->grid, P->block, P->smem_bytes, &launches), "aggregate");
  if (t_timing) cudaEventRecord(t_ev.e[2], st);
  uint64_t* hs = pinned_scratch();
  uint64_t hb[2] = {0, 0};
  uint64_t* dst = hs ? hs : hb;
  CK(cudaMemcpyAsync(dst, small, 8, cudaMemcpyDeviceToHost, st), "flags D2H");
  CK(cudaStreamSynchronize(st), "sync");
  w.drained();
  if (t_timing) {  // the aggregation launches of this call (multi-GPU path (a): the per-rank kernel)
    blu_gby_timing_t tm{};
    cudaEventElapsedTime(&tm.aggregate_ms, t_ev.e[1], t_ev.e[2]);
    tm.aggregate_launches = launches;
    tm.total_ms = tm.aggregate_ms;
    memcpy(tm.kernel, t_last_kernel, sizeof tm.kernel);
    t_last = tm;
  }
  if ((uint32_t)dst[0] & FLAG_KEY_RANGE) return fail(BLU_E_KEY_RANGE, "a key code is outside [0, dict_size)");
  return BLU_OK;
}

blu_status_t blu_gby_finalize_dense_state(blu_gby_plan_t P, void* const* state_arrays, void* stream, blu_gby_result_t* out) {
  env_snapshot();
  if (!P || !state_arrays || !out) return fail(BLU_E_INVALID, "NULL argument");
  if (P->path == BLU_PATH_HASH_GLOBAL) return fail(BLU_E_UNSUPPORTED, "dense state needs path a or b'");
  cudaStream_t st = (cudaStream_t)stream;
  const Layout& L = P->lay;
  // Reuse run_core with a feeder that copies the caller's state in place of init+aggregate.
  Feeder feed = [&](AggParams& base, uint32_t*, Work&, const FinalParams*) -> cudaError_t {
    for (int g = 0; g < 4; ++g) {
      size_t b = (size_t)L.n_group[g] * L.domain * 8;
      if (b) {
        cudaError_t e = cudaMemcpyAsync(base.dense[g], state_arrays[g], b, cudaMemcpyDeviceToDevice, st);
        if (e) return e;
      }
    }
    return cudaSuccess;
  };
  return run_core(P, L, P->path, false, L.domain, L.domain, feed, false, st, out, false, nullptr);
}

blu_status_t blu_gby_execute_records(blu_gby_plan_t P, const void* records, uint64_t n, void* stream, int32_t partial_out,
                                     blu_gby_result_t* out) {
  env_snapshot();
  if (!P || !out || (n && !records)) return fail(BLU_E_INVALID, "bad execute_records arguments");
  if (P->lay.has_q) return fail(BLU_E_UNSUPPORTED, "execute_records: 128-bit payloads have no record format");
  cudaStream_t st = (cudaStream_t)stream;
  const Layout& L = P->lay;
  uint64_t est = std::max<uint64_t>(1, std::min<uint64_t>(n, std::max<uint64_t>(P->est_groups, 1)));
  uint64_t cap = 1024;
  while ((double)cap * 0.7 < (double)est) cap <<= 1;
  uint32_t grid = (uint32_t)P->sms * 8, block = 256;
  RecSrc rs{(const uint64_t*)records, (uint32_t)((L.key_words == 2 ? 2 : 1) + L.n_vals)};
  Feeder feed = [&](AggParams& base, uint32_t* launches, Work&, const FinalParams*) -> cudaError_t {
    if (!n) return cudaSuccess;
    return agg_batch(P, BLU_PATH_HASH_GLOBAL, base, nullptr, nullptr, n, &rs, st, grid, block, 0, launches);
  };
  return run_core(P, L, BLU_PATH_HASH_GLOBAL, false, cap, n, feed, partial_out != 0, st, out, false, nullptr);
}

blu_status_t blu_gby_partition_rows(blu_gby_plan_t P, const void* const* key_cols, const void* const* val_cols,
                                    uint64_t n, int32_t n_parts, void* stream, void* send_buf, uint64_t* send_counts) {
  env_snapshot();
  if (!P || !send_counts || n_parts < 1 || n_parts > 1024) return fail(BLU_E_INVALID, "bad partition_rows arguments");
  if (P->lay.has_q) return fail(BLU_E_UNSUPPORTED, "partition_rows: 128-bit payloads have no record format");
  if (n && (!send_buf || !nonnull_cols(key_cols, P->lay.n_keys) || !nonnull_cols(val_cols, P->lay.n_vals)))
    return fail(BLU_E_INVALID, "NULL column or send_buf");
  cudaStream_t st = (cudaStream_t)stream;
  setup_pool();
  if (!n) {
    for (int i = 0; i < n_parts; ++i) send_counts[i] = 0;
    return BLU_OK;
  }
  Work w(st);
  void* tmp = nullptr;
  CK(w.alloc(&tmp, 8 * (size_t)n_parts + 16 + partition_scratch_bytes(n, n_parts)), "partition workspace");
  uint64_t* d_counts = (uint64_t*)tmp;
  uint32_t* d_flags = (uint32_t*)(d_counts + n_parts);
  CK(cudaMemsetAsync(d_flags, 0, 16, st), "memset");
  CK(launch_partition(P->lay, key_cols, val_cols, n, n_parts, send_buf, d_counts, (uint8_t*)tmp + 8 * (size_t)n_parts + 16,
                      st, d_flags),
     "partition rows");
  uint32_t flags = 0;
  CK(cudaMemcpyAsync(send_counts, d_counts, 8 * (size_t)n_parts, cudaMemcpyDeviceToHost, st), "counts D2H");
  CK(cudaMemcpyAsync(&flags, d_flags, 4, cudaMemcpyDeviceToHost, st), "flags D2H");
  CK(cudaStreamSynchronize(st), "sync");
  w.drained();
  if (flags & FLAG_KEY_RANGE) return fail(BLU_E_KEY_RANGE, "a key code is outside its dictionary (or negative)");
  return BLU_OK;
}

blu_status_t blu_gby_partition(blu_gby_plan_t P, const blu_gby_result_t* partial, int32_t n_parts, void* stream, void* send_buf,
                               uint64_t* send_counts) {
  env_snapshot();
  if (!P || !partial || !send_counts || n_parts < 1 || n_parts > 1024) return fail(BLU_E_INVALID, "bad partition arguments");
  if (P->lay.has_q) return fail(BLU_E_UNSUPPORTED, "partition: 128-bit payloads have no record format");
  if (!partial->is_partial || partial->is_host) return fail(BLU_E_INVALID, "partition needs a device partial result");
  if (partial->n_groups && !send_buf) return fail(BLU_E_INVALID, "NULL send_buf");
  cudaStream_t st = (cudaStream_t)stream;
  setup_pool();
  if (!partial->n_groups) {
    for (int i = 0; i < n_parts; ++i) send_counts[i] = 0;
    return BLU_OK;
  }
  Work w(st);
  void* tmp = nullptr;
  CK(w.alloc(&tmp, 8 * (size_t)n_parts + 16 + partition_scratch_bytes(partial->n_groups, n_parts)), "partition workspace");
  uint64_t* d_counts = (uint64_t*)tmp;
  CK(launch_partition(P->merge_lay, (const void* const*)partial->key_cols, (const void* const*)partial->state_cols,
                      partial->n_groups, n_parts, send_buf, d_counts, (uint8_t*)tmp + 8 * (size_t)n_parts + 16, st),
     "partition");
  CK(cudaMemcpyAsync(send_counts, d_counts, 8 * (size_t)n_parts, cudaMemcpyDeviceToHost, st), "counts D2H");
  CK(cudaStreamSynchronize(st), "sync");
  w.drained();
  return BLU_OK;
}

blu_status_t blu_gby_init_table(blu_gby_plan_t P, void* dev_table, uint64_t n_slots, void* stream) {
  env_snapshot();
  if (!P || (n_slots && !dev_table)) return fail(BLU_E_INVALID, "NULL plan or table");
  CK(launch_init_slots(P->lay, dev_table, n_slots, stream), "init slots");
  return BLU_OK;
}

blu_status_t blu_gby_bind_device(int32_t device) {
  CK(cudaSetDevice(device), "cudaSetDevice");
  return BLU_OK;
}

void blu_gby_result_free(blu_gby_result_t* r, void* stream) {
  if (!r) return;
  Owner* o = (Owner*)r->_owner;
  if (o) {
    for (void* p : o->dev) cudaFreeAsync(p, (cudaStream_t)stream);
    for (void* h : o->host) host_put(h);
    delete o;
  }
  free(r->key_cols);
  free(r->agg_cols);
  free(r->state_cols);
  memset(r, 0, sizeof *r);
}

}  // extern "C"
