// blu_internal.h — libblugby internals: plan layout, state-field kinds, kernel parameter blocks.
// Nothing here is shared with oracle/ (the oracle has its own plain definitions).
#pragma once

#include <stdint.h>

#include <atomic>
#include <string>
#include <vector>

#include "blu_gby.h"
#include "blu_params.h"

namespace blu {





struct AggMap {
  int32_t op;
  int32_t val_col;
  int32_t field;   // SUM / MIN / MAX / COUNT field
  int32_t field2;  // AVG: COUNT field
  int32_t out_dtype;
};

}  // namespace blu

struct blu_gby_plan_s {
  // schema copy
  std::vector<blu_key_desc_t> keys;
  std::vector<blu_dtype_t> vals;
  std::vector<blu_agg_desc_t> aggs;
  blu::Layout lay;        // execute: rows of the fact table
  blu::Layout merge_lay;  // merge: rows are (keys, state columns)
  std::vector<blu::AggMap> amap;

  int32_t path;           // blu_path_t
  uint64_t est_groups;
  uint64_t n_rows;
  uint64_t cap;           // hash slots (path b) or D (paths a, b')
  int32_t hot_front;
  int32_t front_wide;  // 1: one 1024-thread CTA per SM with a double-size front
  uint32_t front_slots;   // entries of the shared-memory front
  uint32_t smem_bytes;    // dynamic shared memory of the aggregation kernel
  uint32_t grid, block;
  int32_t sms;
  uint32_t parts;         // path b: buckets of the partitioned two-pass mode (1 = one pass)
  uint32_t part_shift;    // log2(cap) - log2(parts)
  int32_t part_smem;      // partitioned pass 2: 1 = bucket-local shared-memory tables, 0 = L2-resident slices
  uint32_t bucket_S;      // part_smem: entries of the per-CTA bucket table
  uint32_t bucket_smem;   // part_smem: dynamic shared memory of the bucket kernel
  int32_t bucket_whole;   // part_smem: 1 = one work item per bucket (no piece prefix in shared memory)
  mutable std::atomic<uint64_t> part_chunk{0};  // rows per partitioned chunk (decided at first execute)
  mutable std::atomic<uint32_t> retries_last{0};
};

namespace blu {



// Fill S / key_off / soff / colmask / cntmask of p for a shared-memory table of S entries.
void fill_smem_layout(AggParams& p, uint32_t S, bool with_keys);




// Launchers (kernels.cu). All return cudaError_t as int.
int launch_aggregate_impl(const blu_gby_plan_s* P, int path, const AggParams& p, const RecSrc& rs, bool records,
                          void* stream, uint32_t grid, uint32_t block, uint32_t smem,
                          const FinalParams* fin = nullptr);
uint64_t launches_total();
int launch_scatter(const AggParams& p, const ScatterParams& s, void* stream, uint32_t grid);
// Two-level scatter (bucket tables): first-level fan-out for B buckets (32 x B/32 up to 4096 buckets,
// 128 x B/128 above: C5's 16384 tables behind 128 x 128 measured 58.9 vs 74.3 ms for 32 x 512 per
// 1.6e9 rows); second level B / two_level_b1(B).
inline uint32_t two_level_b1(uint64_t B) { return B > 4096 ? 128u : 32u; }
uint32_t scatter_block(uint32_t B);
uint32_t scatter_grid(uint32_t sms, uint32_t B);
size_t scatter_smem(int nv, uint32_t B, bool tma = false);
int launch_bucket(const AggParams& p, void* stream, uint32_t grid, uint32_t smem);
// bucket table sizing: bytes of an S-entry table (keys + SoA fields) and the kernel's total smem
uint32_t bucket_table_bytes(const Layout& L, uint32_t S);
uint32_t bucket_smem_bytes(const Layout& L, uint32_t S, uint32_t B, bool prefix = true);
blu_status_t fail(blu_status_t s, const char* fmt, ...);
int launch_init_slots(const Layout& lay, void* table, uint64_t n_slots, void* stream, uint64_t* zero = nullptr,
                      uint32_t n_zero = 0);
int launch_init_dense(const Layout& lay, void* const dense[4], uint64_t D, void* stream, uint64_t* zero = nullptr,
                      uint32_t n_zero = 0);
int launch_compact(const CompactParams& p, void* stream, uint32_t* launches);
size_t front_seed_bytes(uint32_t S);
int launch_front_seed(const AggParams& base, uint64_t n, uint32_t S, uint32_t rank_words, void* ws, void* stream, int sms,
                      const uint64_t** front_out, const uint64_t** hot_out = nullptr);
int launch_read_roofline(const void* const* cols, const uint64_t* bytes, int n_cols, void* stream, uint64_t* out,
                         int sms);
// S10 owner partition (three launches, no host sync): records of owner o land contiguously at
// [sum of totals[<o], ...); d_totals (n_parts) receives the per-owner record counts; scratch holds
// partition_scratch_bytes(n, n_parts) bytes.
uint32_t partition_ctas(uint64_t n);
uint64_t partition_scratch_bytes(uint64_t n, int32_t n_parts);
int launch_partition(const Layout& lay, const void* const* key_cols, const void* const* state_cols, uint64_t n,
                     int32_t n_parts, void* send_buf, uint64_t* d_totals, void* scratch, void* stream,
                     uint32_t* d_flags = nullptr);

void count_launch(uint64_t n);

// Workspace block cache (api.cu): cudaMalloc'd blocks reused across calls; a block may be put back
// only after the stream that used it has been synchronised.
cudaError_t cache_get(void** out, size_t bytes);
void setup_pool();  // stream-ordered pool keeps its memory (release threshold = max)
void cache_put(void* p);

// NVRTC specialisation (jit.cpp)
bool jit_enabled();
int jit_hot_reg();
struct JitProbe {  // compile-only mode of the JIT (blu_gby_jit_probe)
  int programs = 0, failed = 0;
  std::string log;
};
void jit_probe_begin(JitProbe* pr);
void jit_probe_end();
bool jit_probe_active();
const void* jit_kernel(const std::string& spec_src, const std::string& entry_src, const char* entry);
// BLU_* knobs (env.cpp): env_snapshot() at every public entry point, benv() reads the snapshot
void env_snapshot();
const char* benv(const char* name);
std::string jit_spec(const char* name, const Layout& L, uint32_t S, const uint32_t* soff);

// Own LSD radix sort of u64 keys (sort.cu), used by the KMV estimate (kmv.cu)
size_t sort_u64_scratch_bytes(uint64_t n);
cudaError_t sort_u64_keys(const uint64_t* kin, uint64_t* kout, uint64_t n, void* ws, cudaStream_t st);

// Planner helpers (plan.cpp)
uint32_t smem_entry_bytes(const Layout& lay);
void build_slot_template(const Layout& lay, uint8_t* out);

}  // namespace blu
