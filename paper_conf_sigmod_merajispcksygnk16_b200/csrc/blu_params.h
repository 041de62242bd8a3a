// blu_params.h — the plain data structures shared by libblugby's host code and its device code.
// Compiles under nvcc, g++ and NVRTC (the JIT-specialised kernels include it verbatim), so it uses
// no standard headers: the integer typedefs come from <stdint.h> on the host and from the JIT
// preamble under NVRTC.
#pragma once

#ifndef __CUDACC_RTC__
#include <stdint.h>
#endif

// dtype / op numbering of include/blu_gby.h (repeated so this header stands alone under NVRTC)
#ifndef BLU_GBY_H
enum { BLU_I32 = 0, BLU_I64 = 1, BLU_F64 = 2, BLU_I128 = 3 };
#endif

namespace blu {

constexpr int kMaxKeys = 8;
constexpr int kMaxVals = 16;
constexpr int kMaxAggs = 16;
constexpr int kMaxFields = 24;
// partitioned pass 2 in the L2-slice mode (global_body SEG): at most this many buckets (per-CTA
// shared prefix of the buckets' warp tiles)
constexpr uint32_t kMaxSegs = 1024;
constexpr uint64_t kEmpty = ~0ull;  // key portion of the mask: M/4 Fs (Table 1)

// State-field kinds. Each aggregate maps to one or two fields (AVG = SUM field + COUNT field);
// fields are deduplicated per (kind, column) so SUM(v) and AVG(v) share one SUM field.
enum FieldKind : int32_t {
  FK_COUNT = 0,   // += 1 per row (COUNT(*)), 64-bit
  FK_SUMI = 1,    // int64 sum with two's-complement wrap (i32/i64 inputs widened)
  FK_SUMF = 2,    // f64 sum
  FK_MINI32 = 3,  // MIN over i32 (32-bit field in the slot, init INT32_MAX as in Table 1)
  FK_MAXI32 = 4,  // MAX over i32 (init INT32_MIN)
  FK_MINI64 = 5,  // MIN over i64 (init INT64_MAX)
  FK_MAXI64 = 6,  // MAX over i64 (init INT64_MIN, Table 1)
  FK_MINF64 = 7,  // MIN over f64 through the order-preserving int64 map (init +INT64_MAX)
  FK_MAXF64 = 8,  // MAX over f64 (init INT64_MIN)
  // 128-bit integer payloads ("128bit Integer or Decimal"): 16-byte fields, low word first
  FK_SUMQ = 9,    // sum mod 2^128: atomic add of the low word, carry into a RED on the high word
  FK_MINQ = 10,   // MIN over i128 (init INT128_MAX): 16-byte CAS loop
  FK_MAXQ = 11,   // MAX over i128 (init INT128_MIN)
};

// Where the dense state of a field lives in the 4 allreduce groups (blu_gby.h execute_dense_state).
enum StateGroup : int32_t { SG_ISUM = 0, SG_FSUM = 1, SG_MIN = 2, SG_MAX = 3 };

struct Field {
  int32_t kind;    // FieldKind
  int32_t col;     // value column (-1: COUNT from the constant 1)
  int32_t gsize;   // bytes in the global AoS slot (4 or 8)
  int32_t goff;    // byte offset in the global AoS slot
  int32_t sgroup;  // StateGroup for dense global state
  int32_t sidx;    // index within its group
  int32_t ssize;   // bytes per entry in a shared-memory table (4 or 8)
  int32_t is_count;
};

// Everything a kernel needs to know about the row format and the fields.
struct Layout {
  int32_t n_keys;
  int32_t key_dtype[kMaxKeys];
  uint64_t dict[kMaxKeys];
  uint64_t stride[kMaxKeys];  // mixed radix: stride_0 = 1, stride_j = prod_{i<j} dict_i
  int32_t sparse;             // 1: single sparse key column (code itself is the packed key)
  uint64_t domain;            // D = prod dict (dense keys only)

  int32_t n_vals;                // value columns the kernel reads (schema columns or states)
  int32_t val_dtype[kMaxVals];
  int32_t n_fields;
  Field f[kMaxFields];
  int32_t count_field;           // index of the COUNT field or -1
  uint32_t slot_bytes;           // global AoS slot (key + fields, padded)
  int32_t n_group[4];            // fields per StateGroup
  uint32_t smem_entry_bytes;     // per entry of a shared-memory table (no key)
  int32_t lock_off;              // kernel 3: byte offset of the slot's row lock, 0 = none
  // wide keys (> 64 bits; NEXT-2): key_words = 2 packs the key columns into two 64-bit words
  // (mixed radix within a word; a sparse code occupies a whole word); kword[k] = word of column k and
  // stride[k] its stride within that word. The slot key is then 16 bytes, claimed with a 16-byte CAS.
  int32_t key_words;
  int32_t kword[kMaxKeys];
  int32_t has_q;  // 1: some value column is i128 / some field is 128-bit (generic k_agg_q kernel)
  // partition records (pass 2 / second scatter level): a sparse key equal to the empty mark is a
  // padding record written to keep bulk-copied runs 16-byte aligned; it is skipped, not an error
  int32_t pad_keys;
};

// ---------------------------------------------------------------------------------------------
// Kernel parameter blocks (passed by value; < 4 KB)
// ---------------------------------------------------------------------------------------------
// ---------------------------------------------------------------------------------------------
// Kernel parameter blocks (passed by value; < 4 KB)
// ---------------------------------------------------------------------------------------------
struct AggParams {
  Layout lay;
  const void* key[kMaxKeys];
  const void* val[kMaxVals];
  uint64_t n_rows;
  int32_t vec_ok;        // bit 0: all column pointers 16-byte aligned; bit 1: 32-byte aligned
  // targets
  void* table;           // path b: AoS slots (cap x slot_bytes)
  uint64_t cap_mask;     // cap - 1 (power of two)
  uint32_t max_probe;
  void* dense[4];        // paths a / b': dense state groups (SG_*), each n_group[g] x D int64
  uint32_t front_slots;  // shared-memory front entries (power of two) or 0
  uint32_t* flags;       // bit 0: overflow (probe bound), bit 1: key out of range
  // shared-memory table layout (path a: S = D; front: S = front_slots), filled by the host
  uint32_t S;
  uint32_t key_off;              // front keys (S x u64)
  uint32_t soff[kMaxFields];     // per field: byte offset of its SoA array
  uint32_t colmask[kMaxFields];  // per kernel value column: bit j = field j reads it
  uint32_t cntmask;              // fields that count the constant 1
  // partitioned pass 2 (segments mode, seg_stride > 0): rows of segment b are
  // [b * seg_stride, b * seg_stride + seg_count[b])
  uint64_t seg_stride;
  const uint64_t* seg_count;
  uint32_t n_segs;
  uint64_t* tile_ctr;            // segments mode: dynamic warp-tile counter (zeroed per launch)
  // device-side gate: the kernel runs only if ((*gate != 0) == gate_run_if); NULL = always
  const uint32_t* gate;
  uint32_t gate_run_if;
  uint32_t jit_ok;               // host: 1 = the launcher may use the NVRTC-specialised kernel
  // path (a) fusion: CTA 0 initialises the dense state (fuse_init) and the last CTA to finish
  // compacts it into the result (FinalParams::enabled); sync[0] = init done, sync[1] = CTAs done
  uint32_t fuse_init;
  uint32_t* sync;
  // seeded hot-key front (heavy hitters from a sample, [20] via P:38): S keys laid out as the
  // front's open-addressing image; CTAs copy it and only look keys up (no inserts). NULL = the
  // front is filled first-come with CAS inserts.
  const uint64_t* front_seed;
  // rank front (path b' only, dense domain D <= 32 * S): the seed is a rank image instead of a key
  // table. Word w (< front_rank_words = ceil(D / 32)) holds in its low half the bitmap of the hot
  // keys 32w..32w+31 and in its high half the number of hot keys below 32w, so a key's front entry is
  // that prefix + popc(bits below it): one shared-memory load per row, no probing. 0 = hash front.
  uint32_t front_rank_words;
  // rank front: the sample's most frequent key (device word written by the seed kernels; ~0 = none).
  // With SP::HOTREG each thread sums that key's rows in registers and flushes them once at the end,
  // so the hottest key (13% of C4's Zipf(1.1) rows) costs no shared-memory atomics. NULL = off.
  const uint64_t* hot_key;
  uint32_t prefetch;             // scatter: L2-prefetch the column bytes of the tile this many tiles ahead (0 = off)
  // partitioned pass 2 with bucket-local shared-memory tables (bucket_body): a bucket's rows are
  // cut into pieces of piece_rows rows (a multiple of the CTA tile); aux_off = byte offset of the
  // per-bucket piece prefix (n_segs + 1 u32) behind the S-entry table in dynamic shared memory.
  uint64_t piece_rows;
  uint32_t aux_off;
  // partitioned pass 2 in the L2-slice mode: warp tiles claimed per atomic on tile_ctr (0 = 16)
  uint32_t grab;
};

// Path (a) in-kernel compaction (S8 fused into S5a/S7 for small dense domains).
struct FinalParams {
  int32_t enabled;
  int32_t n_out;
  int32_t out_kind[kMaxFields];   // 0 field as stored, 1 AVG
  int32_t out_field[kMaxFields];
  int32_t out_field2[kMaxFields];
  int32_t out_dtype[kMaxFields];
  void* out_keys[kMaxKeys];
  void* out_vals[kMaxFields];
  uint64_t* n_groups;
};

// Pass 1 of the partitioned path (b): scatter rows into B buckets by the top bits of their slot.
struct ScatterParams {
  uint32_t B;
  uint32_t shift;            // bucket = (fmix64(key) & cap_mask) >> shift
  uint64_t seg_stride;       // bucket b starts at row b * seg_stride of the partition buffers
  uint64_t* cursor;          // B: rows appended so far (zeroed per chunk)
  uint64_t seg_cap;          // rows per bucket
  uint64_t* out_key;         // packed keys (u64)
  void* out_val[kMaxVals];   // value columns, input dtypes
  uint32_t* gate;            // set to 1 if any bucket overflows (pass 2 then falls back)
  // segmented input (the second level of a two-level scatter, one launch over every first-level
  // bucket): first-level bucket s holds rows [s * in_seg, s * in_seg + in_count[s]) of the input
  // (in_seg a multiple of the tile); its rows go to buckets s * in_B2 + ((h & cap_mask) >> shift).
  // in_seg = 0: plain input rows [0, n).
  uint64_t in_seg;
  const uint64_t* in_count;
  uint32_t in_B2;
  // 1: bucket runs leave shared memory by TMA bulk copies (cp.async.bulk), padded to an even number of
  // rows with empty-key records (all value columns 8 bytes; JIT kernels)
  uint32_t tma;
};

enum : uint32_t { FLAG_OVERFLOW = 1u, FLAG_KEY_RANGE = 2u };

struct CompactParams {
  Layout lay;
  int32_t source;        // 0: AoS hash table, 1: dense state (occupancy = COUNT > 0)
  const void* table;
  const void* dense[4];
  uint64_t n_entries;    // cap or D
  int32_t partial;       // 1: emit state fields, 0: finalized aggregates
  int32_t n_out;         // output value columns
  // finalized: per output column (aggregate) which field(s) and dtype
  int32_t out_kind[kMaxFields];   // 0 field as stored, 1 AVG
  int32_t out_field[kMaxFields];
  int32_t out_field2[kMaxFields];
  int32_t out_dtype[kMaxFields];
  void* out_keys[kMaxKeys];
  void* out_vals[kMaxFields];
  uint64_t* block_counts;
  uint64_t* block_offsets;
  uint64_t* n_groups;    // device
};

// Records-mode input for merges of exchanged partials: rows of `words` u64 (key, states).
struct RecSrc {
  const uint64_t* rec;
  uint32_t words;
};

}  // namespace blu
