// plan.cpp — the planner ("GPU moderator") and plan-level C ABI.
//
// Host only: blu_gby_plan never launches work. It turns (schema, est_groups, n_rows) — the
// metadata the DB2 runtime hands the GPU runtime — into a frozen plan:
//   * state fields and the slot layout (key + one field per payload/aggregate, padded so
//     the row is 1/2/4/8/16-byte aligned; Table 1 P:155-160 is the 32-byte example);
//   * the kernel path (number of rows, estimated groups, number of aggregates):
//       (a) dense shared-memory tables when the whole dictionary domain fits in shared memory
//           ("Second Kernel: Small Number of Groups", §4.3.2);
//       (b') direct-mapped global table when the dense domain is small enough to allocate
//           (the paper's "mod hash" with a table at least as large as the domain);
//       (b) global open-addressing hash table sized from est_groups ("First Kernel", §4.3.1,
//           P:149-162): cap = next_pow2(ceil(max(est,1)/0.7)), >= 1024 (reading A5);
//   * the shared-memory hot-key front for (b)/(b') when rows/groups is high (the moderator's
//     "ratio of rows to number of groups"; "if it gets full ... merge into a global
//     hash table");
//   * shared memory and launch shape.
#include <cuda_runtime.h>
#include <stdarg.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <mutex>

#include "blu_internal.h"

namespace blu {

thread_local std::string g_last_error;

blu_status_t fail(blu_status_t s, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  g_last_error = buf;
  return s;
}

static uint64_t next_pow2(uint64_t x) {
  uint64_t p = 1;
  while (p < x) p <<= 1;
  return p;
}

// Planner constants (SURVEY.md §5 "Config / flags"; reading A16: the paper gives no values).
constexpr uint32_t kSmemDenseMax = 96 * 1024;   // path (a): D x entry bytes, 2 CTAs/SM
constexpr double kMaxLoad = 0.7;                // A5
constexpr double kMaxLoadPart = 0.5;            // partitioned mode (buckets are L2-resident)
constexpr uint64_t kMinCap = 1024;
constexpr uint64_t kFrontRatio = 1000;          // rows/groups above which the front pays off
constexpr uint32_t kFrontBudget = 110 * 1024;
constexpr uint32_t kFrontBudgetWide = 220 * 1024;  // one CTA per SM
constexpr uint64_t kDirectMin = 1ull << 20;
constexpr uint64_t kRowLockRatio = 16;          // kernel 3 when rows/groups <= this
constexpr uint32_t kPartBudgetMB = 48;          // L2 slice per bucket (126 MB L2)
constexpr uint32_t kSmemMax = 232448;           // dynamic shared memory per CTA (227 KB opt-in)
constexpr uint32_t kMaxBuckets = 4096;          // one-pass scatter fan-out
constexpr uint32_t kMaxBuckets2 = 16384;        // two-level scatter (128 x 128)
constexpr bool kSmemDefault2 = true;             // bucket tables by default up to kMaxBuckets2 (C5)
constexpr double kBucketLoad = 0.7;             // mean groups per bucket / bucket table entries
constexpr uint32_t kMaxSlotBytes = 256;         // AoS slot limit (init template size)

static bool field_q(int kind) { return kind == FK_SUMQ || kind == FK_MINQ || kind == FK_MAXQ; }
static int32_t field_gsize(int kind) {
  return field_q(kind) ? 16 : (kind == FK_MINI32 || kind == FK_MAXI32) ? 4 : 8;
}
static int32_t field_ssize(int kind) {
  return field_q(kind) ? 16 : (kind == FK_COUNT || kind == FK_MINI32 || kind == FK_MAXI32) ? 4 : 8;
}
static int32_t field_group(int kind) {
  switch (kind) {
    case FK_COUNT: case FK_SUMI: case FK_SUMQ: return SG_ISUM;
    case FK_SUMF: return SG_FSUM;
    case FK_MINI32: case FK_MINI64: case FK_MINF64: case FK_MINQ: return SG_MIN;
    default: return SG_MAX;
  }
}

uint32_t smem_entry_bytes(const Layout& lay) {
  uint32_t b = 0;
  for (int j = 0; j < lay.n_fields; ++j) b += lay.f[j].ssize;
  return b;
}

// Assign AoS offsets (natural alignment, in field order after the 8-byte key) and dense groups.
static void finish_layout(Layout& L) {
  uint32_t off = 8 * (L.key_words == 2 ? 2 : 1);
  int32_t gcount[4] = {0, 0, 0, 0};
  for (int j = 0; j < L.n_fields; ++j) {
    Field& f = L.f[j];
    f.gsize = field_gsize(f.kind);
    f.ssize = field_ssize(f.kind);
    off = (off + f.gsize - 1) / f.gsize * f.gsize;
    f.goff = (int32_t)off;
    off += f.gsize;
    f.sgroup = field_group(f.kind);
    f.sidx = gcount[f.sgroup]++;
  }
  for (int g = 0; g < 4; ++g) L.n_group[g] = gcount[g];
  L.has_q = 0;
  for (int j = 0; j < L.n_fields; ++j) L.has_q |= field_q(L.f[j].kind) ? 1 : 0;
  for (int c = 0; c < L.n_vals; ++c) L.has_q |= L.val_dtype[c] == BLU_I128 ? 1 : 0;
  uint32_t raw = (off + 7) / 8 * 8;
  uint32_t sb = 16;
  while (sb < raw && sb < 128) sb <<= 1;
  if (sb < raw) sb = (raw + 63) / 64 * 64;
  L.slot_bytes = sb;
  L.smem_entry_bytes = smem_entry_bytes(L);
  if (L.lock_off) {  // kernel 3: a 4-byte row lock after the fields (re-padded slot)
    uint32_t lo = (off + 3) / 4 * 4;
    L.lock_off = (int32_t)lo;
    uint32_t raw2 = (lo + 4 + 7) / 8 * 8;
    uint32_t sb2 = 16;
    while (sb2 < raw2 && sb2 < 128) sb2 <<= 1;
    if (sb2 < raw2) sb2 = (raw2 + 63) / 64 * 64;
    L.slot_bytes = sb2;
  }
}

static int add_field(Layout& L, int kind, int col, int is_count) {
  for (int j = 0; j < L.n_fields; ++j)
    if (L.f[j].kind == kind && L.f[j].col == col) return j;
  Field f{};
  f.kind = kind;
  f.col = col;
  f.is_count = is_count;
  L.f[L.n_fields] = f;
  if (is_count) L.count_field = L.n_fields;
  return L.n_fields++;
}

static int device_sms() {
  static int sms = -1;
  static std::once_flag once;
  std::call_once(once, [] {
    int n = 0;
    if (cudaGetDeviceCount(&n) == cudaSuccess && n > 0) {
      int dev = 0, v = 0;
      cudaGetDevice(&dev);
      if (cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev) == cudaSuccess) sms = v;
    } else {
      cudaGetLastError();
    }
    if (sms <= 0) sms = 148;  // B200
  });
  return sms;
}

static const char* env(const char* k) {
  const char* v = benv(k);
  return (v && *v) ? v : nullptr;
}

void build_slot_template(const Layout& L, uint8_t* out) {
  memset(out, 0, L.slot_bytes);
  uint64_t key = kEmpty;
  memcpy(out, &key, 8);
  if (L.key_words == 2) memcpy(out + 8, &key, 8);
  for (int j = 0; j < L.n_fields; ++j) {
    const Field& f = L.f[j];
    uint8_t* p = out + f.goff;
    int64_t v64 = 0;
    int32_t v32 = 0;
    switch (f.kind) {
      case FK_MINI32: v32 = INT32_MAX; memcpy(p, &v32, 4); break;
      case FK_MAXI32: v32 = INT32_MIN; memcpy(p, &v32, 4); break;
      case FK_MINI64: case FK_MINF64: v64 = INT64_MAX; memcpy(p, &v64, 8); break;
      case FK_MAXI64: case FK_MAXF64: v64 = INT64_MIN; memcpy(p, &v64, 8); break;
      case FK_MINQ: {  // INT128_MAX: low word all ones, high word INT64_MAX
        const uint64_t w[2] = {~0ull, (uint64_t)INT64_MAX};
        memcpy(p, w, 16);
        break;
      }
      case FK_MAXQ: {  // INT128_MIN
        const uint64_t w[2] = {0ull, (uint64_t)INT64_MIN};
        memcpy(p, w, 16);
        break;
      }
      case FK_SUMQ: memset(p, 0, 16); break;
      default: memcpy(p, &v64, 8); break;  // COUNT, SUM: 0
    }
  }
}

uint32_t bucket_table_bytes(const Layout& L, uint32_t S) {
  uint32_t o = S * 8;
  for (int j = 0; j < L.n_fields; ++j) o += (S * (uint32_t)L.f[j].ssize + 15) / 16 * 16;
  return o;
}

uint32_t bucket_smem_bytes(const Layout& L, uint32_t S, uint32_t B, bool prefix) {
  // behind the table: the buckets' piece prefix (B + 1 u32; pieces mode only) and 2 scalars
  return bucket_table_bytes(L, S) + (((prefix ? B + 1 : 0) + 2) * 4 + 15) / 16 * 16;
}

void fill_smem_layout(AggParams& p, uint32_t S, bool with_keys) {
  const Layout& L = p.lay;
  uint32_t o = 0;
  p.S = S;
  p.key_off = 0;
  if (with_keys) o = S * 8;
  for (int j = 0; j < L.n_fields; ++j) {
    p.soff[j] = o;
    o += (S * (uint32_t)L.f[j].ssize + 15) / 16 * 16;
  }
  p.seg_stride = 0;
  p.seg_count = nullptr;
  p.n_segs = 0;
  p.gate = nullptr;
  p.gate_run_if = 0;
  for (int c = 0; c < kMaxFields; ++c) p.colmask[c] = 0;
  p.cntmask = 0;
  for (int j = 0; j < L.n_fields; ++j) {
    if (L.f[j].col < 0) p.cntmask |= 1u << j;
    else p.colmask[L.f[j].col] |= 1u << j;
  }
}

}  // namespace blu

using namespace blu;

extern "C" {

const char* blu_gby_status_str(blu_status_t s) {
  switch (s) {
    case BLU_OK: return "BLU_OK";
    case BLU_E_INVALID: return "BLU_E_INVALID";
    case BLU_E_UNSUPPORTED: return "BLU_E_UNSUPPORTED";
    case BLU_E_KEY_RANGE: return "BLU_E_KEY_RANGE";
    case BLU_E_OOM: return "BLU_E_OOM";
    case BLU_E_CUDA: return "BLU_E_CUDA";
  }
  return "BLU_E_UNKNOWN";
}

const char* blu_gby_last_error(void) { return g_last_error.c_str(); }

blu_status_t blu_gby_plan(const blu_gby_schema_t* s, uint64_t est_groups, uint64_t n_rows,
                          blu_gby_plan_t* out_plan) {
  env_snapshot();
  if (!s || !out_plan) return fail(BLU_E_INVALID, "NULL schema or out_plan");
  *out_plan = nullptr;
  if (s->n_keys < 1 || s->n_keys > kMaxKeys || !s->keys)
    return fail(BLU_E_INVALID, "n_keys must be 1..%d (got %d)", kMaxKeys, s->n_keys);
  if (s->n_vals < 0 || s->n_vals > kMaxVals || (s->n_vals > 0 && !s->vals))
    return fail(BLU_E_INVALID, "n_vals must be 0..%d (got %d)", kMaxVals, s->n_vals);
  if (s->n_aggs < 1 || s->n_aggs > kMaxAggs || !s->aggs)
    return fail(BLU_E_INVALID, "n_aggs must be 1..%d (got %d)", kMaxAggs, s->n_aggs);
  for (int k = 0; k < s->n_keys; ++k)
    if (s->keys[k].dtype != BLU_I32 && s->keys[k].dtype != BLU_I64)
      return fail(BLU_E_INVALID, "key %d: dtype must be BLU_I32 or BLU_I64", k);
  for (int c = 0; c < s->n_vals; ++c)
    if (s->vals[c] != BLU_I32 && s->vals[c] != BLU_I64 && s->vals[c] != BLU_F64 && s->vals[c] != BLU_I128)
      return fail(BLU_E_INVALID, "value %d: bad dtype %d", c, (int)s->vals[c]);
  for (int a = 0; a < s->n_aggs; ++a) {
    int op = s->aggs[a].op;
    if (op < BLU_COUNT || op > BLU_AVG) return fail(BLU_E_INVALID, "agg %d: bad op %d", a, op);
    if (op != BLU_COUNT && (s->aggs[a].val_col < 0 || s->aggs[a].val_col >= s->n_vals))
      return fail(BLU_E_INVALID, "agg %d: val_col %d out of range", a, s->aggs[a].val_col);
  }
  bool sparse = false;
  int n_sparse = 0;
  for (int k = 0; k < s->n_keys; ++k)
    if (s->keys[k].dict_size == 0) {
      sparse = true;
      ++n_sparse;
    }
  for (int k = 0; k < s->n_keys; ++k)
    if (s->keys[k].dtype == BLU_I32 && s->keys[k].dict_size > (1ull << 31))
      return fail(BLU_E_INVALID, "key %d: dict_size %llu exceeds the i32 code range", k,
                  (unsigned long long)s->keys[k].dict_size);
  // one 64-bit word: a single sparse key, or dense keys with D < 2^62; otherwise try two words
  bool wide = false;
  {
    uint64_t Dt = 1;
    bool over = false;
    for (int k = 0; k < s->n_keys && !sparse; ++k) {
      const uint64_t d = s->keys[k].dict_size;
      if (Dt > ((1ull << 62) - 1) / d) over = true;  // one word only while D < 2^62 (strict)
      else Dt *= d;
    }
    wide = (sparse && s->n_keys > 1) || over;
  }
  int kword[kMaxKeys] = {0};
  uint64_t kstride[kMaxKeys] = {0};
  if (wide) {  // greedy two-word packing: each sparse column takes a word; dense columns fill up
    if (n_sparse > 2) return fail(BLU_E_UNSUPPORTED, "more than two sparse key columns (> 128-bit keys)");
    uint64_t prod[2] = {1, 1};
    bool full[2] = {false, false};
    int w = 0;
    for (int k = 0; k < s->n_keys; ++k)
      if (s->keys[k].dict_size == 0) {
        kword[k] = w;
        kstride[k] = 1;
        full[w] = true;
        ++w;
      }
    for (int k = 0; k < s->n_keys; ++k) {
      const uint64_t d = s->keys[k].dict_size;
      if (!d) continue;
      int t = -1;
      for (int c = 0; c < 2 && t < 0; ++c)
        if (!full[c] && prod[c] <= ((1ull << 62) - 1) / d) t = c;  // per-word product < 2^62
      if (t < 0) return fail(BLU_E_UNSUPPORTED, "key tuple does not fit in 128 bits");
      kword[k] = t;
      kstride[k] = prod[t];
      prod[t] *= d;
    }
  }

  {
    bool q = false;
    for (int c = 0; c < s->n_vals; ++c) q = q || s->vals[c] == BLU_I128;
    if (q && wide) return fail(BLU_E_UNSUPPORTED, "128-bit payloads with a key tuple wider than 64 bits");
  }
  auto* P = new blu_gby_plan_s();
  P->keys.assign(s->keys, s->keys + s->n_keys);
  P->vals.assign(s->vals, s->vals + s->n_vals);
  P->aggs.assign(s->aggs, s->aggs + s->n_aggs);
  P->n_rows = n_rows;
  P->est_groups = std::max<uint64_t>(1, std::min<uint64_t>(est_groups, std::max<uint64_t>(n_rows, 1)));

  Layout& L = P->lay;
  memset(&L, 0, sizeof L);
  L.n_keys = s->n_keys;
  L.sparse = sparse ? 1 : 0;
  L.count_field = -1;
  uint64_t D = 1;
  L.key_words = wide ? 2 : 1;
  for (int k = 0; k < s->n_keys; ++k) {
    L.key_dtype[k] = s->keys[k].dtype;
    L.dict[k] = s->keys[k].dict_size;
    if (wide) {
      L.kword[k] = kword[k];
      L.stride[k] = kstride[k];
      continue;
    }
    L.stride[k] = D;
    if (!sparse) D *= s->keys[k].dict_size;
  }
  if (wide) sparse = true;  // no dense domain: hash path only
  L.domain = sparse ? 0 : D;
  L.n_vals = s->n_vals;
  for (int c = 0; c < s->n_vals; ++c) L.val_dtype[c] = s->vals[c];

  P->amap.resize(s->n_aggs);
  for (int a = 0; a < s->n_aggs; ++a) {
    int op = s->aggs[a].op, col = s->aggs[a].val_col;
    AggMap& m = P->amap[a];
    m.op = op;
    m.val_col = col;
    m.field2 = -1;
    int dt = op == BLU_COUNT ? BLU_I64 : s->vals[col];
    if (op == BLU_COUNT) {
      m.field = add_field(L, FK_COUNT, -1, 1);
      m.out_dtype = BLU_I64;
    } else if (op == BLU_SUM || op == BLU_AVG) {
      m.field = add_field(L, dt == BLU_F64 ? FK_SUMF : dt == BLU_I128 ? FK_SUMQ : FK_SUMI, col, 0);
      if (op == BLU_AVG) m.field2 = add_field(L, FK_COUNT, -1, 1);
      m.out_dtype = op == BLU_AVG ? BLU_F64 : (dt == BLU_F64 || dt == BLU_I128 ? dt : BLU_I64);
    } else if (op == BLU_MIN) {
      m.field = add_field(L, dt == BLU_I32 ? FK_MINI32 : dt == BLU_I64 ? FK_MINI64 : dt == BLU_I128 ? FK_MINQ : FK_MINF64,
                          col, 0);
      m.out_dtype = dt;
    } else {
      m.field = add_field(L, dt == BLU_I32 ? FK_MAXI32 : dt == BLU_I64 ? FK_MAXI64 : dt == BLU_I128 ? FK_MAXQ : FK_MAXF64,
                          col, 0);
      m.out_dtype = dt;
    }
  }
  finish_layout(L);

  // ---- moderator: pick the path ---------------------------------------------
  uint64_t cap_est = std::max<uint64_t>(kMinCap, next_pow2((uint64_t)((double)P->est_groups / kMaxLoad + 0.999999)));
  uint32_t entry_with_count = L.smem_entry_bytes + (L.count_field < 0 ? 4u : 0u);
  L.sparse = sparse ? 1 : 0;
  int path;
  // division form: D * entry bytes can wrap u64 for D near 2^62
  if (!sparse && D <= kSmemDenseMax / entry_with_count) path = BLU_PATH_DENSE_SMEM;
  else if (!sparse && D <= std::max<uint64_t>(2 * cap_est, kDirectMin)) path = BLU_PATH_DIRECT_GLOBAL;
  else path = BLU_PATH_HASH_GLOBAL;
  if (const char* fp = env("BLU_GBY_FORCE_PATH")) {
    int want = fp[0] == 'a' ? BLU_PATH_DENSE_SMEM : fp[0] == 'd' ? BLU_PATH_DIRECT_GLOBAL : BLU_PATH_HASH_GLOBAL;
    if (want == BLU_PATH_DENSE_SMEM && (sparse || D > (200u * 1024u) / entry_with_count)) {
      delete P;
      return fail(BLU_E_UNSUPPORTED, "BLU_GBY_FORCE_PATH=a: dense domain does not fit in shared memory");
    }
    if (want == BLU_PATH_DIRECT_GLOBAL && sparse) {
      delete P;
      return fail(BLU_E_UNSUPPORTED, "BLU_GBY_FORCE_PATH=d: needs dictionary-encoded keys");
    }
    path = want;
  }
  if (L.key_words == 2) path = BLU_PATH_HASH_GLOBAL;  // wide keys: 16-byte key CAS, hash path only
  if (L.slot_bytes > kMaxSlotBytes) {  // the init template (kernels.cu SlotTemplate) holds 256 bytes
    delete P;
    return fail(BLU_E_UNSUPPORTED, "slot of %u bytes (key + state fields) exceeds %u bytes", L.slot_bytes, kMaxSlotBytes);
  }
  if (L.has_q) path = BLU_PATH_HASH_GLOBAL;            // 128-bit payloads: 16-byte global fields only
  P->path = path;
  if (path != BLU_PATH_HASH_GLOBAL && L.count_field < 0) {  // dense occupancy = COUNT > 0
    add_field(L, FK_COUNT, -1, 1);
    finish_layout(L);
  }
  P->cap = path == BLU_PATH_HASH_GLOBAL ? cap_est : D;

  // Kernel 3: "if both 1) the number of aggregation functions is large [more than 5] 2) number
  // of rows/number groups is small, this kernel would have very good performance" — lock the slot
  // once and apply every aggregate, instead of one atomic per aggregate. Hash path only (AoS slots).
  // On B200 every aggregate of this library has a native fire-and-forget 64-bit L2 reduction, and the
  // lock costs two round trips per row: measured slower even in the paper's regime (K3: 14.3 vs 11.0
  // ms; C4 hot keys: 53 vs 3 ms per 1e8 rows), so the rule is kept but off unless requested
  // (BLU_GBY_ROW_LOCK=1, or =rule to apply the paper's rule).
  {
    const bool rule = path == BLU_PATH_HASH_GLOBAL && L.n_fields > 5 && n_rows <= kRowLockRatio * P->est_groups;
    bool lock = false;
    if (const char* rl = env("BLU_GBY_ROW_LOCK"))
      lock = path == BLU_PATH_HASH_GLOBAL && !L.has_q && (rl[0] == '1' || (rl[0] == 'r' && rule));
    if (lock) {
      L.lock_off = 1;  // placeholder: finish_layout assigns the real offset
      finish_layout(L);
      if (L.slot_bytes > kMaxSlotBytes) {
        delete P;
        return fail(BLU_E_UNSUPPORTED, "slot with row lock exceeds %u bytes", kMaxSlotBytes);
      }
    }
  }

  // Partitioned two-pass mode for path (b) when the table exceeds an L2-sized budget: rows are
  // first scattered into B buckets by the top bits of their slot, then aggregated bucket by bucket.
  // Pass 2 either applies every row to the bucket's L2-resident slice of the global table (default;
  // 126 MB L2) or builds each bucket's groups in a shared-memory table per CTA
  // and merges them into the global table once per piece (part_smem, BLU_GBY_PART_SMEM=1).
  P->parts = 1;
  P->part_shift = 0;
  P->part_smem = 0;
  P->bucket_S = 0;
  P->bucket_smem = 0;
  P->bucket_whole = 0;
  if (path == BLU_PATH_HASH_GLOBAL && L.key_words == 1 && !L.has_q) {
    uint64_t budget = (uint64_t)kPartBudgetMB << 20;
    if (const char* pm = env("BLU_GBY_PART_MB")) budget = (uint64_t)atoi(pm) << 20;
    uint64_t tbytes = P->cap * (uint64_t)L.slot_bytes;
    // Shared-memory bucket tables: C3 (10^9 rows, 10^7 groups) needs 2048 buckets. Scattered in one
    // pass that costs 31 ms against 9.4 ms for the 32-bucket L2 mode; in two passes (32 x 64, api.cu)
    // 19.4 ms, and pass 2 drops from 25.4 to 12.5 ms: 32.5 vs 35.7 ms. So the mode is
    // the default when the estimated groups fit >= 256 buckets of at most kMaxBuckets (two-level
    // scatter); C5's 5*10^7 groups do not fit and keep the L2 mode. BLU_GBY_PART_SMEM=0/1 overrides.
    // BLU_GBY_BUCKET_S (experiment): cap the entries per bucket table below what shared memory holds
    const uint32_t s_cap = env("BLU_GBY_BUCKET_S") ? (uint32_t)std::max(64, atoi(env("BLU_GBY_BUCKET_S"))) : 1u << 30;
    // work items = whole buckets (default: a bucket is at most its capacity, ~1.1-1.2x the mean, so
    // one item per bucket balances, and the table gets the shared memory a piece prefix would take:
    // 64 KB at 16384 buckets), or pieces of ~1/div of the mean bucket with BLU_GBY_PIECE_DIV=div
    const bool whole = !env("BLU_GBY_PIECE_DIV");
    auto S_of = [&](uint32_t b) {
      uint32_t S = 16;
      while (bucket_smem_bytes(L, S + 16, b, !whole) <= kSmemMax && S + 16 <= s_cap) S += 16;
      return S;
    };
    // smallest B whose buckets hold <= kBucketLoad * S groups on average, within the scatter's
    // shared memory and <= kMaxBuckets; the records' layout has the same fields as L
    // two_level: the fan-outs are two_level_b1(b) and b / two_level_b1(b) (api.cu), so b may exceed the
    // one-pass limit; widest = the larger histogram of the two levels
    auto widest = [&](bool two_level, uint64_t b) {
      return (uint32_t)(two_level && b >= 256 ? std::max<uint64_t>(two_level_b1(b), b / two_level_b1(b)) : b);
    };
    auto smem_B = [&](bool two_level, bool cap_default = false) {
      const uint64_t max_b = two_level && !cap_default ? kMaxBuckets2 : kMaxBuckets;
      uint64_t b = 2;
      while (b < max_b && (double)P->est_groups > kBucketLoad * S_of((uint32_t)b) * (double)b &&
             scatter_smem(L.n_vals, widest(two_level, 2 * b)) <= kSmemMax && b * 2 <= P->cap / 1024)
        b <<= 1;
      return b;
    };
    const char* tl = env("BLU_GBY_PART_2LEVEL");
    const bool two_ok = !(tl && tl[0] == '0');
    bool smem_mode = false;
    if (const char* ps = env("BLU_GBY_PART_SMEM")) {
      smem_mode = !L.lock_off && ps[0] == '1';
    } else if (!L.lock_off && budget && tbytes > budget && !env("BLU_GBY_PARTS") && two_ok) {
      // up to kMaxBuckets2: C5 (5*10^7 groups) in 16384 tables behind a 128 x 128 scatter (second
      // level over two streams) 57.1 vs 61.4 ms per 1.6*10^9 rows in the L2-slice mode (a 32 x 512
      // scatter made it 74.3 ms)
      const uint64_t b = smem_B(true, !kSmemDefault2);
      smem_mode = b >= 256 && (double)P->est_groups <= kBucketLoad * S_of((uint32_t)b) * (double)b;
    }
    uint64_t B = 1;
    const char* forced = env("BLU_GBY_PARTS");
    if (smem_mode && ((budget && tbytes > budget) || (forced && atoi(forced) > 1))) {
      B = smem_B(two_ok, !env("BLU_GBY_PART_SMEM") && !kSmemDefault2);
      if (forced) B = std::max(2, std::min((int)(two_ok ? kMaxBuckets2 : kMaxBuckets), atoi(forced)));
      while (B > 2 && scatter_smem(L.n_vals, widest(two_ok, B)) > kSmemMax) B >>= 1;  // histogram bins per tile
      P->part_smem = 1;
      P->bucket_S = S_of((uint32_t)B);
      P->bucket_whole = whole ? 1 : 0;
      P->bucket_smem = bucket_smem_bytes(L, P->bucket_S, (uint32_t)B, !whole);
    } else {
      while (budget && B < 1024 && tbytes / B > budget && B < P->cap / 1024) B <<= 1;
      // a forced count is clamped to what the L2-slice pass 2 indexes (kMaxSegs: 2048 forced buckets
      // overran its shared prefix array)
      if (const char* pp = env("BLU_GBY_PARTS")) B = std::max(1, std::min((int)kMaxSegs, atoi(pp)));
      if (B > 1 && !env("BLU_GBY_PARTS")) {
        // partitioned tables live in L2 one bucket at a time: trade HBM footprint for short probes
        uint64_t cap2 = std::max<uint64_t>(kMinCap, next_pow2((uint64_t)((double)P->est_groups / kMaxLoadPart + 0.999999)));
        if (cap2 > P->cap) {
          P->cap = cap2;
          tbytes = P->cap * (uint64_t)L.slot_bytes;
          while (budget && B < 1024 && tbytes / B > budget && B < P->cap / 1024) B <<= 1;
        }
      }
    }
    P->parts = (uint32_t)B;
    uint32_t lc = 0, lb = 0;
    while ((1ull << lc) < P->cap) ++lc;
    while ((1u << lb) < P->parts) ++lb;
    P->part_shift = lc - lb;
  }

  // hot-key front (path b / b')
  P->hot_front = 0;
  P->front_slots = 0;
  if (path != BLU_PATH_DENSE_SMEM && L.key_words == 1 && !L.has_q) {
    bool on = n_rows >= kFrontRatio * P->est_groups;
    if (const char* hf = env("BLU_GBY_HOT_FRONT")) on = hf[0] == '1';
    if (on) {
      uint32_t per = 8 + L.smem_entry_bytes;
      uint32_t budget = kFrontBudget;
      uint32_t S = 8192;
      if (const char* fs = env("BLU_GBY_FRONT_SLOTS")) S = (uint32_t)atoi(fs);
      uint32_t S1 = S, S2 = S;
      while (S1 > 64 && S1 * per > budget) S1 >>= 1;  // power of two, >= 64
      while (S2 > 64 && S2 * per > kFrontBudgetWide) S2 >>= 1;
      // a front twice as large in one 1024-thread CTA per SM holds twice the heavy hitters (the
      // seeded front keeps S/2 keys); same threads and registers per SM as 2 x 512
      bool wide = S2 > S1;
      if (const char* fw = env("BLU_GBY_FRONT_WIDE")) wide = wide && fw[0] == '1';
      S = wide ? S2 : S1;
      if (S * per <= 200 * 1024 || wide) {
        P->hot_front = 1;
        P->front_slots = S;
        P->front_wide = wide ? 1 : 0;
      }
    }
  }

  // shared memory and launch shape
  P->sms = device_sms();
  if (path == BLU_PATH_DENSE_SMEM) {
    uint32_t b = 0;
    for (int j = 0; j < L.n_fields; ++j) b += (uint32_t)((D * L.f[j].ssize + 15) / 16 * 16);
    P->smem_bytes = b;
    P->block = 512;
  } else if (P->hot_front) {
    uint32_t b = P->front_slots * 8;
    for (int j = 0; j < L.n_fields; ++j) b += (P->front_slots * L.f[j].ssize + 15) / 16 * 16;
    P->smem_bytes = b;
    // one CTA per SM: 768 threads x 80 registers carry 4 pipelined rows per thread (C4 9.2 ms)
    // where 1024 x 64 carry 2 (10.2 ms); 640 and 512 (x 128) measured the same as 768
    // with the hot keys in registers (BLU_GBY_HOT_REG, +12 registers per key): 640 x 96 (C4 8.87 ms
    // vs 9.10 without; at 768 x 80 those registers spill: 11.2 ms)
    P->block = P->front_wide ? (jit_hot_reg() ? 640 : 768) : 512;
  } else {
    P->smem_bytes = 0;
    P->block = 256;
  }
  if (const char* bs = env("BLU_GBY_BLOCK")) P->block = (uint32_t)atoi(bs);
  uint32_t per_sm_threads = 2048;
  uint32_t by_threads = per_sm_threads / P->block;
  uint32_t by_smem = P->smem_bytes ? std::max<uint32_t>(1, (227 * 1024) / (P->smem_bytes + 1024)) : 32;
  uint32_t ctas = std::max<uint32_t>(1, std::min(by_threads, by_smem));
  // path (a): one resident wave (512 threads x <= 64 registers -> 2 CTAs/SM); a second wave would
  // pay the shared-table init and CTA->global flush again (measured: 0.75 vs 0.76-1.0 ms on C2)
  if (path == BLU_PATH_DENSE_SMEM) ctas = std::min<uint32_t>(ctas, 2);
  if (const char* cs = env("BLU_GBY_CTAS_PER_SM")) ctas = (uint32_t)atoi(cs);
  P->grid = (uint32_t)P->sms * ctas;

  // merge layout: rows are (keys, one column per state field); COUNT becomes SUM of counts.
  Layout& M = P->merge_lay;
  M = L;
  M.lock_off = 0;
  M.n_vals = L.n_fields;
  for (int j = 0; j < L.n_fields; ++j) {
    int k = L.f[j].kind;
    M.val_dtype[j] = (k == FK_MINI32 || k == FK_MAXI32) ? BLU_I32
                     : (k == FK_SUMF || k == FK_MINF64 || k == FK_MAXF64) ? BLU_F64
                     : field_q(k) ? BLU_I128 : BLU_I64;
    M.f[j].col = j;
    if (k == FK_COUNT) M.f[j].kind = FK_SUMI;  // is_count stays 1
  }
  finish_layout(M);

  *out_plan = P;
  return BLU_OK;
}

blu_status_t blu_gby_plan_info(blu_gby_plan_t P, int32_t* path, uint64_t* capacity, uint32_t* smem_bytes,
                               uint32_t* retries_last) {
  if (!P) return fail(BLU_E_INVALID, "NULL plan");
  if (path) *path = P->path;
  if (capacity) *capacity = P->cap;
  if (smem_bytes) *smem_bytes = P->smem_bytes;
  if (retries_last) *retries_last = P->retries_last.load();
  return BLU_OK;
}

blu_status_t blu_gby_plan_describe(blu_gby_plan_t P, blu_gby_plan_desc_t* o) {
  if (!P || !o) return fail(BLU_E_INVALID, "NULL plan or out");
  memset(o, 0, sizeof *o);
  o->path = P->path;
  o->capacity = P->cap;
  o->est_groups = P->est_groups;
  o->slot_bytes = P->lay.slot_bytes;
  o->smem_bytes = P->smem_bytes;
  o->hot_front = P->hot_front;
  o->front_slots = P->front_slots;
  o->partitions = P->parts;
  o->n_states = P->lay.n_fields;
  for (int j = 0; j < P->lay.n_fields && j < 32; ++j) o->state_dtypes[j] = P->merge_lay.val_dtype[j];
  o->grid = P->grid;
  o->block = P->block;
  o->retries_last = P->retries_last.load();
  o->row_lock = P->lay.lock_off ? 1 : 0;
  o->part_smem = P->part_smem;
  o->bucket_entries = P->bucket_S;
  return BLU_OK;
}

blu_status_t blu_gby_dense_state_shape(blu_gby_plan_t P, int32_t* n_isum, int32_t* n_fsum, int32_t* n_min,
                                       int32_t* n_max, uint64_t* domain) {
  if (!P) return fail(BLU_E_INVALID, "NULL plan");
  if (P->path == BLU_PATH_HASH_GLOBAL) return fail(BLU_E_UNSUPPORTED, "dense state needs path a or b'");
  if (n_isum) *n_isum = P->lay.n_group[SG_ISUM];
  if (n_fsum) *n_fsum = P->lay.n_group[SG_FSUM];
  if (n_min) *n_min = P->lay.n_group[SG_MIN];
  if (n_max) *n_max = P->lay.n_group[SG_MAX];
  if (domain) *domain = P->lay.domain;
  return BLU_OK;
}

uint32_t blu_gby_record_bytes(blu_gby_plan_t P) {
  return P ? 8u * ((P->lay.key_words == 2 ? 2u : 1u) + (uint32_t)P->lay.n_fields) : 0u;
}

uint32_t blu_gby_row_record_bytes(blu_gby_plan_t P) {
  return P ? 8u * ((P->lay.key_words == 2 ? 2u : 1u) + (uint32_t)P->lay.n_vals) : 0u;
}

blu_status_t blu_gby_slot_template(blu_gby_plan_t P, void* out, uint32_t cap, uint32_t* slot_bytes) {
  if (!P) return fail(BLU_E_INVALID, "NULL plan");
  if (slot_bytes) *slot_bytes = P->lay.slot_bytes;
  if (out) {
    if (cap < P->lay.slot_bytes) return fail(BLU_E_INVALID, "template buffer too small (%u < %u)", cap, P->lay.slot_bytes);
    build_slot_template(P->lay, (uint8_t*)out);
  }
  return BLU_OK;
}

void blu_gby_plan_destroy(blu_gby_plan_t P) { delete P; }

}  // extern "C"
