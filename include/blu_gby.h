/*
 * blu_gby.h — libblugby: B200-native hash GROUP BY with SUM / COUNT / MIN / MAX / AVG.
 *
 * The method: Meraji et al., "Towards a Hybrid Design for Fast Query Processing in DB2 with BLU
 * Acceleration Using Graphical Processing Units", SIGMOD'16 — `P:n` below is line n of the paper
 * text. The GPU runtime receives the query's metadata — "the exact number of tuples,
 * the estimated number of groups, and the number of aggregation functions" — picks
 * a group-by kernel with its "GPU moderator", sizes the hash table from the
 * estimate and runs hash-based GROUP BY with the aggregate applied "right
 * after the insertion/finding of grouping key".
 *
 * Entry points:
 *   blu_gby_plan        S3  plan-time kernel selection from (schema, est_groups, n_rows)
 *   blu_gby_execute     S0-S8 on device columns -> finalized (group_keys, aggregates, n_groups)
 *   blu_gby_execute_host      same on HOST columns: chunked pinned H2D overlapped with S5
 *   blu_gby_execute_partial   same, but emits mergeable per-group states
 *   blu_gby_merge[_partial]   S9  re-aggregate partial results ("merged together in the
 *                                 final step"; P:107 two-phase local -> global)
 *   blu_gby_execute_dense_state / blu_gby_finalize_dense_state   path (a) multi-GPU helpers
 *   blu_gby_partition / blu_gby_merge_records                    path (b) multi-GPU helpers
 *   blu_gby_init_table / blu_gby_slot_template                   S4 (Table 1)
 *
 * Conventions (all calls):
 *   - Nothing throws across the ABI; every call returns blu_status_t. blu_gby_last_error()
 *     returns a thread-local detail string for the last failing call on this thread.
 *   - Pointers named *dev* or documented "device" are CUDA device pointers on the current
 *     device; "host" pointers are ordinary host memory (pinned memory is faster).
 *   - Input columns are BORROWED: they must stay valid and unchanged until the call returns
 *     (execute* synchronize `stream` before returning).
 *   - Results are LIBRARY-OWNED (device memory from cudaMallocAsync on `stream`, or pinned host
 *     memory for blu_gby_execute_host, taken from a per-process cache of pinned blocks that
 *     blu_gby_result_free returns them to); release them with blu_gby_result_free.
 *   - stream is a cudaStream_t passed as void* (0 = legacy default stream).
 *   - Plans are immutable and may be shared by threads; concurrent executes on different streams
 *     are safe.
 */
#ifndef BLU_GBY_H
#define BLU_GBY_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    BLU_OK = 0,
    BLU_E_INVALID = 1,      /* bad argument or schema                                          */
    BLU_E_UNSUPPORTED = 2,  /* valid SQL, not supported: key tuple wider than 128 bits, > 2 sparse */
    BLU_E_KEY_RANGE = 3,    /* a key code outside [0, dict_size) or a negative sparse code      */
    BLU_E_OOM = 4,          /* device or host allocation failed                                */
    BLU_E_CUDA = 5          /* other CUDA runtime error                                         */
} blu_status_t;

/* Column dtypes. BLU_I128 (value columns only): a 128-bit two's-complement integer stored as 16
 * bytes per row, low 64-bit word first — the paper's "128bit Integer or Decimal data type" whose
 * aggregates it applies with atomicCAS (a DECIMAL(31) column is its scaled 128-bit integer).
 * SUM(i128) wraps mod 2^128 and, like MIN/MAX(i128), returns an i128 column; AVG(i128) returns
 * f64 = (double)SUM / (double)COUNT, both conversions round-to-nearest-even. Plans with an i128
 * column use path (b) in one pass (no hot front, no partitioning, no per-plan JIT); the multi-GPU
 * record helpers (blu_gby_partition, blu_gby_merge_records) return BLU_E_UNSUPPORTED for them. */
typedef enum { BLU_I32 = 0, BLU_I64 = 1, BLU_F64 = 2, BLU_I128 = 3 } blu_dtype_t;

typedef enum { BLU_COUNT = 0, BLU_SUM = 1, BLU_MIN = 2, BLU_MAX = 3, BLU_AVG = 4 } blu_aggop_t;

/* One grouping column: dictionary codes in [0, dict_size) (P:109 LCOG loads "grouping keys";
 * DB2 BLU columns are dictionary encoded). dict_size == 0 means a sparse non-negative code.
 * Keys must be I32 or I64. The key tuple is packed into one 64-bit word when it is a single sparse
 * column or dense columns with prod(dict_size) < 2^62; otherwise into TWO words ("wide keys",
 * P:153 "If the key size is larger than 64 bit ..."): each sparse column (at most two) takes a
 * whole word, dense columns fill the words greedily in column order with a per-word product < 2^62.
 * Wide keys always plan path (b) with a 16-byte key CAS (no hot front, no partitioning). */
typedef struct {
    blu_dtype_t dtype;
    uint64_t dict_size;
} blu_key_desc_t;

/* One aggregate: op over value column val_col ("N different payloads and corresponding N
 * aggregation functions"). COUNT is COUNT(*) and ignores val_col (use -1). */
typedef struct {
    blu_aggop_t op;
    int32_t val_col;
} blu_agg_desc_t;

typedef struct {
    int32_t n_keys;               /* 1..8; composite keys are concatenated (CCAT)           */
    const blu_key_desc_t* keys;
    int32_t n_vals;               /* 0..16 value (payload) columns, dtype I32, I64, F64 or I128     */
    const blu_dtype_t* vals;
    int32_t n_aggs;               /* 1..16                                                         */
    const blu_agg_desc_t* aggs;
} blu_gby_schema_t;

typedef struct blu_gby_plan_s* blu_gby_plan_t;  /* opaque, immutable, thread-safe */

/* Kernel paths the moderator chooses between ("different implementations of hash-based
 * algorithms based on: 1) number of input rows 2) estimated number of groups 3) number of
 * aggregation functions"). */
typedef enum {
    BLU_PATH_DENSE_SMEM = 0,    /* (a) per-CTA shared-memory tables + CTA->global merge (§4.3.2)   */
    BLU_PATH_HASH_GLOBAL = 1,   /* (b) global open-addressing table, 64-bit key CAS (§4.3.1)       */
    BLU_PATH_DIRECT_GLOBAL = 2  /* (b') dense domain, direct-mapped global table ("mod hash" with a
                                       table >= domain); no key CAS                        */
} blu_path_t;

typedef struct {
    uint64_t n_groups;   /* host value, valid on return                                          */
    int32_t n_keys;
    int32_t n_aggs;      /* finalized: one column per schema aggregate                           */
    int32_t n_states;    /* partial: one column per state field (see blu_gby_plan_info)          */
    int32_t is_partial;  /* 1: state_cols valid, agg_cols NULL                                   */
    int32_t is_host;     /* 1: columns are host memory (blu_gby_execute_host)                     */
    void** key_cols;     /* n_keys arrays, length n_groups, same dtype as the input key columns  */
    void** agg_cols;     /* n_aggs arrays: COUNT -> i64; SUM(int) -> i64; SUM(f64) -> f64;
                            MIN/MAX -> input dtype; AVG -> f64 = (double)SUM / (double)COUNT      */
    void** state_cols;   /* n_states arrays (partial): state field dtypes (plan_info)            */
    void* _owner;        /* library-private                                                     */
} blu_gby_result_t;

/* ---- plan (host only; launches no GPU work) --------------------------------------------------
 * The first plan of a process queries the current device's SM count (cudaDeviceGetAttribute) to
 * size the grid; nothing is allocated or launched.
 * Validates the schema and freezes the plan: path, hash-table capacity ("slightly larger than the
 * estimated number of groups": cap = next_pow2(ceil(max(est,1)/0.7)), >= 1024), slot
 * layout (key + state fields padded to a power of two, "1, 2, 4, 8 or 16 byte aligned"),
 * shared-memory bytes and grid. est_groups is clamped to [1, n_rows]; n_rows is the exact row
 * count and may be 0. Errors: BLU_E_INVALID (NULL / bad schema), BLU_E_UNSUPPORTED (a key
 * tuple wider than 128 bits, or an AoS slot of more than 256 bytes, e.g. 16 aggregates over 128-bit
 * payloads).
 * Environment overrides for tests and benchmarks only: BLU_GBY_FORCE_PATH=a|b|d,
 * BLU_GBY_HOT_FRONT=0|1. */
blu_status_t blu_gby_plan(const blu_gby_schema_t* schema, uint64_t est_groups, uint64_t n_rows,
                          blu_gby_plan_t* out_plan);

/* Plan introspection. Any out pointer may be NULL. path: blu_path_t; capacity: slots of the
 * global table (path b) or dense domain size (paths a, b'); smem_bytes: dynamic shared memory per
 * CTA of the aggregation kernel; retries_last: table regrowths in the last execute on this plan
 * (P:141 error path); hot_front: 1 if path (b) uses a per-CTA shared-memory hot-key front. */
blu_status_t blu_gby_plan_info(blu_gby_plan_t plan, int32_t* path, uint64_t* capacity,
                               uint32_t* smem_bytes, uint32_t* retries_last);
/* Full plan description (all fields filled). */
typedef struct {
    int32_t path;            /* blu_path_t                                                         */
    uint64_t capacity;       /* hash slots (b) or dense domain D (a, b')                           */
    uint64_t est_groups;     /* the clamped estimate the plan was sized from                      */
    uint32_t slot_bytes;     /* global AoS slot (key + state fields, padded)                      */
    uint32_t smem_bytes;     /* dynamic shared memory of the aggregation kernel                   */
    int32_t hot_front;       /* 1: shared-memory hot-key front (b, b')                            */
    uint32_t front_slots;
    uint32_t partitions;     /* (b): buckets of the partitioned two-pass mode (1 = one pass)      */
    int32_t n_states;        /* state fields (partial results / records)                         */
    int32_t state_dtypes[32];/* blu_dtype_t of each state field                                   */
    uint32_t grid, block;    /* aggregation launch shape                                          */
    uint32_t retries_last;
    int32_t row_lock;        /* (b): kernel 3 — one row lock per slot, then every aggregate */
    int32_t part_smem;       /* (b) partitioned: 1 = pass 2 aggregates each bucket in a per-CTA
                                shared-memory table and merges it once per piece       */
    uint32_t bucket_entries; /* part_smem: entries of that table                                   */
} blu_gby_plan_desc_t;
blu_status_t blu_gby_plan_describe(blu_gby_plan_t plan, blu_gby_plan_desc_t* out);

/* ---- execute -------------------------------------------------------------------------------
 * key_cols: n_keys DEVICE arrays of n_rows elements (dtype per schema); val_cols: n_vals DEVICE
 * arrays. Runs S4 init, S5 aggregate, S6 overflow check (+ regrow and rerun), S8 compaction
 * on `stream`; synchronizes `stream` once (flags + n_groups) and returns. Groups come out in table
 * order (SQL leaves the order unspecified). Errors: BLU_E_KEY_RANGE (no partial result is
 * returned), BLU_E_OOM, BLU_E_CUDA. n_rows == 0 gives n_groups == 0. */
blu_status_t blu_gby_execute(blu_gby_plan_t plan, const void* const* key_cols, const void* const* val_cols,
                             uint64_t n_rows, void* stream, blu_gby_result_t* out);

/* Same on HOST columns: the rows are copied to the device in chunks (two staging buffers, copy of
 * chunk i+1 overlapped with aggregation of chunk i), the result is returned in host memory
 * (is_host = 1). Host columns that are pinned (cudaHostRegister / cudaMallocHost) copy fastest. */
blu_status_t blu_gby_execute_host(blu_gby_plan_t plan, const void* const* host_key_cols,
                                  const void* const* host_val_cols, uint64_t n_rows, void* stream,
                                  blu_gby_result_t* out);

/* Partial result: per group, the state fields (is_partial = 1) instead of finalized aggregates.
 * State fields (plan_info2): COUNT -> i64; integer SUM -> i64; f64 SUM -> f64; MIN/MAX -> input
 * dtype. AVG is carried as its (SUM, COUNT) fields. */
blu_status_t blu_gby_execute_partial(blu_gby_plan_t plan, const void* const* key_cols,
                                     const void* const* val_cols, uint64_t n_rows, void* stream,
                                     blu_gby_result_t* out);

/* S9: re-aggregate n_partials partial results (device, from execute_partial / merge_partial of a
 * plan with the same schema): COUNT->SUM, SUM->SUM, MIN->MIN, MAX->MAX. merge finalizes,
 * merge_partial keeps states. */
blu_status_t blu_gby_merge(blu_gby_plan_t plan, const blu_gby_result_t* partials, int32_t n_partials,
                           void* stream, blu_gby_result_t* out);
blu_status_t blu_gby_merge_partial(blu_gby_plan_t plan, const blu_gby_result_t* partials,
                                   int32_t n_partials, void* stream, blu_gby_result_t* out);

/* ---- multi-GPU helpers (collectives are issued by the caller's NCCL process group) -----------
 * Dense state (paths a and b'): state_arrays[0..3] are caller-allocated DEVICE arrays grouped by
 * reduce op so that four allreduces combine ranks:
 *   [0] int64 SUM group  (COUNT and integer SUMs)      n_isum x D   int64
 *   [1] f64 SUM group                                  n_fsum x D   double
 *   [2] MIN group (integers widened to int64; f64 via an order-preserving int64 map)  n_min x D
 *   [3] MAX group (same encoding)                      n_max x D   int64
 * blu_gby_dense_state_shape reports (n_isum, n_fsum, n_min, n_max, D). execute_dense_state
 * initializes the arrays (init = 1) or accumulates into them (init = 0). */
blu_status_t blu_gby_dense_state_shape(blu_gby_plan_t plan, int32_t* n_isum, int32_t* n_fsum, int32_t* n_min,
                                       int32_t* n_max, uint64_t* domain);
blu_status_t blu_gby_execute_dense_state(blu_gby_plan_t plan, const void* const* key_cols,
                                         const void* const* val_cols, uint64_t n_rows, void* stream,
                                         void* const* state_arrays, int32_t init);
blu_status_t blu_gby_finalize_dense_state(blu_gby_plan_t plan, void* const* state_arrays, void* stream,
                                          blu_gby_result_t* out);

/* Hash path exchange (path b): records are rows of (W + n_states) 64-bit words, W = 1 (or 2 for
 * wide keys, see blu_key_desc_t):
 *   words 0..W-1 = packed key (the code for a sparse key; mixed radix sum code_j * prod_{i<j} d_i
 *            for a dense composite key; per word for wide keys), words W.. = state fields as 64-bit
 *            (i32 states sign-extended, f64 states as their bits). Wide-key owners use
 *            mulhi(fmix64(w0 ^ fmix64(w1 ^ 0x9E3779B97F4A7C15)), n_parts).
 * blu_gby_partition writes the groups of `partial` into send_buf (DEVICE, capacity
 * n_groups x record bytes) bucketed by owner rank = mulhi(fmix64(packed), n_parts) — bits
 * independent of the slot bits — in rank order, and sets send_counts[p] (HOST) to the number of
 * records for rank p. blu_gby_merge_records aggregates n_records such records (DEVICE) into a
 * finalized (or partial, if partial_out = 1) result. */
blu_status_t blu_gby_partition(blu_gby_plan_t plan, const blu_gby_result_t* partial, int32_t n_parts,
                               void* stream, void* send_buf, uint64_t* send_counts);
blu_status_t blu_gby_merge_records(blu_gby_plan_t plan, const void* records, uint64_t n_records,
                                   void* stream, int32_t partial_out, blu_gby_result_t* out);
uint32_t blu_gby_record_bytes(blu_gby_plan_t plan);

/* Rows mode of the hash-path exchange (chosen when est_groups >= rows per rank,
 * i.e. partial states would not be smaller than the rows): raw ROWS are bucketed by owner and the
 * owner aggregates them. Row records are (W + n_vals) 64-bit words: the packed key as above, then
 * every value column as 64 bits (i32 sign-extended, f64 bits). blu_gby_partition_rows writes the
 * n_rows rows of key_cols / val_cols (DEVICE, the execute layout) into send_buf (DEVICE, capacity
 * n_rows x row record bytes) by owner, sets send_counts[p] (HOST), and synchronises `stream`.
 * Errors: BLU_E_KEY_RANGE (a key outside its dictionary / negative sparse code; nothing usable is
 * written), BLU_E_UNSUPPORTED for 128-bit payloads. blu_gby_execute_records runs S4-S8 over
 * n_records such records (DEVICE) with a hash table sized from the plan's estimate: the rows this
 * rank owns, aggregated into a finalized (or partial) result. */
blu_status_t blu_gby_partition_rows(blu_gby_plan_t plan, const void* const* key_cols, const void* const* val_cols,
                                    uint64_t n_rows, int32_t n_parts, void* stream, void* send_buf,
                                    uint64_t* send_counts);
blu_status_t blu_gby_execute_records(blu_gby_plan_t plan, const void* records, uint64_t n_records, void* stream,
                                     int32_t partial_out, blu_gby_result_t* out);
uint32_t blu_gby_row_record_bytes(blu_gby_plan_t plan);

/* ---- group-count estimate --------------------------------------------
 * KMV ("K-minimum values") estimate of the number of distinct key tuples in n_rows DEVICE key
 * columns — the estimate the paper computes on CPU threads right after hashing and feeds to the GPU
 * runtime ("use a simple hash function and KMV[2] algorithm to estimate the number of
 * groups"). est = (k-1) * 2^64 / (k-th smallest distinct 64-bit key hash); if fewer than k
 * distinct hashes exist the count is exact (*exact = 1). Relative standard error ~ 1/sqrt(k-2).
 * k in [16, 2048]. Depends only on the set of keys (not on row order or launch shape). Synchronises
 * `stream`. Errors: BLU_E_INVALID, BLU_E_UNSUPPORTED, BLU_E_KEY_RANGE (a code outside its
 * dictionary), BLU_E_OOM. */
blu_status_t blu_gby_estimate_groups(const blu_key_desc_t* keys, int32_t n_keys, const void* const* key_cols,
                                     uint64_t n_rows, uint32_t k, void* stream, double* est, int32_t* exact);

/* ---- S4 table initialisation (Table 1) -------------------------------------
 * The slot template ("hash table mask"): key all-ones ("M/4 Fs"), SUM 0, MAX the type minimum,
 * MIN the type maximum, COUNT 0, padding 0. slot_template copies slot_bytes bytes into `out`
 * (HOST, capacity cap bytes); init_table writes the template into n_slots consecutive slots of a
 * DEVICE buffer with parallel threads. */
blu_status_t blu_gby_slot_template(blu_gby_plan_t plan, void* out, uint32_t cap, uint32_t* slot_bytes);
blu_status_t blu_gby_init_table(blu_gby_plan_t plan, void* dev_table, uint64_t n_slots, void* stream);

/* ---- instrumentation ------------------------------------------------------------------------
 * With timing enabled, execute* record CUDA events on `stream` around each phase; last_timing
 * returns the phase times (ms) of the last execute on this thread: init, aggregate (S5, summed
 * over chunks/retries), compact (S8), h2d (execute_host). launch_count: total kernels this
 * library has launched in the process. */
typedef struct {
    float init_ms, aggregate_ms, compact_ms, h2d_ms, total_ms;
    uint32_t aggregate_launches, retries;
    char kernel[64];     /* name of the last aggregation kernel launched (JIT entry or generic) */
    /* partitioned path (b): the two passes of aggregate_ms, summed over chunks/retries */
    float scatter_ms, pass2_ms;
    uint32_t part_chunks;
    uint32_t part_fallbacks; /* chunks in which a bucket overflowed and the one-pass fallback ran */
} blu_gby_timing_t;
void blu_gby_set_timing(int32_t enable);
blu_status_t blu_gby_last_timing(blu_gby_timing_t* out);
uint64_t blu_gby_launch_count(void);

/* Diagnostics: compile (NVRTC, no GPU needed, nothing launched) the plan-specialised kernels that
 * execute would JIT for this plan, with the NVRTC the library loads. Returns BLU_OK if every program
 * compiled; BLU_E_UNSUPPORTED if one failed (its log goes to `log`, HOST, log_cap bytes, may be
 * NULL) or the plan has no JIT kernels (wide keys, BLU_GBY_JIT=0) — execute then runs the generic
 * precompiled kernels. *n_programs (may be NULL) = programs compiled. */
blu_status_t blu_gby_jit_probe(blu_gby_plan_t plan, char* log, uint32_t log_cap, int32_t* n_programs);

/* Measurement helper (SURVEY.md §8(d) roofline denominator (i)): reads n_cols DEVICE columns of
 * bytes[i] bytes each (16-byte aligned) once, with the same 128-bit evict-first streaming loads the
 * aggregation kernels use, and XOR-folds them into *dev_out (DEVICE u64) so nothing is elided. The
 * caller times it; bytes / time is the read-only ceiling for the input stream. Grid = 2 CTAs/SM x
 * 512 threads, like path (a). */
blu_status_t blu_gby_read_roofline(const void* const* cols, const uint64_t* bytes, int32_t n_cols, void* stream,
                                   uint64_t* dev_out);

/* Make `device` the current CUDA device of the calling thread for this library (one process per
 * GPU: pass the local rank). */
blu_status_t blu_gby_bind_device(int32_t device);

/* Workspace (hash tables, dense state, partition buffers) is kept in a per-process cache of device
 * blocks reused by later calls (the "single large memory segment" of P:62), and host results in a
 * cache of pinned host blocks. This frees the idle blocks of the current device and the idle pinned
 * host blocks back to CUDA (after a device synchronisation); blocks in use (a live result, a call on
 * another thread) stay. Returns the bytes freed in *freed (may be NULL). */
blu_status_t blu_gby_release_workspace(uint64_t* freed);

void blu_gby_result_free(blu_gby_result_t* r, void* stream);
void blu_gby_plan_destroy(blu_gby_plan_t plan);
const char* blu_gby_status_str(blu_status_t s);
const char* blu_gby_last_error(void);

#ifdef __cplusplus
}
#endif
#endif /* BLU_GBY_H */
