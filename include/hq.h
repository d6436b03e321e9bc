/*
 * hq.h -- C ABI of libhq, the B200-native (sm_100a) fused query-pipeline engine.
 *
 * Implements the data-parallel hot path of HorseQC (Funke, Bress, Noll, Markl,
 * Teubner, "Pipelined Query Processing in Coprocessor Environments", SIGMOD'18;
 * /root/reference/PAPER.md, cited as P:<line>):
 *
 *   hq_load_columns   columnar input, resident in device memory before the
 *                     query runs.
 *   hq_build_hash     the pipeline breaker of a join: dimension rows filtered by
 *                     their predicates and inserted into an open-addressing hash
 *                     table in global memory with atomics (P:186-195,
 *                     P:1033-1036; Table 4 "Pipeline Breaker").
 *   hq_run_pipeline   one *fusion operator* (P:495-500): a plan descriptor
 *                     scan -> filter -> probe* -> compute -> aggregate |
 *                     materialise, executed as ONE compound kernel (§5.2,
 *                     Fig 12) whose write offsets / aggregates use
 *                     local resolution + global propagation (§6.1, P:1056-1210;
 *                     Fig 25).  The same descriptor can also be run
 *                     operator-at-a-time (Fig 6) as the bytes-moved
 *                     baseline (HQ_EXEC_OAAT).
 *   hq_fetch_result   post-processing outside the pipeline (ORDER BY, LIMIT,
 *                     AVG) and the device->host copy.
 *
 * ---------------------------------------------------------------------------
 * Conventions
 *  - Every call returns hq_status (0 = HQ_OK, negative = error).  Out-params are
 *    written only on HQ_OK.  No exception, abort or exit crosses the ABI.  The
 *    message of the last failing call of the calling thread: hq_last_error().
 *  - Device work is enqueued asynchronously on the context stream (the caller's
 *    cudaStream_t, typically torch's current stream).  Device-side faults
 *    detected inside kernels (duplicate build key, int64 overflow guard, group
 *    key out of its declared domain, hash-table or capacity overflow) are raised
 *    at the next *syncing* call on that object: hq_hash_info, hq_result_info_get,
 *    hq_fetch_result, hq_finalize (when it has to size a sort).
 *  - Ownership: the library owns device memory of tables loaded with
 *    HQ_HOST_COPY, of hash tables and of results; it is allocated through the
 *    caller-supplied hq_allocator (NULL: cudaMallocAsync on the ctx stream).
 *    The caller owns host buffers, device buffers passed with
 *    HQ_DEVICE_BORROW / hq_hash_import (they must outlive the handle) and the
 *    stream.  Handles are reference counted internally: hq_free_* releases the
 *    caller's reference; memory goes away once no hash/result uses it.
 *  - Layout: columns are dense arrays (SoA), one value per row, little endian,
 *    int8 / int32 / int64.  Device column pointers must be 16-byte aligned
 *    (HQ_ERR_ARG otherwise) -- required by the TMA bulk copies of the pipeline.
 *  - Limits: <=16 columns per table, <=16 ops, <=4 probes payload words,
 *    <=4 group keys, <=8 aggregates, <=8 output columns, <=8 temporaries,
 *    <=64 expression instructions per plan.  Larger plans: HQ_ERR_UNSUPPORTED.
 *    There is no CPU fallback: without a CUDA device every call fails with
 *    HQ_ERR_NO_DEVICE.
 *  - Threading: a context may be used by one host thread at a time.
 */
#ifndef HQ_H
#define HQ_H
#include <stddef.h>
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

#define HQ_ABI_VERSION 1

typedef int32_t hq_status;
enum {
  HQ_OK = 0,
  HQ_ERR_ARG = -1,         /* invalid argument / plan */
  HQ_ERR_CUDA = -2,        /* CUDA runtime error */
  HQ_ERR_OOM = -3,         /* allocation failed */
  HQ_ERR_DUP_KEY = -4,     /* duplicate key inserted into a join hash table */
  HQ_ERR_UNSUPPORTED = -5, /* plan exceeds the limits above */
  HQ_ERR_OVERFLOW = -6,    /* int64 guard, group table or output capacity exceeded */
  HQ_ERR_STATE = -7,       /* object in the wrong state for the call */
  HQ_ERR_NO_DEVICE = -8    /* no CUDA device */
};

typedef enum { HQ_I8 = 1, HQ_I32 = 3, HQ_I64 = 4, HQ_F64 = 5 } hq_type;

#define HQ_MAX_COLS 16
#define HQ_MAX_OPS 16
#define HQ_MAX_PAYLOAD 3
#define HQ_MAX_KEYS 4
#define HQ_MAX_AGGS 8
#define HQ_MAX_OUT 8
#define HQ_MAX_TMP 8
#define HQ_MAX_INSN 16
#define HQ_MAX_PREDS 8
#define HQ_MAX_ORDER 4
/* Register numbering inside a plan: 0..ncols-1 are the fact table's columns,
 * HQ_TMP(k) (k < HQ_MAX_TMP) are temporaries written by PROBE payloads (int32)
 * and COMPUTE ops (int64). */
#define HQ_TMP(k) (0x100 + (k))

typedef struct hq_ctx hq_ctx;
typedef struct hq_table hq_table;
typedef struct hq_hash hq_hash;
typedef struct hq_result hq_result;
typedef struct hq_graph hq_graph;

/* Device memory hooks.  alloc returns a device pointer (>= 256-B aligned) or
 * NULL; both are called with the ctx stream. */
typedef struct {
  void* (*alloc)(size_t bytes, void* stream, void* user);
  void (*free)(void* ptr, size_t bytes, void* stream, void* user);
  void* user;
} hq_allocator;

/* ---------------------------------------------------------------- context */
/* device: CUDA ordinal; stream: cudaStream_t (NULL = legacy default stream);
 * alloc: NULL = cudaMallocAsync/cudaFreeAsync on the stream. */
hq_status hq_ctx_create(int32_t device, void* stream, const hq_allocator* alloc, hq_ctx** out);
hq_status hq_ctx_destroy(hq_ctx* ctx);
hq_status hq_ctx_set_stream(hq_ctx* ctx, void* stream);
hq_status hq_ctx_sync(hq_ctx* ctx);
/* Thread-local message of the last non-OK status (never NULL). */
const char* hq_last_error(void);
int32_t hq_abi_version(void);
/* sizeof of the public structs, so bindings can check their mirrors. */
size_t hq_sizeof(const char* struct_name);

/* Kernel timing: when enabled, CUDA events are recorded on the ctx stream
 * around every fused-pipeline kernel launch.  hq_ctx_kernel_times syncs and
 * returns (and clears) the durations in ms, oldest first; *n = count. */
hq_status hq_ctx_enable_timing(hq_ctx* ctx, int32_t on);
hq_status hq_ctx_kernel_times(hq_ctx* ctx, float* ms, int32_t max, int32_t* n);
/* Cumulative number of CUDA kernels this context has launched. */
hq_status hq_ctx_launches(hq_ctx* ctx, int64_t* n);

/* ----------------------------------------------------------------- tables */
typedef struct {
  const char* name; /* informational, may be NULL */
  int32_t type;     /* hq_type: HQ_I8, HQ_I32 or HQ_I64 */
  int32_t reserved;
  const void* data; /* host pointer (HQ_HOST_COPY) or device pointer (HQ_DEVICE_BORROW) */
} hq_column;
#define HQ_HOST_COPY 1     /* library allocates device memory and copies (async; host buffer must stay valid until the next ctx sync) */
#define HQ_DEVICE_BORROW 2 /* data are device pointers kept alive by the caller */
/* HQ_HOST_STREAM: data are HOST pointers kept alive (and unchanged) by the caller until
 * every pipeline over the table has completed; nothing is copied at load time.  A
 * pipeline whose fact table is such a table runs as batch processing (§3,
 * P:220-305; Exp 5): blocks of rows are copied over the host link into a
 * double-buffered device ring on a copy stream while the compound kernel processes the
 * previous block on the context stream, and the sink's state (group table, output
 * counter) carries over the blocks, so the result equals the HBM-resident run.  Pinned
 * host memory (cudaHostAlloc / cudaHostRegister) is needed for the copies to overlap.
 * Only fused execution streams (HQ_EXEC_FUSED / HQ_EXEC_FUSED_INTERP); hash builds and
 * hq_table_column need device tables (HQ_ERR_UNSUPPORTED). */
#define HQ_HOST_STREAM 3
hq_status hq_load_columns(hq_ctx* ctx, const hq_column* cols, int32_t ncols, int64_t nrows,
                          int32_t flags, hq_table** out);
hq_status hq_table_info(const hq_table* t, int64_t* nrows, int32_t* ncols);
/* Column statistics for the planner: min and max of column `col` over all rows (one
 * device reduction, syncs the context).  An empty table gives *min > *max.  Used to
 * declare tight GROUP BY key domains (a dense group table needs no hash claim, see
 * hq_plan::key_card). */
hq_status hq_column_range(hq_ctx* ctx, const hq_table* t, int32_t col, int64_t* min, int64_t* max);
hq_status hq_table_column(const hq_table* t, int32_t col, const void** dev_ptr, int32_t* type);
hq_status hq_free_table(hq_table* t);

/* ------------------------------------------------------------- predicates */
typedef enum {
  HQ_EQ = 1, HQ_NE, HQ_LT, HQ_LE, HQ_GT, HQ_GE,
  HQ_BETWEEN,   /* lo <= v <= hi (SQL BETWEEN, inclusive) */
  HQ_IN_BITMAP  /* 0 <= v < 256 and bit v of bitmap set (IN-lists over dictionary codes) */
} hq_cmp;
typedef struct {
  int32_t reg;   /* column (build side: column of the source table) or HQ_TMP(k) */
  int32_t cmp;   /* hq_cmp */
  int64_t lo;    /* comparison constant (EQ..GE) / lower bound (BETWEEN) */
  int64_t hi;    /* upper bound (BETWEEN) */
  uint64_t bitmap[4];
} hq_pred;

/* ------------------------------------------------------------ hash build */
typedef struct {
  const hq_table* src;   /* dimension table, or hq_result_as_table of a materialised result */
  int32_t npreds;
  hq_pred preds[HQ_MAX_PREDS]; /* conjunction over src columns */
  int32_t key_col;       /* int32 (or int8/int64 whose values fit int32, != INT32_MIN) */
  int32_t npayload;      /* 0 = semi-join table (keys only), 1..3 payload columns (values must fit int32) */
  int32_t payload_cols[HQ_MAX_PAYLOAD];
  int64_t expected_rows; /* >0: capacity sized for this many keys (no count pass, no host sync);
                            <=0: a count pass sizes the table exactly (one ctx sync) */
  int32_t composite;     /* != 0: two-column join key (key_col, payload_cols[0]) (TPC-H Q9's
                            (ps_partkey, ps_suppkey)): the slot is hashed on key_col, stores the
                            second key as payload word 0 and the remaining payload columns after
                            it; key_col alone need not be unique, the pairs must be (not checked).
                            Always HQ_HT_LINEAR; npayload >= 1. */
} hq_build_desc;
/* Slot = {int32 key, payload...} of 4, 8 or 16 bytes, empty key INT32_MIN,
 * claimed with one atomicCAS on the key.  Two layouts:
 *  - HQ_HT_DIRECT (dense keys, chosen when the count pass finds the qualifying
 *    keys' range <= 8 x their number or the array <= 2 MiB): slot = key - key_min,
 *    one load per probe;
 *  - HQ_HT_LINEAR: multiplicative hash, linear probing, power-of-two capacity
 *    >= keys/0.6; probes scan whole aligned 16-B slot groups per load.
 * Duplicate keys: HQ_ERR_DUP_KEY at hq_hash_info. */
hq_status hq_build_hash(hq_ctx* ctx, const hq_build_desc* desc, hq_hash** out);
/* Several builds with ONE host synchronisation (the build
 * pipelines of a query's dimension tables are independent): the count passes of
 * all n descriptors run first, their statistics are read back together, then
 * every table is sized, built and compacted stream-ordered.  descs: n
 * contiguous descriptors (host memory, read during the call); out: n handles,
 * all written on HQ_OK, none on error (nothing leaks).  n >= 1. */
hq_status hq_build_hashes(hq_ctx* ctx, int32_t n, const hq_build_desc* descs, hq_hash** out);
enum { HQ_HT_LINEAR = 0, HQ_HT_DIRECT = 1 };
typedef struct {
  int64_t capacity;     /* slots (power of two for HQ_HT_LINEAR, key range for HQ_HT_DIRECT) */
  int32_t slot_words;   /* 1, 2 or 4 int32 words per slot */
  int32_t npayload;
  int64_t nkeys;        /* keys inserted (valid after hq_hash_info) */
  int64_t bytes;        /* capacity * slot_words * 4 */
  int64_t key_min;      /* HQ_HT_DIRECT: key stored in slot 0 */
  int32_t layout;       /* HQ_HT_LINEAR or HQ_HT_DIRECT */
  int32_t pay_min;      /* min / max of payload 0 over the inserted rows (count pass) */
  int32_t pay_max;
  int32_t key_max;      /* max key inserted (count pass); key range = [key_min, key_max] */
  uint64_t pay_set[4];  /* payload-0 values present: bit (v & 255) (count pass); exact when
                         * pay_max - pay_min < 256, all-zero when unknown (expected_rows builds) */
  int32_t composite;    /* built with hq_build_desc::composite (payload word 0 = second key) */
  int32_t compact_kind; /* hq_hash_device_view / hq_hash_import: 0 = the buffer is the slot array; 1 / 2 / 3 =
                         * the buffer is the compact form of a direct table (1 bitmap of present keys, 2 one
                         * byte per key, 3 one nibble per key; see below) -- tables whose only consumers
                         * read that form are built straight into it; 4 = the ranked form of a linear
                         * table (below; needs key_min / key_max / nkeys) */
} hq_hash_meta;
/* Derived forms (rebuilt on import): direct tables get a compact form -- a
 * bitmap of present keys for semi-join tables, or one byte per key (payload -
 * pay_min, or the payload's rank among the present payload values when they are a
 * sparse set; 0xFF = absent) when payload 0 spans < 255 values, or one nibble per
 * key when it spans < 15 -- that generated kernels stage in shared memory.  Such a
 * direct table is built straight into its compact form (one atomic per row, duplicate
 * keys detected by it); its slot array is derived only if a consumer that reads slots
 * (precompiled interpreter, operator-at-a-time) probes it.  hq_hash_device_view then
 * returns the compact form (meta.compact_kind != 0), which hq_hash_import accepts.
 * Sparse unique keys with a counted range that fits in 64 MiB of bits (layout
 * HQ_HT_LINEAR) are built into the *ranked form* instead of a slot array: one buffer
 * [the bitmap of present keys over [key_min, key_max] in 32-bit words -- with payloads
 * as {bits, dir} word pairs, dir = the number of keys before the word | payload rows
 * by rank, 1 / 2 / 4 int32 words each (npayload 1 / 2 / 3)], the bitmap padded to
 * whole 8,192-word blocks -- a probe tests the key's bit (misses stop there) and reads
 * row dir + popcount(bits below it).  The linear slot array the
 * meta describes (capacity, slot_words, bytes) is derived only for consumers that
 * read slots.  Other linear tables (expected_rows builds, composite keys, wider
 * ranges) keep the slot array, with an exact key-range bitmap in front of it when
 * the range fits in 64 MiB of bits. */
hq_status hq_hash_info(hq_ctx* ctx, const hq_hash* h, hq_hash_meta* meta);  /* syncs, reports build faults */
/* Multi-GPU glue: raw device view of the slot array (to broadcast it with NCCL)
 * and import of such a buffer on another device (borrowed, caller keeps it). */
hq_status hq_hash_device_view(const hq_hash* h, void** dev_ptr, hq_hash_meta* meta);
hq_status hq_hash_import(hq_ctx* ctx, const hq_hash_meta* meta, void* dev_ptr, hq_hash** out);
hq_status hq_free_hash(hq_hash* h);

/* ------------------------------------------------------------------ plans */
typedef enum { HQ_OP_FILTER = 1, HQ_OP_PROBE = 2, HQ_OP_COMPUTE = 3 } hq_op_kind;
/* INNER: row survives on a match, payload words -> payload_dst temps.
 * SEMI / ANTI: row survives on a match / on no match (EXISTS / NOT EXISTS).
 * OUTER: LEFT OUTER JOIN: the row always survives; payload_dst temps get the
 *        matching slot's payload words, or 0 when the key is absent
 *        (COALESCE(payload, 0)); build keys are unique, so at most one match. */
typedef enum { HQ_PROBE_INNER = 0, HQ_PROBE_SEMI = 1, HQ_PROBE_ANTI = 2, HQ_PROBE_OUTER = 3 } hq_probe_mode;
/* Expression code: an accumulator machine evaluated per row in int64.
 * operand = register `reg`, or the immediate `imm` when reg < 0. */
typedef enum {
  HQ_I_LOAD = 1, /* acc = operand            */
  HQ_I_ADD,      /* acc = acc + operand      */
  HQ_I_SUB,      /* acc = acc - operand      */
  HQ_I_RSUB,     /* acc = operand - acc      */
  HQ_I_MUL,      /* acc = acc * operand      */
  HQ_I_DIV,      /* acc = acc / operand (C truncation; /0 -> HQ_ERR_ARG) */
  HQ_I_MOD,      /* acc = acc % operand (C semantics; %0 -> HQ_ERR_ARG) */
  /* Predicate instructions (boolean acc, 0/1): acc = (acc != 0 && reg CMP imm).
   * They read BOTH fields: reg (>= 0, a column or temp) and the constant imm, so a
   * conjunction over several registers is one expression (e.g. one disjunct of
   * TPC-H Q19's WHERE clause). */
  HQ_I_AND_EQ,   /* acc = acc && reg == imm */
  HQ_I_AND_NE,   /* acc = acc && reg != imm */
  HQ_I_AND_LT,   /* acc = acc && reg <  imm */
  HQ_I_AND_LE,   /* acc = acc && reg <= imm */
  HQ_I_AND_GT,   /* acc = acc && reg >  imm */
  HQ_I_AND_GE,   /* acc = acc && reg >= imm */
  HQ_I_AND_IN,   /* acc = acc && 0 <= reg < 64 && bit reg of (uint64)imm (IN-list over codes < 64) */
  HQ_I_OR        /* acc = acc || operand != 0 (disjunction with another predicate temp) */
} hq_opcode;
typedef struct {
  int32_t opc;
  int32_t reg;
  int64_t imm;
} hq_insn;
typedef struct {
  int32_t kind;           /* hq_op_kind */
  /* FILTER */
  hq_pred filter;
  /* PROBE: row survives if key found (INNER/SEMI) or not found (ANTI);
   * INNER copies the matching slot's payload words to payload_dst temps. */
  const hq_hash* ht;
  int32_t key_reg;
  int32_t mode;           /* hq_probe_mode */
  int32_t npayload;
  int32_t payload_dst[HQ_MAX_PAYLOAD];
  /* COMPUTE: dst temp = value of code[0..ninsn) */
  int32_t dst;
  int32_t ninsn;
  hq_insn code[HQ_MAX_INSN];
  /* PROBE of a composite table: register holding the second key (compared with the
   * slot's payload word 0); payload_dst[k] then receive payload words 1 + k. */
  int32_t key2_reg;
} hq_op;

typedef enum { HQ_AGG_SUM = 1, HQ_AGG_COUNT, HQ_AGG_MIN, HQ_AGG_MAX, HQ_AGG_AVG } hq_agg_fn;
typedef enum { HQ_SINK_AGG = 1, HQ_SINK_MATERIALISE = 2 } hq_sink_kind;
/* Reduction technique of the sink (Table 4):
 * LRGP = local resolution in registers/shared memory + global propagation with
 *        one atomic per block and tile (A3, B3, C3) -- the default; its local
 *        resolution is SIMD-style (warp shuffles/ballots, App C "SIMD Reduction");
 * ATOMIC = per-row global atomics (A2, B2, C2), kept as an ablation;
 * WE = local resolution by work-efficient (Blelloch) trees in shared memory with one
 *        barrier per level, one pre-aggregate / write offset per workgroup and tile
 *        (App C "Work-Efficient Reduction", Fig 24): A3-WE exclusive scan
 *        of the row flags, B3-WE tree reduction, C3-WE sort by key + segmented scan +
 *        atomic hash reduce of each segment.  Generated fused kernels
 *        only (HQ_EXEC_FUSED; HQ_ERR_UNSUPPORTED otherwise); an ablation. */
typedef enum { HQ_RES_LRGP = 0, HQ_RES_ATOMIC = 1, HQ_RES_WE = 2 } hq_resolution;
/* Execution of a plan:
 * FUSED        one compound kernel, compiled for this plan with NVRTC (query
 *              compilation); falls back to FUSED_INTERP
 *              only if HQ_JIT=0 is set in the environment;
 * OAAT         operator-at-a-time baseline (Fig 6);
 * FUSED_INTERP the same compound kernel as a precompiled descriptor interpreter;
 * MULTIPASS    multi-pass query compilation (§4, Fig 7-9; Table 4
 *              A1/B1/C1): a generated count kernel (selections and join probes
 *              -> one int32 flag per row), a prefix sum over the flags, a
 *              generated write kernel (projections / aggregation inputs of the
 *              flagged rows at their prefix-sum positions) and, for AGG sinks,
 *              library reductions (reduce; radix sort + reduce-by-key).  Same
 *              results as FUSED (materialised rows in row order); one host
 *              synchronisation (the qualifying count sizes the outputs). */
typedef enum { HQ_EXEC_FUSED = 0, HQ_EXEC_OAAT = 1, HQ_EXEC_FUSED_INTERP = 2, HQ_EXEC_MULTIPASS = 3 } hq_exec;

typedef struct {
  const hq_table* fact;
  int64_t row_begin, row_end; /* range partition of the fact table; row_end < 0 = all rows */
  int32_t nops;
  hq_op ops[HQ_MAX_OPS];
  int32_t sink;               /* hq_sink_kind */
  int32_t resolution;         /* hq_resolution */
  int32_t exec;               /* hq_exec */
  int32_t ntmp_types;         /* unused, must be 0 */
  /* AGG sink: GROUP BY key_reg[] (each value v must satisfy key_min <= v <
   * key_min + key_card; the packed index sum((v-min)*stride) selects a dense
   * table when prod(card) <= 65536, else a global hash table -- or, for fused
   * execution, a dense global table when prod(card) <= 2^28 and its size is at
   * most twice the hash table's: a group update is then two fire-and-forget
   * atomics instead of a claim round trip); aggregates. */
  int32_t nkeys;
  int32_t key_reg[HQ_MAX_KEYS];
  int64_t key_min[HQ_MAX_KEYS];
  int64_t key_card[HQ_MAX_KEYS];
  int32_t naggs;
  int32_t agg_fn[HQ_MAX_AGGS];    /* hq_agg_fn */
  int32_t agg_reg[HQ_MAX_AGGS];   /* ignored for COUNT */
  int32_t agg_scale[HQ_MAX_AGGS]; /* AVG: result = sum / count / 10^scale (fp64) */
  int64_t group_capacity;         /* hash group-by: expected #groups (0 = auto) */
  /* MATERIALISE sink: output columns out_reg[] cast to out_type[] */
  int32_t nout;
  int32_t out_reg[HQ_MAX_OUT];
  int32_t out_type[HQ_MAX_OUT];
  int64_t capacity;               /* output rows (0 = rows of the range) */
  /* post-processing of AGG results: ORDER BY result columns
   * (keys first, then aggregates), remaining ties by the group keys; LIMIT. */
  int32_t norder;
  int32_t order_col[HQ_MAX_ORDER];
  int32_t order_desc[HQ_MAX_ORDER];
  int64_t limit;                  /* <= 0: no limit */
} hq_plan;

/* Enqueue the pipeline (async).  The plan is copied; hash tables and the fact
 * table it references are retained by the result. */
hq_status hq_run_pipeline(hq_ctx* ctx, const hq_plan* plan, hq_result** out);
/* Batch processing over an HQ_HOST_STREAM fact table with an explicit block size:
 * block_rows > 0 is rounded up to the kernel's tile (hq_run_pipeline uses
 * HQ_STREAM_BLOCK_ROWS).  Device memory: 2 x block_rows x (bytes of the referenced
 * columns).  HQ_ERR_ARG when the fact table is not HQ_HOST_STREAM. */
#define HQ_STREAM_BLOCK_ROWS (1 << 24)
hq_status hq_run_pipeline_streamed(hq_ctx* ctx, const hq_plan* plan, int64_t block_rows, hq_result** out);
/* Post-process an AGG result in place (compaction, AVG, ORDER BY, LIMIT);
 * idempotent; implied by hq_result_info_get / hq_fetch_result. */
hq_status hq_finalize(hq_ctx* ctx, hq_result* r);

typedef struct {
  int64_t nrows;            /* rows of the (finalized, limited) result */
  int64_t qualifying_rows;  /* rows that reached the sink (COUNT(*)) */
  int32_t ncols;
  int32_t types[HQ_MAX_KEYS + HQ_MAX_AGGS]; /* hq_type of each result column */
  int32_t segment_rows;     /* MATERIALISE: fact rows per LRGP segment (the kernel's tile);
                               output is ordered within a segment's rows, segments permuted.
                               0: warp workgroups (generated kernels behind a global probe) --
                               each warp's buffered rows are one segment, in row order */
} hq_result_info;
hq_status hq_result_info_get(hq_ctx* ctx, hq_result* r, hq_result_info* out); /* syncs */
/* Copy the result into caller host buffers host_cols[c] (capacity_rows rows
 * each, typed as hq_result_info.types).  Syncs. */
hq_status hq_fetch_result(hq_ctx* ctx, hq_result* r, void* const* host_cols, int64_t capacity_rows,
                          int64_t* nrows_out);
/* Materialised or (finalized, integer-only) aggregation result viewed as a
 * table (borrows the result's buffers): build input of a later pipeline, or the
 * input of the root's merge pipeline for distributed hash group-bys. */
hq_status hq_result_as_table(hq_ctx* ctx, hq_result* r, hq_table** out);
/* Multi-GPU glue for dense AGG results: the raw partial-aggregate array
 * (int64, ngroups x (1+naggs): [count, agg...]) before finalization, so ranks
 * can sum it with NCCL; only SUM/COUNT/AVG plans (HQ_ERR_UNSUPPORTED else). */
hq_status hq_result_partials_view(hq_result* r, void** dev_ptr, size_t* bytes);
/* Rebuild the dense partial-aggregate array of `r` from the caller's device buffer
 * (same layout as hq_result_partials_view: ngroups x (1+naggs) int64), e.g. after the
 * ranks' partials were summed into a buffer of their own: copies `bytes` bytes into
 * the result's group table on the ctx stream (async).  The result must not be
 * finalized yet; bytes must equal the view's size (HQ_ERR_ARG).  (The reduce itself
 * may also run in place on the view, which needs no call.) */
hq_status hq_result_from_partials(hq_ctx* ctx, hq_result* r, const void* dev_ptr, size_t bytes);
/* The reverse copy: the result's dense partials into the caller's device buffer
 * dev_dst (bytes = the view's size, HQ_ERR_ARG otherwise), async on the ctx stream --
 * e.g. into the [partials | fault words] buffer a multi-rank caller all-reduces, so no
 * collective writes library memory. */
hq_status hq_result_to_partials(hq_ctx* ctx, const hq_result* r, void* dev_dst, size_t bytes);
/* Multi-GPU glue: copy the device views of n hash tables (hq_hash_device_view's
 * buffers, meta.bytes each) into ONE caller buffer dev_dst at byte offsets offs[i]
 * (host array; each 16-B aligned, the caller sized the buffer), async on the ctx
 * stream -- the packed payload of a single table broadcast. */
hq_status hq_hash_pack(hq_ctx* ctx, const hq_hash* const* hashes, int32_t n, const int64_t* offs, void* dev_dst);

/* Fault words gathered on the device, without a host synchronisation, so that a
 * multi-rank caller can combine every rank's faults with the collective it runs
 * anyway and raise on all ranks or on none (a fault seen by one rank alone would
 * leave the others blocked in the next collective).  Writes HQ_FAULT_WORDS int64 to
 * the device buffer dev_out (async, ctx stream): word k (k < 16) = 1 if fault bit k
 * is set in any of the hashes' build fault words, word 16 + k = 1 if bit k is set in
 * any of the results' pipeline fault words, 0 otherwise -- so a SUM reduce over the
 * ranks keeps "some rank saw fault k" as word k != 0.  Imported hashes (no build on
 * this device) contribute nothing.  nh / nr may be 0. */
#define HQ_FAULT_WORDS 32
hq_status hq_gather_faults(hq_ctx* ctx, const hq_hash* const* hashes, int32_t nh, const hq_result* const* results,
                           int32_t nr, int64_t* dev_out);
/* Map HQ_FAULT_WORDS host words (as written by hq_gather_faults, possibly summed over
 * ranks) to a status: HQ_OK when no error fault is set, else the status a syncing call
 * would raise for it (HQ_ERR_DUP_KEY, HQ_ERR_ARG, HQ_ERR_OVERFLOW), with the message in
 * hq_last_error().  The re-runnable pipeline faults (group table full, materialise
 * capacity) are not errors here: the owning result re-runs at its own finalize. */
hq_status hq_raise_faults(const int64_t* host_words);
hq_status hq_free_result(hq_result* r);

/* ------------------------------------------------- prepared queries (CUDA graphs)
 * A query whose steps need no host synchronisation -- its hash builds have cached
 * statistics (a previous build of the same descriptor over the same table, see
 * hq_build_hash), its pipelines are fused, its results are dense aggregates of at most
 * 8,192 groups -- can be recorded once and replayed: between hq_ctx_capture_begin and
 * hq_ctx_capture_end the calls the caller makes (hq_build_hash(es), hq_run_pipeline,
 * hq_finalize) are enqueued into a CUDA graph instead of executed.  Every launch
 * re-executes ALL the recorded device work -- builds (slot fill, insert, compact,
 * statistics verification), the compound kernels, finalization -- into the same
 * buffers, and leaves each finalized result readable (hq_result_info_get /
 * hq_fetch_result) until the next launch.  Only the host-side planning (plan
 * validation, layout, kernel selection, launch configuration) is done once, as for a
 * prepared statement.  Calls that need the host while capturing fail with
 * HQ_ERR_STATE (nothing is recorded after that; call hq_ctx_capture_abort): a build
 * without cached statistics, hq_*_info / fetch, large or materialised finalizes,
 * multi-pass / operator-at-a-time execution, batch processing, hq_load_columns.
 * The graph keeps the objects its nodes use (results, hashes, build source tables)
 * until hq_graph_destroy.  The capture runs on a private stream; launches run on the
 * context stream and synchronise it (the rows are decoded on the host) -- a graph that
 * finalizes no result (e.g. the part of a distributed step before its collective) is
 * launched asynchronously.  Needs the
 * default stream-ordered allocator (no hq_allocator hooks: HQ_ERR_UNSUPPORTED). */
hq_status hq_ctx_capture_begin(hq_ctx* ctx);
hq_status hq_ctx_capture_end(hq_ctx* ctx, hq_graph** out);
hq_status hq_ctx_capture_abort(hq_ctx* ctx);
hq_status hq_graph_launch(hq_ctx* ctx, hq_graph* g);
hq_status hq_graph_destroy(hq_graph* g);

#ifdef __cplusplus
}
#endif
#endif
