// hq_internal.h -- internal objects and the device plan of libhq (not part of
// the ABI).  See include/hq.h for the public contract and DESIGN.md for the
// kernel design.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>
#include <atomic>
#include <cstring>
#include <map>
#include <string>
#include <vector>

#include "hq.h"

// probes whose payload words reach registers (INNER, and OUTER with 0 on a miss)
__host__ __device__ inline bool hq_probe_has_payload(int mode) {
  return mode == HQ_PROBE_INNER || mode == HQ_PROBE_OUTER;
}

// predicate instructions of the expression machine (hq.h HQ_I_AND_* / HQ_I_OR):
// acc is boolean, o the register operand (OR: register or immediate), imm the constant
__host__ __device__ inline long long hq_pred_insn(int opc, long long acc, long long o, long long imm) {
  bool c;
  switch (opc) {
    case HQ_I_AND_EQ: c = o == imm; break;
    case HQ_I_AND_NE: c = o != imm; break;
    case HQ_I_AND_LT: c = o < imm; break;
    case HQ_I_AND_LE: c = o <= imm; break;
    case HQ_I_AND_GT: c = o > imm; break;
    case HQ_I_AND_GE: c = o >= imm; break;
    case HQ_I_AND_IN: c = o >= 0 && o < 64 && (((unsigned long long)imm >> o) & 1ull); break;
    default: return (acc != 0 || o != 0) ? 1 : 0;  // HQ_I_OR
  }
  return (acc != 0 && c) ? 1 : 0;
}

// ---------------------------------------------------------------- errors
struct HqError {
  hq_status code;
  std::string msg;
};
void hq_set_error(const std::string& msg);
#define HQ_THROW(code, msg)               \
  do {                                    \
    throw HqError{(code), (msg)};         \
  } while (0)
#define HQ_CUDA(call)                                                                    \
  do {                                                                                   \
    cudaError_t e_ = (call);                                                             \
    if (e_ != cudaSuccess)                                                               \
      throw HqError{HQ_ERR_CUDA, std::string(#call) + ": " + cudaGetErrorString(e_)};    \
  } while (0)

// Device-side fault bits (KPlan::err), reported at the next syncing call.
enum : int {
  HQF_CAPACITY = 1,     // materialise output capacity exceeded
  HQF_KEY_DOMAIN = 2,   // group key outside [key_min, key_min+key_card)
  HQF_GROUP_FULL = 4,   // global group hash table full
  HQF_DIV_ZERO = 8,     // division / modulo by zero
  HQF_DUP_KEY = 16,     // duplicate build key
  HQF_BAD_KEY = 32,     // build key INT32_MIN or outside int32
  HQF_BAD_PAYLOAD = 64, // build payload outside int32
  HQF_HT_FULL = 128,    // join hash table full (cannot happen when sized by the count pass)
  HQF_OVERFLOW = 256,   // int64 guard tripped (|aggregate| >= 2^62)
  HQF_STALE = 512       // a build's cached statistics do not describe its source rows (hq_build.cu)
};

// Statistics of a build's qualifying rows (count pass): number, key range, payload-0
// range and value set (bit v & 255).  Cached per (source table, descriptor) so that a
// repeated build skips the count pass and its host synchronisation; the insert kernel
// then re-derives them on the device and flags HQF_STALE on any difference.
struct BuildStats {
  unsigned long long cnt;
  int kmin, kmax, pmin, pmax;
  unsigned set[8];
};

// ---------------------------------------------------------------- objects
struct hq_ctx {
  int device = 0;
  cudaStream_t stream = nullptr;
  hq_allocator alloc{};
  bool has_alloc = false;
  int num_sms = 148;
  size_t max_smem = 232448;
  bool timing = false;
  int64_t launches = 0;  // kernels this context has launched (hq_ctx_launches)
  std::vector<std::pair<cudaEvent_t, cudaEvent_t>> events;  // recorded, not yet read
  std::vector<cudaEvent_t> event_pool;
  void* pinned = nullptr;  // host staging for small results (cudaHostAlloc, grown on demand)
  size_t pinned_bytes = 0;
  void* pinned_build = nullptr;  // host staging of the builds' count-pass statistics
  size_t pinned_build_bytes = 0;
  // batch processing of HQ_HOST_STREAM tables: host->device copies run on their own
  // stream, ordered against the pipeline kernels by events (created on first use)
  cudaStream_t copy_stream = nullptr;
  cudaEvent_t ev_copied[2] = {nullptr, nullptr}, ev_consumed[2] = {nullptr, nullptr};
  // concurrent hash builds (hq_build_hashes): side streams forked from / joined to
  // the context stream by events (created on first use)
  static constexpr int NSIDE = 4;
  cudaStream_t side[NSIDE] = {};
  cudaEvent_t ev_fork = nullptr, ev_join[NSIDE] = {};
  // build statistics by (source table uid, descriptor bytes); HQ_BUILD_STATS=0 disables
  std::map<std::string, BuildStats> build_stats;
  // row counts of materialised results viewed as tables, by derived table identity
  // (hq_result_as_table): a repeated view skips the finalize's host synchronisation
  std::map<uint64_t, int64_t> derived_rows;
  // CUDA-graph capture of a prepared query (hq_ctx_capture_begin/_end): the work is
  // captured on cap_stream; allocations come from the pool through alloc_stream (not
  // captured), frees are deferred to the graph's destruction, objects created or
  // read by captured work are retained by the graph, and results finalized during the
  // capture leave their rows in their own pinned staging (decoded after each launch)
  bool capturing = false;
  cudaStream_t user_stream = nullptr, cap_stream = nullptr, alloc_stream = nullptr;
  std::vector<std::pair<void*, size_t>> cap_frees;
  std::vector<struct RefObj*> cap_objs;
  std::vector<struct hq_result*> cap_results;
  int64_t cap_launches0 = 0;
  void* alloc_bytes(size_t bytes);
  void free_bytes(void* p, size_t bytes);
  // Reference count: every table / hash / result holds the context (CtxPtr), so
  // hq_ctx_destroy only drops the caller's reference and the context's streams and
  // staging live until the last object that may still free device memory through it.
  std::atomic<int> refs{1};
  void retain() { refs.fetch_add(1); }
  void release();  // hq_api.cu: the last reference destroys the context
};

// An owning reference to the context, declared as the FIRST member of the library's
// objects so that it is destroyed after their device buffers were freed through it.
struct CtxPtr {
  hq_ctx* c = nullptr;
  CtxPtr() = default;
  CtxPtr(const CtxPtr&) = delete;
  CtxPtr& operator=(const CtxPtr&) = delete;
  CtxPtr& operator=(hq_ctx* n) {
    if (n) n->retain();
    if (c) c->release();
    c = n;
    return *this;
  }
  ~CtxPtr() {
    if (c) c->release();
  }
  operator hq_ctx*() const { return c; }
  hq_ctx* operator->() const { return c; }
};

// A device allocation owned through the context allocator.
struct DevBuf {
  hq_ctx* ctx = nullptr;
  void* p = nullptr;
  size_t bytes = 0;
  DevBuf() = default;
  DevBuf(hq_ctx* c, size_t n) : ctx(c), bytes(n) { p = c->alloc_bytes(n); }
  DevBuf(const DevBuf&) = delete;
  DevBuf& operator=(const DevBuf&) = delete;
  DevBuf(DevBuf&& o) noexcept : ctx(o.ctx), p(o.p), bytes(o.bytes) { o.p = nullptr; }
  DevBuf& operator=(DevBuf&& o) noexcept {
    release();
    ctx = o.ctx; p = o.p; bytes = o.bytes; o.p = nullptr;
    return *this;
  }
  ~DevBuf() { release(); }
  void release() {
    if (p && ctx) ctx->free_bytes(p, bytes);
    p = nullptr;
  }
  template <class T> T* as() const { return (T*)p; }
};

struct RefObj {
  std::atomic<int> refs{1};
  // called for objects created or used by work captured into a CUDA graph
  void capture_retain(hq_ctx* c);
  virtual ~RefObj() {}
  void retain() { refs.fetch_add(1); }
  void release() {
    if (refs.fetch_sub(1) == 1) delete this;
  }
};

inline void RefObj::capture_retain(hq_ctx* c) {
  if (!c || !c->capturing) return;
  retain();
  c->cap_objs.push_back(this);
}

struct hq_result;

struct TableCol {
  const void* ptr = nullptr;
  int type = 0;
  int width = 0;
};

struct hq_table : RefObj {
  CtxPtr ctx;
  uint64_t uid = next_uid();  // never reused (a freed table's address may be)
  static uint64_t next_uid() {
    static std::atomic<uint64_t> n{1};
    return n.fetch_add(1);
  }
  int64_t nrows = 0;
  int ncols = 0;
  TableCol cols[HQ_MAX_COLS];
  std::vector<DevBuf> owned;
  hq_result* backing = nullptr;  // retained when the table views a result
  // a view of a materialised result sized by its cached row count (no host sync): the
  // result's device row counter; consumers check it (builds on the device, pipelines by
  // a host read) and raise HQ_ERR_STATE when it differs from nrows
  const unsigned long long* dev_rows = nullptr;
  bool host_stream = false;      // HQ_HOST_STREAM: cols[].ptr are caller-owned host pointers
  ~hq_table() override;
};

struct hq_hash : RefObj {
  CtxPtr ctx;
  hq_hash_meta meta{};
  int log2cap = 0;
  uint32_t* slots = nullptr;
  DevBuf owned;      // slot array (empty when imported)
  DevBuf dstate;     // [0] fault bits (int), [1..2] nkeys (u64) -- see hq_build.cu
  bool checked = false;
  std::string stats_key;  // its entry in hq_ctx::build_stats (dropped on HQF_STALE)
  // compact form of a direct table (hq_build.cu): 1 = bitmap of present keys
  // (semi-join), 2 = one byte per key (payload0 - pay_min, 0xFF absent),
  // 3 = one nibble per key (payload0 - pay_min < 15, 0xF absent)
  DevBuf compact;
  int ckind = 0;
  int crank = 0;  // ckind 2 holds the rank of payload 0 in meta.pay_set instead of payload - pay_min
  // built straight into the compact form (no slot array until a consumer asks for it:
  // hq_hash_slots); compact_borrow = an imported compact form (not owned)
  bool compact_only = false;
  void* compact_borrow = nullptr;
  const void* compact_ptr() const { return compact.p ? compact.p : compact_borrow; }
  int64_t cbytes = 0;
  // linear tables: exact bitmap over [key_min, key_max] (prefilter before the slots)
  DevBuf prefilter;
  int64_t pf_words = 0;
  // ckind 4 (compact_only): the *ranked* form of a sparse-key (linear) table, one buffer
  // [bitmap of present keys over key_max - key_min + 1 -- with payloads as {bits, dir}
  // word pairs, dir = the number of keys before the word | payload rows by rank, rstride
  // int32 words each] (hq_ranked_layout); a key's payload row = dir + popc(bits below it)
  int64_t src_rows = -1;  // rows of the build's source table (-1: imported / unknown)
  uint64_t src_uid = 0;    // the build's source table (its cached derived row count is dropped on HQF_STALE)
  int64_t roff_dir = 0, roff_pay = 0;
  int rstride = 0;
  bool ranked() const { return ckind == 4; }
};
// byte offsets of the ranked form's parts (and its size) for a key range / key count
void hq_ranked_layout(int64_t range, int64_t nkeys, int npay, int64_t* off_dir, int64_t* off_pay, int64_t* total,
                      int* stride);
void hq_build_compact(hq_ctx* ctx, hq_hash* h);  // derive hq_hash::compact from the slots
int hq_compact_kind(int npayload, int pay_min, int pay_max);
long long hq_compact_words(int kind, long long range);
int hq_rank_lut(const hq_hash_meta& m, unsigned char* lut);
// the slot array of a compact-only table, derived on first use (hq_build.cu)
const uint32_t* hq_hash_slots(hq_ctx* ctx, hq_hash* h);

// ------------------------------------------------- device plan (kernel param)
namespace hqk {
constexpr int NW = 16;                   // consumer warps per CTA
constexpr int NTHREADS = (NW + 1) * 32;  // + 1 TMA producer warp
constexpr int MAX_STAGES = 10;
constexpr int MAX_PREDS = 16;
constexpr int MAX_PROBES = 8;
constexpr int MAX_COMPUTES = 8;
constexpr int MAX_INSNS = 64;
constexpr int NREGS = HQ_MAX_COLS + HQ_MAX_TMP;
constexpr int SMEM_AGG_BYTES = 32 * 1024;
constexpr int64_t DENSE_LIMIT = 65536;
// shared-memory header of the fused kernels (mbarriers, block-scan and scalar-reduction
// slots, < 2,800 B) and, in its last 128 B, the per-warp words of the stage-release
// dependency (hq_jit.cu)
constexpr uint32_t MISC_BYTES = 3072;
constexpr uint32_t MISC_DEP = MISC_BYTES - 128;
constexpr int64_t DENSE_GLOBAL_LIMIT = 1LL << 28;  // dense global group tables (fused execution)
constexpr unsigned long long EMPTY_KEY = ~0ULL;

enum : uint8_t { OP_FILTER = 1, OP_PROBE = 2, OP_COMPUTE = 3 };
enum : uint8_t { GM_SCALAR = 0, GM_DENSE = 1, GM_HASH = 2 };   // global group table
// smem pre-aggregation table: none, shared dense (atomics), shared hash (atomics),
// lane-private dense accumulators (no atomics; tiny group domains, 8 warps)
enum : uint8_t { SM_NONE = 0, SM_DENSE = 1, SM_HASH = 2, SM_LANE = 3 };
constexpr int LANE_NW = 8;                 // consumer warps when SM_LANE
constexpr int SMEM_LANE_BYTES = 96 * 1024; // lane-private table budget

struct KReg {
  uint32_t off;      // byte offset of row 0 in the stage (column) or tmp region (temporary)
  uint8_t width;     // 1, 4, 8
  uint8_t in_stage;  // 1 = fact column staged by TMA, 2 = lazy fact column (global loads), 0 = temporary
  uint8_t pad[2];
};
struct KCol {
  const char* ptr;
  uint32_t width;
  uint32_t soff;     // byte offset inside a stage
  uint32_t lazy;     // 1 = not streamed: the rows still live at its first use read it from global memory
};
struct KPred {
  int16_t reg;
  uint8_t kind;      // 0 = range [lo, hi], 1 = bitmap
  uint8_t neg;       // result negated (NE)
  int32_t lo32, hi32;
  int64_t lo, hi;
  uint64_t bm[4];
};
struct KProbe {
  const uint32_t* slots;
  uint32_t mask;     // LINEAR: capacity - 1; DIRECT: key range (capacity)
  int32_t dmin;      // DIRECT: key of slot 0
  uint8_t log2cap;
  uint8_t words;     // 1, 2, 4
  uint8_t mode;      // hq_probe_mode
  uint8_t npay;
  uint8_t direct;    // 1 = direct-mapped (dense keys)
  uint8_t ckind;     // compact form available (hq_hash::ckind)
  int16_t key_reg;
  int16_t dst[HQ_MAX_PAYLOAD];
  const void* compact;
  int32_t pay_min;   // ckind 2/3: payload = byte (nibble) + pay_min; range of payload 0 (count pass)
  int32_t pay_max;
  uint32_t cbytes;
  uint32_t smem_off; // generated kernels: byte offset of the staged compact table (0 = not staged)
  uint64_t pay_set[4];  // payload-0 values present, bit (v & 255) (hq_hash_meta::pay_set)
  float pass_est;      // expected fraction of probing rows that pass (key density of the build side)
  float pass_src;      // the same over the build side's source rows (lazy-load decision)
  const uint32_t* pf;  // linear tables: key-range bitmap (NULL = none)
  int32_t pf_min;
  uint32_t pf_range;
  uint8_t composite;   // two-column key: slot word 1 must equal key2_reg; payloads from word 2
  int16_t key2_reg;
  uint8_t crank;       // ckind 2: the byte is the payload's RANK in pay_set (sparse value sets)
  // ranked form of a linear table (hq_hash::ranked): pf = its bitmap (rstride > 0: the
  // {bits, rank directory} word pairs), rpay = payload rows (rstride words) by rank
  uint8_t ranked, rstride;
  const int32_t* rpay;
};
struct KCompute {
  int16_t dst;
  uint8_t first;
  uint8_t n;
};
struct KInsn {
  uint8_t opc;
  uint8_t pad;
  int16_t reg;       // < 0: immediate
  int32_t pad2;
  int64_t imm;
};
struct KOp {
  uint8_t kind;
  uint8_t idx;
};

struct KPlan {
  int64_t row_begin, row_end;
  int32_t nw;                // consumer warps (blockDim = (nw + 1) * 32)
  int32_t R, tile_rows, nstages;
  uint32_t stage_bytes;      // bytes of one stage's columns (= tile_rows * row width)
  uint32_t stage_stride;     // stage spacing in smem (>= stage_bytes, 128-B multiple)
  uint32_t off_tmp, off_agg, off_stage;  // dynamic smem layout
  uint32_t off_tab, tab_bytes;           // staged compact probe tables (generated kernels)
  int32_t ncols;
  KCol cols[HQ_MAX_COLS];
  KReg regs[NREGS];
  int32_t nops;
  KOp ops[HQ_MAX_OPS];
  KPred preds[MAX_PREDS];
  KProbe probes[MAX_PROBES];
  KCompute comps[MAX_COMPUTES];
  KInsn insns[MAX_INSNS];
  // sink
  int32_t sink, resolution;
  int32_t nkeys;
  int16_t key_reg[HQ_MAX_KEYS];
  int64_t key_min[HQ_MAX_KEYS];
  int64_t key_card[HQ_MAX_KEYS];
  int64_t key_stride[HQ_MAX_KEYS];
  int32_t naggs;
  uint8_t agg_fn[HQ_MAX_AGGS];
  int16_t agg_reg[HQ_MAX_AGGS];
  uint8_t gmode, smode;
  uint32_t vwords;           // 1 + naggs: [count, agg...] per group
  // generated kernels' shared pre-aggregation entries: [count, non-COUNT aggs...]
  // (COUNT aggregates read the count word); lcol[a] = the aggregate's word
  uint32_t lvwords;
  uint8_t lcol[HQ_MAX_AGGS];
  long long* gtab;           // global dense table or hash entries [key, count, agg...]
  uint64_t gmask;            // hash capacity - 1
  int32_t glog2;
  uint32_t smem_cap;         // smem dense groups or smem hash slots
  uint32_t scopies;          // generated kernels, SM_DENSE: table replicas (warp w updates copy w % scopies)
  // generated kernels: the shared dense table may index a narrowed key domain
  // (group keys that are probe payloads span only their build-side value range)
  uint8_t local_keys;
  // generated kernels: copy the tile's columns into registers and release the
  // stage before the operators run (long-latency probes do not hold the ring)
  uint8_t early_release;
  // generated A3 variants: 1 = deferred write-out, a tile's rows are staged in shared
  // memory (two buffers of a3_buf bytes at off_agg, column j at a3_col[j]) and written to
  // global memory during the next tile, when its atomicAdd has returned (opt-in);
  // 2 = warp workgroups: each consumer warp collects its rows in its own shared buffer
  // (a3_rows rows, a3_buf bytes per warp at off_agg + warp * a3_buf, column j at a3_col[j])
  // and claims global positions for a full buffer with one atomicAdd -- no block barrier
  // per tile (behind a global probe)
  uint8_t a3stage;
  uint32_t a3_buf;
  uint32_t a3_rows;
  uint32_t a3_col[HQ_MAX_OUT];
  // multi-pass execution (HQ_EXEC_MULTIPASS, hq_multipass.cu): 1 = count kernel
  // (relational primitives -> one flag per row), 2 = write kernel (rows whose
  // flag is set; projections / aggregation inputs written at the prefix-sum
  // positions); op_skip marks the ops a pass does not execute
  uint8_t mp_pass;
  uint8_t op_skip[HQ_MAX_OPS];
  int16_t mp_flag_reg, mp_pos_reg;  // pass 2: stage registers of the flag and position columns
  int64_t lkey_min[HQ_MAX_KEYS];
  int64_t lkey_stride[HQ_MAX_KEYS];
  // ... and a key whose payload takes few distinct values (SSB Q3.1: 5 ASIA
  // nations spread over codes 4..24) is indexed by its rank in this set of
  // values (bit v - lkey_min); all-zero = plain offset v - lkey_min
  uint64_t lkey_set[HQ_MAX_KEYS][4];
  int32_t slog2;
  // SM_LANE: deduplicated accumulators (0 = count; SUM and AVG of one register share)
  int32_t nacc;
  uint8_t acc_fn[HQ_MAX_AGGS + 1];
  int16_t acc_reg[HQ_MAX_AGGS + 1];
  uint8_t acc_of[HQ_MAX_AGGS];  // aggregate -> accumulator
  // materialise
  int32_t nout;
  int16_t out_reg[HQ_MAX_OUT];
  uint8_t out_width[HQ_MAX_OUT];
  void* out_ptr[HQ_MAX_OUT];
  int64_t capacity;
  // status
  unsigned long long* counter;  // qualifying rows / write counter
  int* err;
  // generated kernels, global hash group table without a shared table: each consumer warp
  // queues its live rows' group updates in shared memory (gq_cap entries at
  // off_agg + warp * gq_cap * (2 + naggs) * 8, column-major: keys, counts, values) and
  // applies a full queue with one update per lane -- the hash round trips of up to
  // gq_cap rows overlap instead of stalling every tile that has a live row (0 = off)
  uint16_t gq_cap;
};
}  // namespace hqk

struct hq_result : RefObj {
  CtxPtr ctx;
  hq_plan plan{};
  hq_table* fact = nullptr;
  std::vector<hq_hash*> hashes;
  int sink = 0;
  uint8_t gmode = 0;
  int64_t ngroups = 0;        // dense groups or hash capacity
  uint32_t vwords = 0;
  DevBuf gtab;                // group table
  DevBuf dstate;              // [0..1] counter (u64), [2] fault bits (int), [3] spare
  // materialise
  std::vector<DevBuf> outcols;
  int64_t capacity = 0;
  int32_t segment_rows = 0;   // tile rows of the launch that wrote it
  // finalized AGG rows
  bool finalized = false;
  bool checked = false;
  int64_t checked_counter = -1;  // the output counter read by the fault check (materialise: row count)
  int64_t nrows = 0;
  int64_t qualifying = 0;
  int ncols = 0;
  int types[HQ_MAX_KEYS + HQ_MAX_AGGS] = {0};
  std::vector<DevBuf> rescols;  // finalized result columns (int64 / f64) ...
  DevBuf respack;                // ... or packed in one buffer (small results)
  std::vector<void*> rescol;     // device pointer of each finalized column
  // multi-pass execution: per-row flags and prefix-sum positions (int32), the
  // materialised aggregation inputs (pass 2) and the library-reduction scratch
  DevBuf mp_flags, mp_pos, mp_keys, mp_vals, mp_scratch;
  const char* mp_flags_col = nullptr;  // flags / positions indexed by absolute row
  const char* mp_pos_col = nullptr;
  int64_t stream_block = 0;  // > 0: batch processing of a host-resident fact table, rows per block
  DevBuf ring;               // its double-buffered device blocks
  std::vector<long long> host_rows;  // small results: the finalized rows already on the host
  bool host_ready = false;           // (column-major, nrows per column)
  // finalized inside a graph capture: rows + stats land in stage_host at every launch
  void* stage_host = nullptr;        // pinned (cudaHostAlloc), owned
  int64_t stage_rcap = 0;
  bool stage_topk = false;           // staged by the top-k finalize (stats word 5: too many ties)
  ~hq_result() override;
};

// ---------------------------------------------------------------- launchers
namespace hqk {
void launch_fused(hq_ctx* ctx, const KPlan& kp, int grid, size_t smem);
void launch_init_groups(hq_ctx* ctx, long long* tab, int64_t ngroups, uint32_t vwords, bool hash,
                        const uint8_t* agg_fn, int naggs);
int64_t fused_smem_bytes(const KPlan& kp);
}  // namespace hqk

// finalize: compaction + AVG + ORDER BY + LIMIT (hq_finalize.cu)
void hq_column_range_impl(hq_ctx* ctx, const hq_table* t, int col, int64_t* mn, int64_t* mx);
void* pinned_staging(hq_ctx* ctx, size_t bytes);
// hq_finalize.cu: OR of fault words into HQ_FAULT_WORDS int64 (hq_gather_faults)
void hq_launch_gather_faults(hq_ctx* ctx, const std::vector<const int*>& hw, const std::vector<const int*>& rw,
                             long long* out);  // hq_finalize.cu: per-context pinned host buffer
// unordered: a pure GROUP BY (no ORDER BY / LIMIT) skips the sort (hq_result_as_table)
void hq_finalize_impl(hq_ctx* ctx, hq_result* r, bool unordered = false);
// op-at-a-time execution of a plan (hq_oaat.cu)
void hq_run_oaat(hq_ctx* ctx, const hq_plan* plan, hq_result* r);
// shared plan preparation (hq_plan.cu)
void hq_prepare_result(hq_ctx* ctx, const hq_plan* plan, hq_result* r);
void hq_build_kplan(hq_ctx* ctx, hq_result* r, hqk::KPlan& kp, int64_t group_cap, int64_t mat_cap,
                    bool jit = false, int mp_pass = 0);
// multi-pass execution of a plan (hq_multipass.cu): count kernel, prefix sum,
// write kernel, library reductions (§4, Fig 7-9; A1/B1/C1 of Table 4)
void hq_run_multipass(hq_ctx* ctx, const hq_plan* plan, hq_result* r, int64_t group_cap = 0);
// query compilation (hq_jit.cu): NVRTC-specialised fused kernels
bool hq_jit_enabled();
void hq_jit_prepare(hq_ctx* ctx, const hqk::KPlan& kp, size_t smem);  // compile (cached) + attributes
void hq_jit_launch(hq_ctx* ctx, const hqk::KPlan& kp, int grid, size_t smem);
std::string hq_jit_source(const hqk::KPlan& kp);
void hq_check_result_faults(hq_ctx* ctx, hq_result* r);
// host synchronisation of the context stream; illegal while a graph is captured
void hq_sync(hq_ctx* ctx, const char* what);
void hq_require_eager(hq_ctx* ctx, const char* what);  // throws HQ_ERR_STATE while capturing
// decode a result finalized during a capture from its pinned staging (after a launch)
void hq_decode_captured(hq_ctx* ctx, hq_result* r);
void hq_hash_check(hq_ctx* ctx, hq_hash* h);  // hq_build.cu: sync + raise build faults
int hq_type_width(int type);
