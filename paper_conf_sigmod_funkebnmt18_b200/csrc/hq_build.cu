// hq_build.cu -- hash-join build, the pipeline breaker of a join (PAPER.md
// P:186-195 "build hash table", P:1033-1036 inserts isolated with atomics,
// P:1719-1720 dimension hash tables in GPU global memory).
//
// Open addressing with linear probing in a power-of-two slot array; a slot is
// {int32 key, int32 payload[0..3]} of 1, 2 or 4 words (16-B slots load as one
// int4 sector-aligned vector in the probe); the empty key is INT32_MIN.  A key
// is claimed with ONE atomicCAS on the key word; payload words are then written
// by the claiming thread (readers only run in later kernels, stream-ordered).
// Capacity: next_pow2(ceil(keys / 0.6)) >= 16, keys counted exactly by a
// predicate-only count pass unless the caller supplies expected_rows.
#include <cub/block/block_reduce.cuh>
#include <cub/block/block_scan.cuh>

#include <climits>

#include "hq_internal.h"

namespace {

struct KBuildPred {
  int16_t col;
  uint8_t kind, neg;
  int64_t lo, hi;
  uint64_t bm[4];
};
struct KBuild {
  int64_t n;
  const char* col[HQ_MAX_COLS];
  int32_t colw[HQ_MAX_COLS];
  int32_t npreds;
  KBuildPred preds[HQ_MAX_PREDS];
  int32_t key_col, npay;
  int32_t pay_col[HQ_MAX_PAYLOAD];
  uint32_t* slots;
  uint32_t mask;     // LINEAR: capacity - 1; DIRECT: key range
  int32_t log2cap, words;
  int32_t direct, dmin;
  int* err;
  unsigned long long* nkeys;
  int* kminmax;      // count pass: [min, max] of the qualifying keys, [min, max] of payload 0
  unsigned* pset;    // count pass: payload-0 values present, bit (v & 255) (8 words)
  void* part;        // count pass: per-block partials (CountPart[grid])
  unsigned* ticket;  // count pass: blocks done
  int count_inserts; // build pass: accumulate the inserted-key count (no count pass ran)
  int composite;     // two-column key: equal key_col values take separate slots (no dup check)
  // cached statistics (no count pass ran): the insert pass checks that the qualifying
  // rows match them -- keys in [kmin, kmax], payload 0 in [pmin, pmax] and in set, as
  // many rows -- and flags HQF_STALE otherwise
  int verify;
  BuildStats vs;
  unsigned long long* vqual;  // qualifying rows seen by the insert pass
  // a source table sized by a cached row count (hq_table::dev_rows): the real count
  // on the device; rows at or past it do not qualify, and a difference is HQF_STALE
  const unsigned long long* ndev;
};

__device__ __forceinline__ long long live_rows(const KBuild& b) {
  if (!b.ndev) return b.n;
  // (written by an earlier kernel: the read-only path, so that an SM's warps share one
  // L2 request -- a volatile load from every warp made one hot L2 line)
  const long long d = (long long)__ldg(b.ndev);
  if (d != b.n && blockIdx.x == 0 && threadIdx.x == 0) atomicOr(b.err, HQF_STALE);
  return d < b.n ? d : b.n;
}

__device__ __forceinline__ long long ld_col(const KBuild& b, int c, long long row) {
  const int w = b.colw[c];
  if (w == 4) return ((const int*)b.col[c])[row];
  if (w == 8) return ((const long long*)b.col[c])[row];
  return ((const signed char*)b.col[c])[row];
}
__device__ __forceinline__ bool row_passes(const KBuild& b, long long row) {
  for (int i = 0; i < b.npreds; ++i) {
    const KBuildPred& f = b.preds[i];
    const long long v = ld_col(b, f.col, row);
    bool ok;
    if (f.kind == 0) ok = (v >= f.lo && v <= f.hi) != (bool)f.neg;
    else ok = (unsigned long long)v < 256 && ((f.bm[v >> 6] >> (v & 63)) & 1ull);
    if (!ok) return false;
  }
  return true;
}

// Both passes give every thread U rows (stride blockDim) with all column loads
// issued before any is used, and no grid-stride loop: a dimension table's rows
// are all in flight at once (a grid-stride loop made each thread walk ~10 rows
// through 2-3 dependent DRAM round trips each).
#ifndef HQ_BUILD_U
#define HQ_BUILD_U 4
#endif
constexpr int BUILD_U = HQ_BUILD_U;  // (-DHQ_BUILD_U=..: A/B builds of the library)
constexpr int BUILD_BLOCK = 256;
// the count and compact-build kernels are latency-bound: at 72 registers only 3 blocks
// fit an SM; capped at 64 (4 blocks, a few spilled bytes) the SSB Q4.1 SF100 customer
// build takes 31.8 instead of 38 us, TPC-H Q3's customer / orders builds 37 / 41 instead
// of 45 / 46 us (measured)
#ifndef HQ_BUILD_MINB
#define HQ_BUILD_MINB 8
#endif
constexpr int BUILD_MINB = HQ_BUILD_MINB;
// (round 2: 4 rows per thread at 8 blocks per SM beat 8 rows at 4 -- more warps, fewer waves'
// worth of latency per thread: SSB Q4.1 SF100 customer / part builds 26.3 / 17.0 -> 23.2 /
// 14.6 us, TPC-H Q3 SF30 customer / orders bitmap / ranked scatter 30.3 / 32.1 / 33.0 ->
// 27.0 / 26.0 / 29.9 us; 16 rows at 4 blocks spilled 820 bytes, measured)
static_assert(BUILD_U <= 10, "the compact build packs a 3-bit slot shift per row into 32 bits");

// column c for the thread's U rows: the width dispatch is uniform, the U loads
// are independent (all in flight)
__device__ __forceinline__ void ld_rows(const KBuild& b, int c, long long base, long long (&out)[BUILD_U]) {
  const int w = b.colw[c];
  const char* p = b.col[c];
  if (w == 4) {
#pragma unroll
    for (int u = 0; u < BUILD_U; ++u) {
      const long long r = base + (long long)u * BUILD_BLOCK;
      out[u] = r < b.n ? __ldg((const int*)p + r) : 0;
    }
  } else if (w == 8) {
#pragma unroll
    for (int u = 0; u < BUILD_U; ++u) {
      const long long r = base + (long long)u * BUILD_BLOCK;
      out[u] = r < b.n ? __ldg((const long long*)p + r) : 0;
    }
  } else {
#pragma unroll
    for (int u = 0; u < BUILD_U; ++u) {
      const long long r = base + (long long)u * BUILD_BLOCK;
      out[u] = r < b.n ? (long long)__ldg((const signed char*)p + r) : 0;
    }
  }
}
// predicates, key and payload 0 of the thread's U rows
__device__ __forceinline__ void load_rows(const KBuild& b, long long base, bool (&pass)[BUILD_U],
                                          long long (&kv)[BUILD_U], long long (&pv)[BUILD_U]) {
  ld_rows(b, b.key_col, base, kv);
  if (b.npay > 0) ld_rows(b, b.pay_col[0], base, pv);
  const long long nl = live_rows(b);
#pragma unroll
  for (int u = 0; u < BUILD_U; ++u) pass[u] = base + (long long)u * BUILD_BLOCK < nl;
  for (int i = 0; i < b.npreds; ++i) {
    const KBuildPred& f = b.preds[i];
    long long v[BUILD_U];
    ld_rows(b, f.col, base, v);
    if (f.kind == 0) {
#pragma unroll
      for (int u = 0; u < BUILD_U; ++u) pass[u] &= (v[u] >= f.lo && v[u] <= f.hi) != (bool)f.neg;
    } else {
#pragma unroll
      for (int u = 0; u < BUILD_U; ++u)
        pass[u] &= (unsigned long long)v[u] < 256 && ((f.bm[(v[u] >> 6) & 3] >> (v[u] & 63)) & 1ull);
    }
  }
}

// count pass: number of qualifying rows, min/max of their keys and of payload 0.
// Block partials go to b.part; the last block to finish (ticket) reduces them
// and writes the totals -- no contended global atomics.
struct CountPart {
  unsigned long long cnt;
  int kmin, kmax, pmin, pmax;
  unsigned set[8];  // payload-0 values present, bit (v & 255)
};
__global__ void __launch_bounds__(BUILD_BLOCK, BUILD_MINB) hq_build_count_kernel(const __grid_constant__ KBuild b) {
  unsigned long long c = 0;
  int kmin = INT_MAX, kmax = INT_MIN, pmin = INT_MAX, pmax = INT_MIN;
  unsigned pset[8] = {0u, 0u, 0u, 0u, 0u, 0u, 0u, 0u};  // registers: constant indices only
  const long long base = (long long)blockIdx.x * BUILD_BLOCK * BUILD_U + threadIdx.x;
  bool pass[BUILD_U];
  long long kv[BUILD_U], pv[BUILD_U] = {};
  load_rows(b, base, pass, kv, pv);
#pragma unroll
  for (int u = 0; u < BUILD_U; ++u) {
    if (!pass[u]) continue;
    ++c;
    if (kv[u] > (long long)INT_MIN && kv[u] <= (long long)INT_MAX) {
      kmin = min(kmin, (int)kv[u]);
      kmax = max(kmax, (int)kv[u]);
    }
    if (b.npay > 0) {
      const int pc = pv[u] < (long long)INT_MIN ? INT_MIN : (pv[u] > (long long)INT_MAX ? INT_MAX : (int)pv[u]);
      pmin = min(pmin, pc);
      pmax = max(pmax, pc);
      const int pw = (pc & 255) >> 5;
#pragma unroll
      for (int w8 = 0; w8 < 8; ++w8) pset[w8] |= pw == w8 ? 1u << (pc & 31) : 0u;
    }
  }
  kmin = __reduce_min_sync(0xffffffffu, kmin);
  kmax = __reduce_max_sync(0xffffffffu, kmax);
  pmin = __reduce_min_sync(0xffffffffu, pmin);
  pmax = __reduce_max_sync(0xffffffffu, pmax);
#pragma unroll
  for (int w8 = 0; w8 < 8; ++w8) pset[w8] = __reduce_or_sync(0xffffffffu, pset[w8]);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
  __shared__ CountPart wp[BUILD_BLOCK / 32];
  __shared__ bool last;
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (lane == 0) wp[w] = {c, kmin, kmax, pmin, pmax, {pset[0], pset[1], pset[2], pset[3], pset[4], pset[5], pset[6], pset[7]}};
  __syncthreads();
  if (threadIdx.x == 0) {
    CountPart t{0, INT_MAX, INT_MIN, INT_MAX, INT_MIN, {}};
    for (int k = 0; k < BUILD_BLOCK / 32; ++k) {
      t.cnt += wp[k].cnt;
      t.kmin = min(t.kmin, wp[k].kmin); t.kmax = max(t.kmax, wp[k].kmax);
      t.pmin = min(t.pmin, wp[k].pmin); t.pmax = max(t.pmax, wp[k].pmax);
    }
    for (int k = 0; k < BUILD_BLOCK / 32; ++k)
      for (int w8 = 0; w8 < 8; ++w8) t.set[w8] |= wp[k].set[w8];
    ((CountPart*)b.part)[blockIdx.x] = t;
    __threadfence();
    last = atomicAdd(b.ticket, 1u) == gridDim.x - 1;
  }
  __syncthreads();
  if (!last) return;
  // last block: reduce every block's partial
  __threadfence();
  CountPart t{0, INT_MAX, INT_MIN, INT_MAX, INT_MIN, {}};
  for (unsigned k = threadIdx.x; k < gridDim.x; k += BUILD_BLOCK) {
    const volatile CountPart* q = (const volatile CountPart*)b.part + k;
    t.cnt += q->cnt;
    t.kmin = min(t.kmin, q->kmin); t.kmax = max(t.kmax, q->kmax);
    t.pmin = min(t.pmin, q->pmin); t.pmax = max(t.pmax, q->pmax);
#pragma unroll
    for (int w8 = 0; w8 < 8; ++w8) t.set[w8] |= q->set[w8];
  }
#pragma unroll
  for (int w8 = 0; w8 < 8; ++w8) t.set[w8] = __reduce_or_sync(0xffffffffu, t.set[w8]);
  t.kmin = __reduce_min_sync(0xffffffffu, t.kmin);
  t.kmax = __reduce_max_sync(0xffffffffu, t.kmax);
  t.pmin = __reduce_min_sync(0xffffffffu, t.pmin);
  t.pmax = __reduce_max_sync(0xffffffffu, t.pmax);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) t.cnt += __shfl_xor_sync(0xffffffffu, t.cnt, o);
  __syncthreads();
  if (lane == 0) wp[w] = t;
  __syncthreads();
  if (threadIdx.x == 0) {
    CountPart z{0, INT_MAX, INT_MIN, INT_MAX, INT_MIN, {}};
    for (int k = 0; k < BUILD_BLOCK / 32; ++k) {
      z.cnt += wp[k].cnt;
      z.kmin = min(z.kmin, wp[k].kmin); z.kmax = max(z.kmax, wp[k].kmax);
      z.pmin = min(z.pmin, wp[k].pmin); z.pmax = max(z.pmax, wp[k].pmax);
      for (int w8 = 0; w8 < 8; ++w8) z.set[w8] |= wp[k].set[w8];
    }
    *b.nkeys = z.cnt;
    b.kminmax[0] = z.kmin; b.kminmax[1] = z.kmax; b.kminmax[2] = z.pmin; b.kminmax[3] = z.pmax;
    for (int w8 = 0; w8 < 8; ++w8) b.pset[w8] = z.set[w8];
  }
}

// A direct table whose only consumers read its compact form (generated kernels) is
// built straight into that form: one pass over the dimension rows, one atomic per
// qualifying row on the (memset) bitmap / byte map / nibble map, which also detects a
// duplicate key (the atomic returns the previous bits) -- no slot array, no fill, no
// separate compaction.  kind: 1 bitmap, 2 byte (payload - pay_min, or its rank through
// lut), 3 nibble.  The slot array is derived later only if a consumer needs it.
struct CLut {
  unsigned char r[256];
};
__global__ void __launch_bounds__(BUILD_BLOCK, BUILD_MINB) hq_build_direct_compact_kernel(const __grid_constant__ KBuild b, int kind,
                                                                             uint32_t* out, long long range, int pay_min,
                                                                             int use_lut, const __grid_constant__ CLut lut) {
  int fault = 0;
  unsigned long long qual = 0;
  const long long base = (long long)blockIdx.x * BUILD_BLOCK * BUILD_U + threadIdx.x;
  bool pass[BUILD_U];
  long long kv[BUILD_U], pv[BUILD_U] = {};
  load_rows(b, base, pass, kv, pv);
  int aw[BUILD_U];  // target word of the row's atomic (< 2^30: range <= 2^32 keys), -1: none
  uint32_t am[BUILD_U], ash = 0;  // ash: the slot's shift / 4, 3 bits per row
#pragma unroll
  for (int u = 0; u < BUILD_U; ++u) { aw[u] = -1; am[u] = 0; }
#pragma unroll
  for (int u = 0; u < BUILD_U; ++u) {
    if (!pass[u]) continue;
    int pc = 0;
    if (b.npay > 0) {
      pc = pv[u] < (long long)INT_MIN ? INT_MIN : (pv[u] > (long long)INT_MAX ? INT_MAX : (int)pv[u]);
      if (pv[u] < (long long)INT_MIN || pv[u] > (long long)INT_MAX) fault |= HQF_BAD_PAYLOAD;
    }
    if (b.verify) {
      ++qual;
      if (kv[u] > (long long)INT_MIN && kv[u] <= (long long)INT_MAX && (kv[u] < b.vs.kmin || kv[u] > b.vs.kmax))
        fault |= HQF_STALE;
      if (b.npay > 0 && (pc < b.vs.pmin || pc > b.vs.pmax || !((b.vs.set[(pc & 255) >> 5] >> (pc & 31)) & 1u)))
        fault |= HQF_STALE;
    }
    if (kv[u] <= (long long)INT_MIN || kv[u] > (long long)INT_MAX) {
      fault |= HQF_BAD_KEY;
      continue;
    }
    const long long d = kv[u] - (long long)b.dmin;
    if (d < 0 || d >= range) {  // cannot happen with exact or verified statistics
      fault |= HQF_HT_FULL;
      continue;
    }
    // word index and bits of the row; the atomics are issued in a separate loop
    if (kind == 1) {
      aw[u] = (int)(d >> 5);
      am[u] = 1u << (d & 31);
    } else if (kind == 2) {
      uint32_t v = (uint32_t)(pc - pay_min) & 0xFFu;
      if (use_lut) v = lut.r[v];
      const uint32_t sh = (uint32_t)(d & 3) * 8u;
      aw[u] = (int)(d >> 2);
      am[u] = ~((0xFFu ^ v) << sh);
      ash |= (sh >> 2) << (3 * u);
    } else {
      const uint32_t v = (uint32_t)(pc - pay_min) & 0xFu;
      const uint32_t sh = (uint32_t)(d & 7) * 4u;
      aw[u] = (int)(d >> 3);
      am[u] = ~((0xFu ^ v) << sh);
      ash |= (sh >> 2) << (3 * u);
    }
  }
  // all of the thread's atomics in flight at once: a duplicate-key test right after each
  // one made every atomic a dependent L2 round trip (the test branches on its result)
  uint32_t old[BUILD_U];
#pragma unroll
  for (int u = 0; u < BUILD_U; ++u)
    if (aw[u] >= 0) old[u] = kind == 1 ? atomicOr(out + aw[u], am[u]) : atomicAnd(out + aw[u], am[u]);
#pragma unroll
  for (int u = 0; u < BUILD_U; ++u) {
    if (aw[u] < 0) continue;
    const uint32_t sh = ((ash >> (3 * u)) & 7u) * 4u, full = kind == 2 ? 0xFFu : 0xFu;
    const uint32_t f = kind == 1 ? (old[u] & am[u]) : ((old[u] >> sh) & full) ^ full;
    if (f) fault |= HQF_DUP_KEY;
  }
  if (fault) atomicOr(b.err, fault);
  if (b.verify) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) qual += __shfl_xor_sync(0xffffffffu, qual, o);
    __shared__ unsigned long long vred[BUILD_BLOCK / 32];
    if ((threadIdx.x & 31) == 0) vred[threadIdx.x >> 5] = qual;
    __syncthreads();
    if (threadIdx.x == 0) {
      unsigned long long t = 0;
      for (int k = 0; k < BUILD_BLOCK / 32; ++k) t += vred[k];
      // the block's count and its ticket in ONE 64-bit atomic (count: low 40 bits, blocks
      // done: high 24): the last block reads the total from the returned word -- no fences
      // (two atomics ordered by __threadfence held every block's exit for microseconds)
      const unsigned long long old = atomicAdd(b.vqual, (1ull << 40) | t);
      if ((old >> 40) == gridDim.x - 1 && (old & ((1ull << 40) - 1)) + t != b.vs.cnt) atomicOr(b.err, HQF_STALE);
    }
  }
}

// the slot array of a compact-only direct table, derived from its compact form (for the
// consumers that read slots: interpreter, operator-at-a-time, hq_hash_device_view)
__global__ void hq_slots_from_compact_kernel(const uint32_t* c, int kind, long long range, int key_min, int pay_min,
                                             int use_rv, const __grid_constant__ CLut rv_lo, const __grid_constant__ CLut rv_hi,
                                             uint32_t* slots) {
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < range; i += (long long)gridDim.x * blockDim.x) {
    if (kind == 1) {
      slots[i] = ((c[i >> 5] >> (i & 31)) & 1u) ? (uint32_t)(key_min + (int)i) : 0x80000000u;
      continue;
    }
    const uint32_t v = kind == 2 ? (c[i >> 2] >> ((i & 3) * 8)) & 0xFFu : (c[i >> 3] >> ((i & 7) * 4)) & 0xFu;
    const bool present = kind == 2 ? v != 0xFFu : v != 0xFu;
    // rank -> offset from pay_min (two byte tables: offsets up to 65535 are not needed, < 256)
    const int off = use_rv ? (int)rv_lo.r[v] | ((int)rv_hi.r[v] << 8) : (int)v;
    slots[2 * i] = present ? (uint32_t)(key_min + (int)i) : 0x80000000u;
    slots[2 * i + 1] = present ? (uint32_t)(pay_min + off) : 0u;
  }
}

__global__ void hq_fill_kernel(uint32_t* p, long long n, uint32_t v) {
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
    p[i] = v;
}

// ---- ranked form of a sparse-key table (hq_hash::ranked): the bitmap of
// present keys over the key range (built by hq_build_direct_compact_kernel, kind 1), a
// rank directory (keys before each bitmap word: an exclusive scan of the words' popcounts)
// and the payload rows stored densely by rank.  A table with payloads interleaves bitmap
// and directory as {bits, dir} word pairs (ws = 2): a probe's one 8-B load gives both, so a
// hit costs two dependent L2 loads (pair, payload row), not three.  It replaces a linear
// table's slot array, its fill and its key-range prefilter: no CAS, no probe sequence.
constexpr int RSCAN_T = 1024, RSCAN_W = 8;  // directory scan: 8 bitmap words per thread
// the thread's 8 bitmap words (16-B loads; ws = 2: the .x of 8 {bits, dir} pairs)
__device__ __forceinline__ void rank_words(const uint32_t* bm, int ws, long long base, uint32_t (&c)[RSCAN_W]) {
  if (ws == 1) {
    const uint4 a = __ldg((const uint4*)(bm + base)), b = __ldg((const uint4*)(bm + base) + 1);
    c[0] = a.x; c[1] = a.y; c[2] = a.z; c[3] = a.w; c[4] = b.x; c[5] = b.y; c[6] = b.z; c[7] = b.w;
    return;
  }
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    const uint4 a = __ldg((const uint4*)(bm + 2 * base) + q);
    c[2 * q] = a.x;
    c[2 * q + 1] = a.z;
  }
}
// per block (8,192 words): number of present keys
__global__ void __launch_bounds__(RSCAN_T) hq_rank_blocksum_kernel(const uint32_t* bm, int ws, unsigned* bsum) {
  uint32_t c[RSCAN_W];
  rank_words(bm, ws, ((long long)blockIdx.x * RSCAN_T + threadIdx.x) * RSCAN_W, c);
  unsigned n = 0;
#pragma unroll
  for (int j = 0; j < RSCAN_W; ++j) n += __popc(c[j]);
  typedef cub::BlockReduce<unsigned, RSCAN_T> BR;
  __shared__ typename BR::TempStorage tmp;
  const unsigned t = BR(tmp).Sum(n);
  if (threadIdx.x == 0) bsum[blockIdx.x] = t;
}
// exclusive scan of the block sums (one block, chunks of 1,024 with a carry)
__global__ void __launch_bounds__(RSCAN_T) hq_rank_topscan_kernel(unsigned* bsum, int n) {
  typedef cub::BlockScan<unsigned, RSCAN_T> BS;
  __shared__ typename BS::TempStorage tmp;
  unsigned carry = 0;
  for (int b = 0; b < n; b += RSCAN_T) {
    const int i = b + (int)threadIdx.x;
    unsigned v = i < n ? bsum[i] : 0u, ex, tot;
    BS(tmp).ExclusiveSum(v, ex, tot);
    if (i < n) bsum[i] = carry + ex;
    carry += tot;
    __syncthreads();  // tmp reuse
  }
}
// directory: keys before each word = block offset + block-exclusive scan + running sum,
// written with the bitmap words as the {bits, dir} pairs
__global__ void __launch_bounds__(RSCAN_T) hq_rank_dir_kernel(const uint32_t* bm, const unsigned* bsum, uint32_t* bd) {
  const long long base = ((long long)blockIdx.x * RSCAN_T + threadIdx.x) * RSCAN_W;
  uint32_t c[RSCAN_W];
  rank_words(bm, 1, base, c);
  unsigned n = 0;
#pragma unroll
  for (int j = 0; j < RSCAN_W; ++j) n += __popc(c[j]);
  typedef cub::BlockScan<unsigned, RSCAN_T> BS;
  __shared__ typename BS::TempStorage tmp;
  unsigned ex;
  BS(tmp).ExclusiveSum(n, ex);
  unsigned run = bsum[blockIdx.x] + ex;
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    const unsigned d0 = run;
    run += __popc(c[2 * q]);
    const unsigned d1 = run;
    run += __popc(c[2 * q + 1]);
    ((uint4*)(bd + 2 * base))[q] = make_uint4(c[2 * q], d0, c[2 * q + 1], d1);
  }
}
// the directory in ONE pass (replaces blocksum + topscan + dir: one bitmap read, two
// launches less): blocks take their tile in launch order from a ticket, publish the tile's
// key count, and warp 0 looks back over the 32 preceding status words at a time (decoupled
// look-back) until it meets an inclusive prefix.  status: 0 = not ready, flag 1 = the tile's
// count only, flag 2 = the inclusive prefix through the tile (value in the low 62 bits).
constexpr unsigned long long RS_AGG = 1ull << 62, RS_INC = 2ull << 62, RS_VAL = RS_AGG - 1;
__global__ void __launch_bounds__(RSCAN_T) hq_rank_dir1_kernel(const uint32_t* bm, unsigned long long* status,
                                                             unsigned* ticket, uint32_t* bd) {
  __shared__ unsigned s_blk;
  __shared__ unsigned long long s_excl;
  if (threadIdx.x == 0) s_blk = atomicAdd(ticket, 1u);
  __syncthreads();
  const unsigned blk = s_blk;
  const long long base = ((long long)blk * RSCAN_T + threadIdx.x) * RSCAN_W;
  uint32_t c[RSCAN_W];
  rank_words(bm, 1, base, c);
  unsigned n = 0;
#pragma unroll
  for (int j = 0; j < RSCAN_W; ++j) n += __popc(c[j]);
  typedef cub::BlockScan<unsigned, RSCAN_T> BS;
  __shared__ typename BS::TempStorage tmp;
  unsigned ex, tot;
  BS(tmp).ExclusiveSum(n, ex, tot);
  if (threadIdx.x < 32) {
    const int lane = threadIdx.x;
    unsigned long long excl = 0;
    if (blk == 0) {
      if (lane == 0) atomicExch(status, RS_INC | tot);
    } else {
      if (lane == 0) atomicExch(status + blk, RS_AGG | tot);
      long long j = (long long)blk - 1 - lane;  // this lane's predecessor in the window
      for (;;) {
        const unsigned long long v = j >= 0 ? *(volatile const unsigned long long*)(status + j) : RS_INC;
        if (__any_sync(0xffffffffu, v == 0)) continue;  // a predecessor not ready yet: re-read the window
        const unsigned inc = __ballot_sync(0xffffffffu, (v & ~RS_VAL) == RS_INC);
        const int stop = inc ? __ffs(inc) - 1 : 32;  // nearest inclusive prefix in the window
        unsigned long long part = lane <= stop ? (v & RS_VAL) : 0ull;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) part += __shfl_xor_sync(0xffffffffu, part, o);
        excl += part;
        if (inc) break;
        j -= 32;
      }
      if (lane == 0) atomicExch(status + blk, RS_INC | (excl + tot));
    }
    if (lane == 0) s_excl = excl;
  }
  __syncthreads();
  unsigned run = (unsigned)s_excl + ex;
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    const unsigned d0 = run;
    run += __popc(c[2 * q]);
    const unsigned d1 = run;
    run += __popc(c[2 * q + 1]);
    ((uint4*)(bd + 2 * base))[q] = make_uint4(c[2 * q], d0, c[2 * q + 1], d1);
  }
}
// payload rows by rank: each qualifying row finds its key's rank and writes its payloads
__global__ void __launch_bounds__(BUILD_BLOCK) hq_build_ranked_scatter_kernel(const __grid_constant__ KBuild b,
                                                                             const uint2* bd, int* rpay, int stride,
                                                                             long long range, unsigned long long nkeys) {
  int fault = 0;
  const long long base = (long long)blockIdx.x * BUILD_BLOCK * BUILD_U + threadIdx.x;
  bool pass[BUILD_U];
  long long kv[BUILD_U], pv0[BUILD_U] = {};
  int pay[BUILD_U][HQ_MAX_PAYLOAD] = {};
  load_rows(b, base, pass, kv, pv0);
#pragma unroll
  for (int k = 0; k < HQ_MAX_PAYLOAD; ++k) {
    if (k >= b.npay) break;
    long long v[BUILD_U];
    if (k == 0) {
#pragma unroll
      for (int u = 0; u < BUILD_U; ++u) v[u] = pv0[u];
    } else {
      ld_rows(b, b.pay_col[k], base, v);
    }
#pragma unroll
    for (int u = 0; u < BUILD_U; ++u) pay[u][k] = (int)v[u];
  }
  unsigned rk[BUILD_U];
  bool ok[BUILD_U];
#pragma unroll
  for (int u = 0; u < BUILD_U; ++u) {  // the pair loads of all U rows in flight together
    const long long d = kv[u] - (long long)b.dmin;
    ok[u] = pass[u] && kv[u] > (long long)INT_MIN && kv[u] <= (long long)INT_MAX && d >= 0 && d < range;
    rk[u] = 0;
    if (ok[u]) {
      const uint2 q = __ldg(bd + (d >> 5));
      const uint32_t bit = 1u << (d & 31);
      ok[u] = (q.x & bit) != 0;
      rk[u] = q.y + __popc(q.x & (bit - 1u));
    }
  }
#pragma unroll
  for (int u = 0; u < BUILD_U; ++u) {
    if (!ok[u]) continue;  // (bad keys and out-of-range keys were flagged by the bitmap pass)
    if (rk[u] >= nkeys) {  // more keys than the (cached) statistics said: flagged stale by the bitmap pass
      fault |= HQF_STALE;
      continue;
    }
    int* dst = rpay + (size_t)rk[u] * stride;
#pragma unroll
    for (int k = 0; k < HQ_MAX_PAYLOAD; ++k)
      if (k < b.npay) dst[k] = pay[u][k];
  }
  if (fault) atomicOr(b.err, fault);
}
// the linear slot array of a ranked table, for consumers that read slots (interpreter,
// operator-at-a-time): every present key claims a slot as in hq_build_hash_kernel
__global__ void hq_slots_from_ranked_kernel(const uint32_t* bm, const int* rpay, int stride, int npay, long long range,
                                            int kmin, uint32_t* slots, uint32_t mask, int log2cap, int words, int* err) {
  const int ws = stride ? 2 : 1;
  for (long long d = blockIdx.x * (long long)blockDim.x + threadIdx.x; d < range; d += (long long)gridDim.x * blockDim.x) {
    const uint32_t w = bm[(d >> 5) * ws], bit = 1u << (d & 31);
    if (!(w & bit)) continue;
    const int key = kmin + (int)d;
    const int* src = stride ? rpay + (size_t)(bm[(d >> 5) * 2 + 1] + __popc(w & (bit - 1u))) * stride : nullptr;
    uint32_t pos = ((uint32_t)key * 0x9E3779B1u) >> (32 - log2cap);
    for (uint32_t n = 0;; ++n) {
      if (n > mask) {
        atomicOr(err, HQF_HT_FULL);
        break;
      }
      uint32_t* slot = slots + (size_t)pos * words;
      if (atomicCAS((int*)slot, INT_MIN, key) == INT_MIN) {
        for (int k = 0; k < npay; ++k) slot[1 + k] = (uint32_t)src[k];
        break;
      }
      pos = (pos + 1) & mask;
    }
  }
}

__global__ void __launch_bounds__(BUILD_BLOCK) hq_build_hash_kernel(const __grid_constant__ KBuild b) {
  unsigned long long inserted = 0, qual = 0;
  int fault = 0;
  const uint32_t shift = 32u - b.log2cap;
  const long long base = (long long)blockIdx.x * BUILD_BLOCK * BUILD_U + threadIdx.x;
  bool pass[BUILD_U];
  long long kv[BUILD_U], pv0[BUILD_U] = {};
  int pay[BUILD_U][HQ_MAX_PAYLOAD] = {};
  load_rows(b, base, pass, kv, pv0);
#pragma unroll
  for (int k = 0; k < HQ_MAX_PAYLOAD; ++k) {
    if (k >= b.npay) break;
    long long v[BUILD_U];
    if (k == 0) {
#pragma unroll
      for (int u = 0; u < BUILD_U; ++u) v[u] = pv0[u];
    } else {
      ld_rows(b, b.pay_col[k], base, v);
    }
#pragma unroll
    for (int u = 0; u < BUILD_U; ++u) {
      if (pass[u] && (v[u] < (long long)INT_MIN || v[u] > (long long)INT_MAX)) fault |= HQF_BAD_PAYLOAD;
      pay[u][k] = (int)v[u];
    }
  }
  // The thread's rows claim their slots in rounds: every pending row issues its CAS at
  // its current slot before any result is inspected, so the U atomics of a thread are in
  // flight together (a row-after-row loop waited one memory round trip per row: TPC-H
  // Q3's orders table, 4.4 M keys into 16-B slots, took 0.45 ms); a row that lost its
  // slot to another key moves on to the next slot in the following round.
  const uint32_t lmask = b.direct ? 0xFFFFFFFFu : b.mask;
  uint32_t pos[BUILD_U];
  bool pend[BUILD_U];
#pragma unroll
  for (int u = 0; u < BUILD_U; ++u) {
    pend[u] = false;
    pos[u] = 0;
    if (!pass[u]) continue;
    if (b.verify) {  // the rows the count pass would have summarised
      ++qual;
      if (kv[u] > (long long)INT_MIN && kv[u] <= (long long)INT_MAX && (kv[u] < b.vs.kmin || kv[u] > b.vs.kmax))
        fault |= HQF_STALE;
      if (b.npay > 0) {
        const int pc = pv0[u] < (long long)INT_MIN ? INT_MIN : (pv0[u] > (long long)INT_MAX ? INT_MAX : (int)pv0[u]);
        if (pc < b.vs.pmin || pc > b.vs.pmax || !((b.vs.set[(pc & 255) >> 5] >> (pc & 31)) & 1u)) fault |= HQF_STALE;
      }
    }
    if (kv[u] <= (long long)INT_MIN || kv[u] > (long long)INT_MAX) {
      fault |= HQF_BAD_KEY;
      continue;
    }
    const int key = (int)kv[u];
    pos[u] = b.direct ? (uint32_t)(key - b.dmin) : ((uint32_t)key * 0x9E3779B1u) >> shift;
    if (b.direct && pos[u] >= b.mask) {  // cannot happen: the range comes from the count pass
      fault |= HQF_HT_FULL;
      continue;
    }
    pend[u] = true;
  }
  for (uint32_t round = 0;; ++round) {
    bool any = false;
#pragma unroll
    for (int u = 0; u < BUILD_U; ++u) any = any || pend[u];
    if (!any) break;
    if (round > b.mask || (b.direct && round > 0)) {  // every slot visited: full
      fault |= HQF_HT_FULL;
      break;
    }
    int old[BUILD_U];
#pragma unroll
    for (int u = 0; u < BUILD_U; ++u)
      old[u] = pend[u] ? atomicCAS((int*)(b.slots + (size_t)pos[u] * b.words), INT_MIN, (int)kv[u]) : 0;
#pragma unroll
    for (int u = 0; u < BUILD_U; ++u) {
      if (!pend[u]) continue;
      if (old[u] == INT_MIN) {
        uint32_t* slot = b.slots + (size_t)pos[u] * b.words;
#pragma unroll
        for (int k = 0; k < HQ_MAX_PAYLOAD; ++k)
          if (k < b.npay) slot[1 + k] = (uint32_t)pay[u][k];
        ++inserted;
        pend[u] = false;
      } else if (!b.composite && (old[u] == (int)kv[u] || b.direct)) {
        fault |= HQF_DUP_KEY;  // join keys must be unique (R6)
        pend[u] = false;
      } else {
        pos[u] = (pos[u] + 1) & lmask;
      }
    }
  }
  if (fault) atomicOr(b.err, fault);
  if (b.verify) {  // the number of qualifying rows must equal the cached count
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) qual += __shfl_xor_sync(0xffffffffu, qual, o);
    __shared__ unsigned long long vred[BUILD_BLOCK / 32];
    if ((threadIdx.x & 31) == 0) vred[threadIdx.x >> 5] = qual;
    __syncthreads();
    if (threadIdx.x == 0) {
      unsigned long long t = 0;
      for (int k = 0; k < BUILD_BLOCK / 32; ++k) t += vred[k];
      // the block's count and its ticket in ONE 64-bit atomic (count: low 40 bits, blocks
      // done: high 24): the last block reads the total from the returned word -- no fences
      // (two atomics ordered by __threadfence held every block's exit for microseconds)
      const unsigned long long old = atomicAdd(b.vqual, (1ull << 40) | t);
      if ((old >> 40) == gridDim.x - 1 && (old & ((1ull << 40) - 1)) + t != b.vs.cnt) atomicOr(b.err, HQF_STALE);
    }
  }
  if (!b.count_inserts) return;  // counted builds know their key count already
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) inserted += __shfl_xor_sync(0xffffffffu, inserted, o);
  __shared__ unsigned long long red[BUILD_BLOCK / 32];
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = inserted;
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long t = 0;
    for (int k = 0; k < BUILD_BLOCK / 32; ++k) t += red[k];
    if (t) atomicAdd(b.nkeys, t);
  }
}

int64_t next_pow2(int64_t x) {
  int64_t c = 1;
  while (c < x) c <<= 1;
  return c;
}

bool stats_cache_on() {
  const char* e = getenv("HQ_BUILD_STATS");
  return !(e && e[0] == '0');
}

}  // namespace

// compact form of a direct table: 1 = bitmap (no payload), 2 = byte per key (payload 0
// spans < 255 values), 3 = nibble per key (< 15 values), 0 = none
int hq_compact_kind(int npayload, int pay_min, int pay_max) {
  if (npayload == 0) return 1;
  if (npayload != 1 || pay_min > pay_max) return 0;
  const long long pr = (long long)pay_max - pay_min;
  return pr < 15 ? 3 : (pr < 255 ? 2 : 0);
}
long long hq_compact_words(int kind, long long range) {
  return kind == 1 ? (range + 31) / 32 : (kind == 3 ? (range + 7) / 8 : (range + 3) / 4);
}
// ranked form: [bitmap words | payload rows], or with payloads [{bits, dir} word pairs |
// payload rows]; the bitmap padded to whole 8,192-word scan blocks (the scan kernels read
// and write them without bounds checks; the padding is zero), the rows 256-B aligned.
// off_dir: byte offset of directory word 0 (word w's at off_dir + 8 w), 0 without payload.
void hq_ranked_layout(int64_t range, int64_t nkeys, int npay, int64_t* off_dir, int64_t* off_pay, int64_t* total,
                      int* stride) {
  const int64_t blk = 1024 * 8;
  const int64_t words = ((range + 31) / 32 + blk - 1) / blk * blk;
  const int st = npay == 0 ? 0 : (npay == 1 ? 1 : (npay == 2 ? 2 : 4));
  *stride = st;
  *off_dir = st ? 4 : 0;
  *off_pay = words * 4 * (st ? 2 : 1);
  *total = *off_pay + (int64_t)st * 4 * (nkeys > 0 ? nkeys : 0);
}
// rank LUT of a byte map over a sparse payload set (value - pay_min -> rank, 0xFF
// absent); returns 1 when the map is rank-coded (the set is known and sparse)
int hq_rank_lut(const hq_hash_meta& m, unsigned char* lut) {
  for (int i = 0; i < 256; ++i) lut[i] = 0xFF;
  int n = 0;
  const int span = m.pay_max - m.pay_min + 1;
  if (span < 1 || span > 255) return 0;
  for (int d = 0; d < span; ++d) {
    const uint32_t v = (uint32_t)(m.pay_min + d) & 255u;
    if ((m.pay_set[v >> 6] >> (v & 63)) & 1ull) lut[d] = (unsigned char)n++;
  }
  const int crank = (n > 0 && n < span && !getenv("HQ_NO_RANKMAP")) ? 1 : 0;
  if (!crank)
    for (int d = 0; d < span; ++d) lut[d] = (unsigned char)d;
  return crank;
}

namespace {
void to_kpred(const hq_pred& in, KBuildPred& out, int ncols) {
  if (in.reg < 0 || in.reg >= ncols) HQ_THROW(HQ_ERR_ARG, "build predicate column out of range");
  out.col = (int16_t)in.reg;
  out.kind = 0;
  out.neg = 0;
  std::memset(out.bm, 0, sizeof(out.bm));
  switch (in.cmp) {
    case HQ_EQ: out.lo = out.hi = in.lo; break;
    case HQ_NE: out.lo = out.hi = in.lo; out.neg = 1; break;
    case HQ_LT:
      if (in.lo == LLONG_MIN) { out.lo = 1; out.hi = 0; } else { out.lo = LLONG_MIN; out.hi = in.lo - 1; }
      break;
    case HQ_LE: out.lo = LLONG_MIN; out.hi = in.lo; break;
    case HQ_GT:
      if (in.lo == LLONG_MAX) { out.lo = 1; out.hi = 0; } else { out.lo = in.lo + 1; out.hi = LLONG_MAX; }
      break;
    case HQ_GE: out.lo = in.lo; out.hi = LLONG_MAX; break;
    case HQ_BETWEEN: out.lo = in.lo; out.hi = in.hi; break;
    case HQ_IN_BITMAP: out.kind = 1; std::memcpy(out.bm, in.bitmap, sizeof(out.bm)); break;
    default: HQ_THROW(HQ_ERR_ARG, "unknown comparison");
  }
}

}  // namespace

// Host side of hq_build_hash / hq_build_hashes (called from hq_api.cu).  The
// builds of one call share ONE host synchronisation: every table's count pass
// is launched first, their statistics come back together, then the slot arrays
// are sized, filled, built and compacted (all stream-ordered, no further sync).
namespace {
struct BuildState {
  KBuild b{};
  int grid = 0;
  int words = 0;
  bool counted = false;
  bool cached = false;     // statistics from hq_ctx::build_stats (no count pass, verified on device)
  std::string stats_key;   // cache key; empty when the cache is off
  DevBuf scratch;  // count-pass block partials
  struct { unsigned long long cnt; int kmin, kmax, pmin, pmax; unsigned set[8]; } st{};
  void* host_st = nullptr;  // this build's slot in hq_ctx::pinned_build (st's layout)
};

void build_prepare(hq_ctx* ctx, const hq_build_desc* d, hq_hash* h, BuildState& bs) {
  const hq_table* t = d->src;
  if (!t) HQ_THROW(HQ_ERR_ARG, "build: NULL source table");
  if (t->host_stream) HQ_THROW(HQ_ERR_UNSUPPORTED, "build: the source is an HQ_HOST_STREAM (host) table");
  if (d->npreds < 0 || d->npreds > HQ_MAX_PREDS) HQ_THROW(HQ_ERR_UNSUPPORTED, "build: too many predicates");
  if (d->npayload < 0 || d->npayload > HQ_MAX_PAYLOAD) HQ_THROW(HQ_ERR_UNSUPPORTED, "build: 0..3 payload columns");
  if (d->key_col < 0 || d->key_col >= t->ncols) HQ_THROW(HQ_ERR_ARG, "build: key column out of range");
  KBuild& b = bs.b;
  b.n = t->nrows;
  b.ndev = t->dev_rows;
  for (int c = 0; c < t->ncols; ++c) {
    b.col[c] = (const char*)t->cols[c].ptr;
    b.colw[c] = t->cols[c].width;
  }
  b.npreds = d->npreds;
  for (int i = 0; i < d->npreds; ++i) to_kpred(d->preds[i], b.preds[i], t->ncols);
  b.key_col = d->key_col;
  b.npay = d->npayload;
  b.composite = d->composite != 0;
  if (b.composite && d->npayload < 1) HQ_THROW(HQ_ERR_ARG, "build: a composite key needs payload_cols[0] (the second key)");
  for (int k = 0; k < d->npayload; ++k) {
    if (d->payload_cols[k] < 0 || d->payload_cols[k] >= t->ncols) HQ_THROW(HQ_ERR_ARG, "build: payload column out of range");
    b.pay_col[k] = d->payload_cols[k];
  }
  h->dstate = DevBuf(ctx, 128);
  HQ_CUDA(cudaMemsetAsync(h->dstate.p, 0, 128, ctx->stream));
  b.err = h->dstate.as<int>();
  b.nkeys = (unsigned long long*)(h->dstate.as<char>() + 8);
  b.kminmax = (int*)(h->dstate.as<char>() + 16);
  b.pset = (unsigned*)(h->dstate.as<char>() + 64);
  bs.grid = (int)std::max<int64_t>(1, (b.n + BUILD_BLOCK * BUILD_U - 1) / (BUILD_BLOCK * BUILD_U));
  bs.words = d->npayload == 0 ? 1 : (d->npayload == 1 ? 2 : 4);
  bs.counted = d->expected_rows <= 0;
  if (bs.counted && stats_cache_on()) {
    // the descriptor's identity: source table uid + everything the statistics depend on
    std::string& k = bs.stats_key;
    auto put = [&](const void* p, size_t n) { k.append((const char*)p, n); };
    put(&t->uid, sizeof(t->uid));
    put(&b.n, sizeof(b.n));
    put(&b.npreds, sizeof(b.npreds));
    put(b.preds, sizeof(KBuildPred) * (size_t)b.npreds);
    put(&b.key_col, sizeof(b.key_col));
    put(&b.npay, sizeof(b.npay));
    put(b.pay_col, sizeof(b.pay_col));
    put(&b.composite, sizeof(b.composite));
    auto it = ctx->build_stats.find(k);
    if (it != ctx->build_stats.end()) {
      const BuildStats& c = it->second;
      bs.cached = true;
      bs.st.cnt = c.cnt;
      bs.st.kmin = c.kmin; bs.st.kmax = c.kmax; bs.st.pmin = c.pmin; bs.st.pmax = c.pmax;
      for (int w = 0; w < 8; ++w) bs.st.set[w] = c.set[w];
      b.verify = 1;
      b.vs = c;
      b.vqual = (unsigned long long*)(h->dstate.as<char>() + 40);  // zeroed with dstate
      b.ticket = (unsigned*)(h->dstate.as<char>() + 32);
      return;
    }
  }
  if (bs.counted) {  // exact count pass: number and range of the qualifying keys
    // (kminmax needs no initial values: the count kernel's last block writes
    // them; an empty table has count 0 and its range is never read)
    bs.scratch = DevBuf(ctx, (size_t)bs.grid * sizeof(CountPart) + 16);
    b.part = bs.scratch.p;
    b.ticket = (unsigned*)(h->dstate.as<char>() + 32);  // zeroed with dstate
    if (b.n > 0) { ctx->launches++; hq_build_count_kernel<<<bs.grid, BUILD_BLOCK, 0, ctx->stream>>>(b); }
    HQ_CUDA(cudaGetLastError());
    // statistics -> pinned staging (truly asynchronous copies; read after the one sync)
    HQ_CUDA(cudaMemcpyAsync(bs.host_st, b.nkeys, 24, cudaMemcpyDeviceToHost, ctx->stream));
    HQ_CUDA(cudaMemcpyAsync((char*)bs.host_st + 24, b.pset, 32, cudaMemcpyDeviceToHost, ctx->stream));
  }
}

void build_finish(hq_ctx* ctx, const hq_build_desc* d, hq_hash* h, BuildState& bs) {
  KBuild& b = bs.b;
  const int words = bs.words;
  int64_t keys = d->expected_rows;
  bool direct = false;
  int64_t kmin = 0, range = 0;
  h->meta.pay_min = INT_MAX;  // payload range unknown unless counted
  h->meta.pay_max = INT_MIN;
  if (bs.counted) {
    HQ_CUDA(cudaMemsetAsync(b.nkeys, 0, 8, ctx->stream));
    keys = (int64_t)bs.st.cnt;
    h->meta.pay_min = bs.st.pmin;
    h->meta.pay_max = bs.st.pmax;
    for (int k = 0; k < 4; ++k) h->meta.pay_set[k] = (uint64_t)bs.st.set[2 * k] | ((uint64_t)bs.st.set[2 * k + 1] << 32);
    if (keys > 0 && bs.st.kmin <= bs.st.kmax) {
      kmin = bs.st.kmin;
      range = (int64_t)bs.st.kmax - bs.st.kmin + 1;
      // dense keys: direct-mapped slot array (one load per probe)
      direct = !b.composite && range <= (1LL << 30) && (range <= 8 * keys || range * words * 4 <= (2LL << 20));
    }
  }
  const int64_t cap = direct ? range : std::max<int64_t>(16, next_pow2((keys * 5 + 2) / 3));  // load <= 0.6
  if (cap > (1LL << 31)) HQ_THROW(HQ_ERR_UNSUPPORTED, "build: hash table too large");
  int log2 = 0;
  while ((1LL << log2) < cap) ++log2;
  // compact-only direct table (hq_build_direct_compact_kernel): the compact form is
  // derived from the statistics alone, so no slot array is written at all
  const int ckind = direct && bs.counted ? hq_compact_kind(d->npayload, bs.st.pmin, bs.st.pmax) : 0;
  const bool conly = ckind != 0 && !b.composite && !getenv("HQ_BUILD_SLOTS");
  // sparse unique keys with a known range (counted): the ranked form instead of a slot array
  const bool rform = !direct && !b.composite && bs.counted && keys > 0 && range > 0 &&
                     (range + 31) / 32 * 4 <= (64LL << 20) && !getenv("HQ_BUILD_SLOTS");
  if (!conly && !rform) {
    h->owned = DevBuf(ctx, (size_t)cap * words * 4);
    h->slots = h->owned.as<uint32_t>();
  }
  h->log2cap = log2;
  h->meta.capacity = cap;
  h->meta.slot_words = words;
  h->meta.npayload = d->npayload;
  h->meta.composite = b.composite;
  h->meta.nkeys = bs.counted ? keys : -1;  // exact after the count pass (confirmed at hq_hash_info)
  h->src_rows = b.n;
  h->src_uid = d->src->uid;
  h->meta.bytes = cap * words * 4;
  h->meta.layout = direct ? HQ_HT_DIRECT : HQ_HT_LINEAR;
  h->meta.key_min = kmin;
  h->meta.key_max = range > 0 ? (int32_t)(kmin + range - 1) : (int32_t)kmin - 1;  // empty range when unknown
  h->stats_key = bs.stats_key;
  if (rform) {
    int64_t od = 0, op = 0, tot = 0;
    int stride = 0;
    hq_ranked_layout(range, keys, d->npayload, &od, &op, &tot, &stride);
    h->compact = DevBuf(ctx, (size_t)tot + 16);
    // the bitmap is built apart (dense words: contiguous atomics, a half-size scan) and the
    // directory kernel writes it out with the directory as the {bits, dir} pairs
    const int64_t bwords = stride ? op / 8 : op / 4;
    DevBuf scratch;
    uint32_t* bm = h->compact.as<uint32_t>();
    if (stride) {
      scratch = DevBuf(ctx, (size_t)bwords * 4 + 16);
      bm = scratch.as<uint32_t>();
    }
    HQ_CUDA(cudaMemsetAsync(bm, 0, (size_t)bwords * 4, ctx->stream));  // the bitmap and its padding
    b.dmin = (int32_t)kmin;
    if (b.n > 0) {  // bitmap + duplicate / bad-key / statistics checks
      ctx->launches++;
      hq_build_direct_compact_kernel<<<bs.grid, BUILD_BLOCK, 0, ctx->stream>>>(b, 1, bm, range, 0, 0, CLut{});
    }
    HQ_CUDA(cudaGetLastError());
    if (stride) {
      const int nblk = (int)(bwords / (RSCAN_T * RSCAN_W));
      if (!getenv("HQ_RANK_3PASS")) {  // single-pass directory (decoupled look-back)
        DevBuf st(ctx, (size_t)nblk * 8 + 16);
        HQ_CUDA(cudaMemsetAsync(st.p, 0, (size_t)nblk * 8 + 16, ctx->stream));
        ctx->launches += 1;
        hq_rank_dir1_kernel<<<nblk, RSCAN_T, 0, ctx->stream>>>(bm, st.as<unsigned long long>(),
                                                               (unsigned*)(st.as<char>() + (size_t)nblk * 8), h->compact.as<uint32_t>());
      } else {
      DevBuf bsum(ctx, (size_t)nblk * 4 + 16);
      ctx->launches += 3;
      hq_rank_blocksum_kernel<<<nblk, RSCAN_T, 0, ctx->stream>>>(bm, 1, bsum.as<unsigned>());
      hq_rank_topscan_kernel<<<1, RSCAN_T, 0, ctx->stream>>>(bsum.as<unsigned>(), nblk);
      hq_rank_dir_kernel<<<nblk, RSCAN_T, 0, ctx->stream>>>(bm, bsum.as<unsigned>(), h->compact.as<uint32_t>());
      }
      if (b.n > 0) {
        ctx->launches++;
        hq_build_ranked_scatter_kernel<<<bs.grid, BUILD_BLOCK, 0, ctx->stream>>>(
            b, h->compact.as<uint2>(), (int*)(h->compact.as<char>() + op), stride, range, (unsigned long long)keys);
      }
      HQ_CUDA(cudaGetLastError());
    }
    h->ckind = 4;
    h->cbytes = tot;
    h->roff_dir = od;
    h->roff_pay = op;
    h->rstride = stride;
    h->compact_only = true;
    return;
  }
  if (conly) {
    const long long cwords = hq_compact_words(ckind, range);
    h->compact = DevBuf(ctx, (size_t)cwords * 4 + 16);
    HQ_CUDA(cudaMemsetAsync(h->compact.p, ckind == 1 ? 0x00 : 0xFF, (size_t)cwords * 4 + 16, ctx->stream));
    CLut lut{};
    const int crank = ckind == 2 ? hq_rank_lut(h->meta, lut.r) : 0;
    b.dmin = (int32_t)kmin;
    if (b.n > 0) {
      ctx->launches++;
      hq_build_direct_compact_kernel<<<bs.grid, BUILD_BLOCK, 0, ctx->stream>>>(b, ckind, h->compact.as<uint32_t>(), range,
                                                                               h->meta.pay_min, crank, lut);
    }
    HQ_CUDA(cudaGetLastError());
    h->ckind = ckind;
    h->crank = crank;
    h->cbytes = cwords * 4;
    h->compact_only = true;
    return;
  }
  const int64_t nw = cap * words;
  const int fgrid = (int)std::max<int64_t>(1, std::min<int64_t>((nw + 255) / 256, (int64_t)ctx->num_sms * 8));
  ctx->launches++;
  hq_fill_kernel<<<fgrid, 256, 0, ctx->stream>>>(h->slots, nw, 0x80000000u);
  HQ_CUDA(cudaGetLastError());
  b.slots = h->slots;
  b.mask = direct ? (uint32_t)cap : (uint32_t)(cap - 1);
  b.log2cap = log2;
  b.words = words;
  b.direct = direct;
  b.dmin = (int32_t)kmin;
  b.count_inserts = bs.counted ? 0 : 1;
  if (b.n > 0) { ctx->launches++; hq_build_hash_kernel<<<bs.grid, BUILD_BLOCK, 0, ctx->stream>>>(b); }
  HQ_CUDA(cudaGetLastError());
  hq_build_compact(ctx, h);
}
}  // namespace

void hq_build_hashes_impl(hq_ctx* ctx, int n, const hq_build_desc* d, hq_hash* const* h) {
  std::vector<BuildState> bs((size_t)n);
  bool any_count = false;
  const size_t slot = 64;
  static_assert(sizeof(BuildState::st) <= 64, "stats slot");
  if (ctx->pinned_build_bytes < (size_t)n * slot) {
    if (ctx->pinned_build) HQ_CUDA(cudaFreeHost(ctx->pinned_build));
    ctx->pinned_build = nullptr;
    ctx->pinned_build_bytes = 0;
    const size_t want = std::max<size_t>((size_t)n * slot, 16 * slot);
    HQ_CUDA(cudaHostAlloc(&ctx->pinned_build, want, cudaHostAllocDefault));
    ctx->pinned_build_bytes = want;
  }
  // Independent builds run concurrently: build i is enqueued on side stream i % NSIDE,
  // forked from the context stream by an event and joined back by another, so the
  // small dimension tables' kernels overlap instead of queueing behind each other.
  // Every allocation of a build is made while ctx->stream points at its side stream
  // (stream-ordered); the join makes the context stream wait for all of them.  With
  // caller allocator hooks (which may not order frees across streams) builds stay on
  // the context stream.
  const int nside = (n > 1 && !ctx->has_alloc) ? std::min(n, hq_ctx::NSIDE) : 0;
  if (nside && !ctx->ev_fork) {
    HQ_CUDA(cudaEventCreateWithFlags(&ctx->ev_fork, cudaEventDisableTiming));
    for (int k = 0; k < hq_ctx::NSIDE; ++k) {
      HQ_CUDA(cudaStreamCreateWithFlags(&ctx->side[k], cudaStreamNonBlocking));
      HQ_CUDA(cudaEventCreateWithFlags(&ctx->ev_join[k], cudaEventDisableTiming));
    }
  }
  cudaStream_t main = ctx->stream;
  auto fork = [&] {
    if (!nside) return;
    HQ_CUDA(cudaEventRecord(ctx->ev_fork, main));
    for (int k = 0; k < nside; ++k) HQ_CUDA(cudaStreamWaitEvent(ctx->side[k], ctx->ev_fork, 0));
  };
  auto join = [&] {
    ctx->stream = main;
    if (!nside) return;
    for (int k = 0; k < nside; ++k) {
      HQ_CUDA(cudaEventRecord(ctx->ev_join[k], ctx->side[k]));
      HQ_CUDA(cudaStreamWaitEvent(main, ctx->ev_join[k], 0));
    }
  };
  try {
    fork();
    for (int i = 0; i < n; ++i) {
      bs[i].host_st = (char*)ctx->pinned_build + (size_t)i * slot;
      if (nside) ctx->stream = ctx->side[i % nside];
      build_prepare(ctx, d + i, h[i], bs[i]);
      any_count = any_count || (bs[i].counted && !bs[i].cached);
    }
    join();
    if (any_count) {
      ctx->stream = main;
      hq_sync(ctx, "a hash build without cached statistics (its count pass)");
    }
    for (int i = 0; i < n; ++i)
      if (bs[i].counted && !bs[i].cached) {
        std::memcpy(&bs[i].st, bs[i].host_st, sizeof(bs[i].st));
        if (!bs[i].stats_key.empty()) {
          BuildStats c;
          c.cnt = bs[i].st.cnt;
          c.kmin = bs[i].st.kmin; c.kmax = bs[i].st.kmax; c.pmin = bs[i].st.pmin; c.pmax = bs[i].st.pmax;
          for (int w = 0; w < 8; ++w) c.set[w] = bs[i].st.set[w];
          if (ctx->build_stats.size() > 4096) ctx->build_stats.clear();
          ctx->build_stats[bs[i].stats_key] = c;
        }
      }
    fork();
    for (int i = 0; i < n; ++i) {
      if (nside) ctx->stream = ctx->side[i % nside];
      build_finish(ctx, d + i, h[i], bs[i]);
    }
    join();
  } catch (...) {
    ctx->stream = main;
    throw;
  }
}

namespace {
// bitmap of present keys: a warp reads 32 consecutive slots (coalesced) and
// one ballot is the word
__global__ void hq_compact_bitmap_kernel(const uint32_t* slots, long long range, uint32_t* out) {
  const long long nwords = (range + 31) / 32;
  const int lane = threadIdx.x & 31;
  const long long wstride = (long long)gridDim.x * (blockDim.x >> 5);
  for (long long w = blockIdx.x * (long long)(blockDim.x >> 5) + (threadIdx.x >> 5); w < nwords; w += wstride) {
    const long long i = w * 32 + lane;
    const uint32_t bits = __ballot_sync(0xffffffffu, i < range && (int)slots[i] != INT_MIN);
    if (lane == 0) out[w] = bits;
  }
}
// key-range bitmap of a linear table: one bit per key in [kmin, kmin + range)
__global__ void hq_prefilter_kernel(const uint32_t* slots, long long cap, int words, int kmin, long long range,
                                    uint32_t* bm) {
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < cap; i += (long long)gridDim.x * blockDim.x) {
    const int k = (int)slots[i * words];
    if (k == INT_MIN) continue;
    const long long d = (long long)k - kmin;
    if (d >= 0 && d < range) atomicOr(bm + (d >> 5), 1u << (d & 31));
  }
}
// one byte per key: payload0 - pay_min, or its rank in the payload set when a LUT is
// given (sparse value sets: the generated kernel then indexes a ranked group key with
// the byte itself); 0xFF = absent (8-B slots {key, payload}); thread per key,
// coalesced 8-B slot reads and byte writes
struct RankLut {
  unsigned char r[256];
};
__global__ void hq_compact_u8_kernel(const uint32_t* slots, long long range, int pay_min, uint32_t* out, int use_lut,
                                     const __grid_constant__ RankLut lut) {
  unsigned char* o = (unsigned char*)out;
  const long long n = (range + 3) / 4 * 4;  // whole words (the tail bytes read as absent)
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
    uint32_t byte = 0xFFu;
    if (i < range) {
      const uint2 s = ((const uint2*)slots)[i];
      if ((int)s.x != INT_MIN) {
        byte = (uint32_t)((int)s.y - pay_min) & 0xFFu;
        if (use_lut) byte = lut.r[byte];
      }
    }
    o[i] = (unsigned char)byte;
  }
}
// one nibble per key: payload0 - pay_min (< 15), 0xF = absent (8-B slots
// {key, payload}); thread per key, eight lanes OR their nibbles into a word
__global__ void hq_compact_u4_kernel(const uint32_t* slots, long long range, int pay_min, uint32_t* out) {
  const long long n = (range + 255) / 256 * 256;  // whole warps (the tail reads as absent)
  const int lane = threadIdx.x & 31;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
    uint32_t nib = 0xFu;
    if (i < range) {
      const uint2 s = ((const uint2*)slots)[i];
      if ((int)s.x != INT_MIN) nib = (uint32_t)((int)s.y - pay_min) & 0xFu;
    }
    uint32_t v = nib << (4 * (lane & 7));
#pragma unroll
    for (int o = 1; o < 8; o <<= 1) v |= __shfl_xor_sync(0xffffffffu, v, o);
    if ((lane & 7) == 0 && i / 8 < (range + 7) / 8) out[i / 8] = v;
  }
}
}  // namespace

// Compact derived form of a direct table (used by generated kernels to stage
// small probe tables in shared memory): bitmap for semi-joins, bytes for one
// small payload.  Also run on import (multi-GPU) from the broadcast slots.
void hq_build_compact(hq_ctx* ctx, hq_hash* h) {
  h->ckind = 0;
  h->crank = 0;
  h->cbytes = 0;
  h->pf_words = 0;
  if (h->meta.layout == HQ_HT_LINEAR) {
    // exact key-range bitmap in front of the slot array (semi-join prefilter)
    const long long range = (long long)h->meta.key_max - h->meta.key_min + 1;
    const long long words = (range + 31) / 32;
    if (range <= 0 || words * 4 > (64LL << 20)) return;
    h->prefilter = DevBuf(ctx, (size_t)words * 4 + 16);
    HQ_CUDA(cudaMemsetAsync(h->prefilter.p, 0, (size_t)words * 4 + 16, ctx->stream));
    const long long cap = h->meta.capacity;
    const int grid = (int)std::max<long long>(1, std::min<long long>((cap + 255) / 256, (long long)ctx->num_sms * 8));
    ctx->launches++;
    hq_prefilter_kernel<<<grid, 256, 0, ctx->stream>>>(h->slots, cap, h->meta.slot_words, (int)h->meta.key_min,
                                                       range, h->prefilter.as<uint32_t>());
    HQ_CUDA(cudaGetLastError());
    h->pf_words = words;
    return;
  }
  if (h->meta.layout != HQ_HT_DIRECT) return;
  const long long range = h->meta.capacity;
  const int kind = h->meta.composite ? 0 : hq_compact_kind(h->meta.npayload, h->meta.pay_min, h->meta.pay_max);
  if (!kind) return;
  const long long words = hq_compact_words(kind, range);
  h->compact = DevBuf(ctx, (size_t)words * 4 + 16);
  const int grid = (int)std::max<long long>(1, std::min<long long>((range + 255) / 256, (long long)ctx->num_sms * 8));
  ctx->launches++;
  if (kind == 1) hq_compact_bitmap_kernel<<<grid, 256, 0, ctx->stream>>>(h->slots, range, h->compact.as<uint32_t>());
  else if (kind == 2) {
    // a sparse payload-value set (SSB Q3.1's five ASIA nations among codes 8..24): rank-code
    RankLut lut{};
    h->crank = hq_rank_lut(h->meta, lut.r);
    hq_compact_u8_kernel<<<grid, 256, 0, ctx->stream>>>(h->slots, range, h->meta.pay_min, h->compact.as<uint32_t>(),
                                                        h->crank, lut);
  }
  else hq_compact_u4_kernel<<<grid, 256, 0, ctx->stream>>>(h->slots, range, h->meta.pay_min, h->compact.as<uint32_t>());
  HQ_CUDA(cudaGetLastError());
  h->ckind = kind;
  h->cbytes = words * 4;
}

const uint32_t* hq_hash_slots(hq_ctx* ctx, hq_hash* h) {
  if (h->slots || !h->compact_only) return h->slots;
  if (h->ranked()) {  // a linear slot array with the same capacity the meta describes
    const long long cap = h->meta.capacity;
    const int words = h->meta.slot_words;
    h->owned = DevBuf(ctx, (size_t)cap * words * 4 + 16);
    const int fgrid = (int)std::max<long long>(1, std::min<long long>((cap * words + 255) / 256, (long long)ctx->num_sms * 8));
    const long long range = (long long)h->meta.key_max - h->meta.key_min + 1;
    const int grid = (int)std::max<long long>(1, std::min<long long>((range + 255) / 256, (long long)ctx->num_sms * 8));
    const char* base = (const char*)h->compact_ptr();
    if (!h->dstate.p) {  // an imported table: a fault word for the derivation
      h->dstate = DevBuf(ctx, 128);
      HQ_CUDA(cudaMemsetAsync(h->dstate.p, 0, 128, ctx->stream));
    }
    ctx->launches += 2;
    hq_fill_kernel<<<fgrid, 256, 0, ctx->stream>>>(h->owned.as<uint32_t>(), cap * words, 0x80000000u);
    hq_slots_from_ranked_kernel<<<grid, 256, 0, ctx->stream>>>(
        (const uint32_t*)base, (const int*)(base + h->roff_pay), h->rstride, h->meta.npayload, range,
        (int)h->meta.key_min, h->owned.as<uint32_t>(), (uint32_t)(cap - 1), h->log2cap, words, h->dstate.as<int>());
    HQ_CUDA(cudaGetLastError());
    h->slots = h->owned.as<uint32_t>();
    return h->slots;
  }
  const long long range = h->meta.capacity;
  const int words = h->meta.slot_words;
  h->owned = DevBuf(ctx, (size_t)range * words * 4 + 16);
  CLut lo{}, hi{};
  int use_rv = 0;
  if (h->ckind == 2 && h->crank) {  // rank -> offset from pay_min
    unsigned char lut[256];
    hq_rank_lut(h->meta, lut);
    for (int d = 0; d < 255; ++d)
      if (lut[d] != 0xFF) {
        lo.r[lut[d]] = (unsigned char)(d & 255);
        hi.r[lut[d]] = (unsigned char)(d >> 8);
      }
    use_rv = 1;
  }
  const int grid = (int)std::max<long long>(1, std::min<long long>((range + 255) / 256, (long long)ctx->num_sms * 8));
  ctx->launches++;
  hq_slots_from_compact_kernel<<<grid, 256, 0, ctx->stream>>>((const uint32_t*)h->compact_ptr(), h->ckind, range,
                                                                (int)h->meta.key_min, h->meta.pay_min, use_rv, lo, hi,
                                                                h->owned.as<uint32_t>());
  HQ_CUDA(cudaGetLastError());
  h->slots = h->owned.as<uint32_t>();
  return h->slots;
}

// Sync and report build faults (HQ_ERR_DUP_KEY etc.).
void hq_hash_check(hq_ctx* ctx, hq_hash* h) {
  if (h->checked || !h->dstate.p) return;
  hq_require_eager(ctx, "a hash build's fault check");
  int st[4];
  HQ_CUDA(cudaMemcpyAsync(st, h->dstate.p, 16, cudaMemcpyDeviceToHost, ctx->stream));
  HQ_CUDA(cudaStreamSynchronize(ctx->stream));
  if (h->meta.nkeys < 0) h->meta.nkeys = (int64_t)(*(unsigned long long*)(st + 2));  // expected_rows builds
  h->checked = true;
  // stale statistics first: a table sized from them can also report keys out of range
  if (st[0] & HQF_STALE) {
    ctx->build_stats.erase(h->stats_key);  // the next build of this descriptor counts again
    ctx->derived_rows.erase(h->src_uid);   // (and a result view re-reads its row count)
    HQ_THROW(HQ_ERR_STATE, "hash build: the source table's rows differ from the statistics cached when it was "
                           "last built (tables are immutable; the statistics were dropped, re-run the query)");
  }
  if (st[0] & HQF_DUP_KEY) HQ_THROW(HQ_ERR_DUP_KEY, "hash build: duplicate key (join keys must be unique)");
  if (st[0] & HQF_BAD_KEY) HQ_THROW(HQ_ERR_ARG, "hash build: key INT32_MIN or outside int32");
  if (st[0] & HQF_BAD_PAYLOAD) HQ_THROW(HQ_ERR_ARG, "hash build: payload outside int32");
  if (st[0] & HQF_HT_FULL) HQ_THROW(HQ_ERR_OVERFLOW, "hash build: table full (expected_rows too small)");
}

// ------------------------------------------------------------ column statistics
namespace {
__global__ void hq_column_range_kernel(const char* col, int w, long long n, long long* out) {
  long long mn = LLONG_MAX, mx = LLONG_MIN;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
    const long long v = w == 4 ? (long long)((const int*)col)[i] : (w == 8 ? ((const long long*)col)[i] : (long long)((const signed char*)col)[i]);
    mn = v < mn ? v : mn;
    mx = v > mx ? v : mx;
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const long long a = __shfl_xor_sync(0xffffffffu, mn, o), b = __shfl_xor_sync(0xffffffffu, mx, o);
    mn = a < mn ? a : mn;
    mx = b > mx ? b : mx;
  }
  if ((threadIdx.x & 31) == 0) {
    atomicMin(out, mn);
    atomicMax(out + 1, mx);
  }
}
}  // namespace

void hq_column_range_impl(hq_ctx* ctx, const hq_table* t, int col, int64_t* mn, int64_t* mx) {
  if (t->host_stream) HQ_THROW(HQ_ERR_UNSUPPORTED, "column range: HQ_HOST_STREAM table");
  DevBuf out(ctx, 16);
  const long long init[2] = {LLONG_MAX, LLONG_MIN};
  long long* h = (long long*)pinned_staging(ctx, 16);
  std::memcpy(h, init, 16);
  HQ_CUDA(cudaMemcpyAsync(out.p, h, 16, cudaMemcpyHostToDevice, ctx->stream));
  if (t->nrows > 0) {
    const int grid = (int)std::max<long long>(1, std::min<long long>((t->nrows + 255) / 256, (long long)ctx->num_sms * 8));
    ctx->launches++;
    hq_column_range_kernel<<<grid, 256, 0, ctx->stream>>>((const char*)t->cols[col].ptr, t->cols[col].width, t->nrows,
                                                          out.as<long long>());
    HQ_CUDA(cudaGetLastError());
  }
  HQ_CUDA(cudaMemcpyAsync(h, out.p, 16, cudaMemcpyDeviceToHost, ctx->stream));
  HQ_CUDA(cudaStreamSynchronize(ctx->stream));
  *mn = h[0];
  *mx = h[1];
}
