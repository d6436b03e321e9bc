// hq_finalize.cu -- post-processing of aggregation results outside the
// pipeline (sorting and decompression run after the
// compiled kernels): compaction of the global group table into rows, AVG,
// ORDER BY with a total tie-break, LIMIT.  Runs on the device of the context
// (GPU 0 in the multi-GPU flow).
#include <cub/device/device_radix_sort.cuh>

#include <algorithm>
#include <climits>
#include <cstring>

#include "hq_internal.h"

using namespace hqk;

namespace {

constexpr int SORT_CHUNK = 2048;  // rows sorted per block in shared memory
constexpr int MAXRC = HQ_MAX_KEYS + HQ_MAX_AGGS;

struct KCompact {
  const long long* gtab;
  long long ngroups;  // dense groups or hash capacity
  uint32_t vwords;
  int hash;
  int nkeys, naggs;
  long long key_min[HQ_MAX_KEYS], key_card[HQ_MAX_KEYS], key_stride[HQ_MAX_KEYS];
  uint8_t agg_fn[HQ_MAX_AGGS];
  double agg_div[HQ_MAX_AGGS];  // 10^scale for AVG
  long long* out[MAXRC];
  unsigned long long* nout;     // [0] rows, [1] qualifying
  int* err;
  int scalar;
};

// write one live group entry as result row `row` (keys decoded from the packed index)
__device__ __forceinline__ void compact_emit(const KCompact& k, const long long* e, unsigned long long key,
                                             long long cnt, unsigned long long row) {
  for (int i = 0; i < k.nkeys; ++i)
    k.out[i][row] = k.key_min[i] + (long long)((key / (unsigned long long)k.key_stride[i]) % (unsigned long long)k.key_card[i]);
  bool big = false;
  for (int a = 0; a < k.naggs; ++a) {
    const long long v = e[1 + a];
    long long* o = k.out[k.nkeys + a];
    if (k.agg_fn[a] == HQ_AGG_AVG) {
      const double d = cnt ? (double)v / (double)cnt / k.agg_div[a] : __longlong_as_double(0x7ff8000000000000LL);
      o[row] = __double_as_longlong(d);
    } else {
      o[row] = v;
    }
    if ((k.agg_fn[a] == HQ_AGG_SUM || k.agg_fn[a] == HQ_AGG_AVG) && (v >= (1LL << 62) || v <= -(1LL << 62))) big = true;
  }
  if (big) atomicOr(k.err, HQF_OVERFLOW);
}

// Compaction of the group table into result rows: a block takes tiles of
// blockDim x COMPACT_PER_THREAD entries, scans its live-entry counts in shared
// memory and claims its output range with ONE atomic per tile (a warp-level
// atomic on the single row counter serialised: a 60 M-entry dense table -- TPC-H
// Q18's GROUP BY l_orderkey -- spent 4 ms in 1.9 M same-address atomics).
constexpr int COMPACT_PER_THREAD = 8;
__global__ void __launch_bounds__(256) hq_compact_kernel(const __grid_constant__ KCompact k) {
  const uint32_t stride = k.vwords + (k.hash ? 1 : 0);
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  __shared__ unsigned long long s_cnt[32], s_qual[32], s_base;
  const long long tile = (long long)blockDim.x * COMPACT_PER_THREAD;
  for (long long t0 = blockIdx.x * tile; t0 < k.ngroups; t0 += (long long)gridDim.x * tile) {
    unsigned live = 0;
    int nl = 0;
    unsigned long long q = 0;
#pragma unroll
    for (int c = 0; c < COMPACT_PER_THREAD; ++c) {
      const long long g = t0 + (long long)c * blockDim.x + threadIdx.x;
      if (g >= k.ngroups) continue;
      const long long* e = k.gtab + g * stride;
      bool l = true;
      if (k.hash) {
        l = (unsigned long long)e[0] != EMPTY_KEY;
        ++e;
      }
      const long long cnt = l ? e[0] : 0;
      l = l && (cnt != 0 || k.scalar);
      if (l) {
        live |= 1u << c;
        ++nl;
        q += (unsigned long long)cnt;
      }
    }
    int incl = nl;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int t = __shfl_up_sync(0xffffffffu, incl, o);
      if (lane >= o) incl += t;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) q += __shfl_xor_sync(0xffffffffu, q, o);
    if (lane == 31) s_cnt[warp] = (unsigned long long)incl;
    if (lane == 0) s_qual[warp] = q;
    __syncthreads();
    if (threadIdx.x == 0) {
      unsigned long long tot = 0, qt = 0;
      for (int w = 0; w < nw; ++w) {
        const unsigned long long c = s_cnt[w];
        s_cnt[w] = tot;  // exclusive prefix of the warps
        tot += c;
        qt += s_qual[w];
      }
      s_base = tot ? atomicAdd(k.nout, tot) : 0ull;
      if (qt) atomicAdd(k.nout + 1, qt);
    }
    __syncthreads();
    unsigned long long row = s_base + s_cnt[warp] + (unsigned long long)(incl - nl);
#pragma unroll
    for (int c = 0; c < COMPACT_PER_THREAD; ++c) {
      if (!((live >> c) & 1u)) continue;
      const long long g = t0 + (long long)c * blockDim.x + threadIdx.x;
      const long long* e = k.gtab + g * stride;
      unsigned long long key = (unsigned long long)g;
      if (k.hash) key = (unsigned long long)*e++;
      compact_emit(k, e, key, e[0], row++);
    }
    __syncthreads();  // s_cnt / s_base are reused by the next tile
  }
}

struct KSort {
  const long long* col[MAXRC];
  uint8_t isf[MAXRC];
  int norder;
  int ocol[HQ_MAX_ORDER];
  int odesc[HQ_MAX_ORDER];
  int nkeys;
};

__device__ __forceinline__ int cmp_val(const KSort& s, int c, int a, int b) {
  const long long x = s.col[c][a], y = s.col[c][b];
  if (s.isf[c]) {
    const double dx = __longlong_as_double(x), dy = __longlong_as_double(y);
    return dx < dy ? -1 : (dx > dy ? 1 : 0);
  }
  return x < y ? -1 : (x > y ? 1 : 0);
}
// the same order over columns at `col` (the small finalize's shared-memory copies)
__device__ __forceinline__ bool row_less_at(const KSort& s, const long long* const* col, int a, int b) {
  if (a < 0) return false;
  if (b < 0) return true;
  auto cmp = [&](int c) {
    const long long x = col[c][a], y = col[c][b];
    if (s.isf[c]) {
      const double dx = __longlong_as_double(x), dy = __longlong_as_double(y);
      return dx < dy ? -1 : (dx > dy ? 1 : 0);
    }
    return x < y ? -1 : (x > y ? 1 : 0);
  };
  for (int i = 0; i < s.norder; ++i) {
    int c = cmp(s.ocol[i]);
    if (s.odesc[i]) c = -c;
    if (c) return c < 0;
  }
  for (int i = 0; i < s.nkeys; ++i) {
    const int c = cmp(i);
    if (c) return c < 0;
  }
  return a < b;
}
// the same order over the small finalize's staged columns (column c at st + c * n); ord[i]:
// column | 0x100 descending | 0x200 float
__device__ __forceinline__ bool row_less_st(const long long* st, int n, const int* ord, int nord, int a, int b) {
  if (a < 0) return false;
  if (b < 0) return true;
  for (int i = 0; i < nord; ++i) {
    const int c = ord[i] & 0xFF;
    const long long x = st[c * n + a], y = st[c * n + b];
    int r;
    if (ord[i] & 0x200) {
      const double dx = __longlong_as_double(x), dy = __longlong_as_double(y);
      r = dx < dy ? -1 : (dx > dy ? 1 : 0);
    } else {
      r = x < y ? -1 : (x > y ? 1 : 0);
    }
    if (ord[i] & 0x100) r = -r;
    if (r) return r < 0;
  }
  return a < b;
}
// total order: ORDER BY columns, then the group keys ascending, then row id
__device__ __forceinline__ bool row_less(const KSort& s, int a, int b) {
  if (a < 0) return false;  // padding sorts last
  if (b < 0) return true;
  for (int i = 0; i < s.norder; ++i) {
    int c = cmp_val(s, s.ocol[i], a, b);
    if (s.odesc[i]) c = -c;
    if (c) return c < 0;
  }
  for (int i = 0; i < s.nkeys; ++i) {
    const int c = cmp_val(s, i, a, b);
    if (c) return c < 0;
  }
  return a < b;
}

// Each block sorts one chunk of <= SORT_CHUNK indices (bitonic network in
// shared memory) and keeps its first `keep` rows.

__global__ void __launch_bounds__(1024) hq_chunk_sort_kernel(const __grid_constant__ KSort s, const int* in, long long n,
                                                             int* out, int keep, int net) {
  // net: power-of-two network size (<= SORT_CHUNK); chunks of `net` rows per block.
  // The first sort column travels with the indices in shared memory as an
  // order-preserving unsigned image, so a comparison reads global memory only on
  // a tie (TPC-H Q3's top 10 of ~1 M groups: every comparison loaded 2-5 columns)
  __shared__ int idx[SORT_CHUNK];
  __shared__ unsigned long long pk[SORT_CHUNK];
  const long long base = (long long)blockIdx.x * net;
  const int cnt = (int)(n - base < net ? n - base : net);
  const int c0 = s.norder > 0 ? s.ocol[0] : 0;
  const bool d0 = s.norder > 0 && s.odesc[0];
  const bool have0 = s.norder > 0 || s.nkeys > 0;
  for (int i = threadIdx.x; i < net; i += blockDim.x) {
    const int r = i < cnt ? (in ? in[base + i] : (int)(base + i)) : -1;
    idx[i] = r;
    unsigned long long t = ~0ull;  // padding (r < 0) sorts last
    if (r >= 0 && have0) {
      const long long v = s.col[c0][r];
      t = s.isf[c0] ? (v < 0 ? ~(unsigned long long)v : (unsigned long long)v ^ 0x8000000000000000ull)
                    : (unsigned long long)v ^ 0x8000000000000000ull;
      if (d0) t = ~t;
    } else if (r >= 0) {
      t = 0;
    }
    pk[i] = t;
  }
  __syncthreads();
  for (int k = 2; k <= net; k <<= 1) {
    for (int j = k >> 1; j > 0; j >>= 1) {
      for (int i = threadIdx.x; i < net; i += blockDim.x) {
        const int l = i ^ j;
        if (l > i) {
          const int a = idx[i], b = idx[l];
          const unsigned long long ka = pk[i], kb = pk[l];
          const bool up = (i & k) == 0;
          // (a < b) under the total order: the shared key first, the full row on a tie
          const bool b_lt_a = kb != ka ? kb < ka : row_less(s, b, a);
          const bool a_lt_b = kb != ka ? ka < kb : row_less(s, a, b);
          const bool sw = up ? b_lt_a : a_lt_b;
          if (sw) { idx[i] = b; idx[l] = a; pk[i] = kb; pk[l] = ka; }
        }
      }
      __syncthreads();
    }
  }
  const int m = keep < cnt ? keep : cnt;
  for (int i = threadIdx.x; i < m; i += blockDim.x) out[(long long)blockIdx.x * keep + i] = idx[i];
  for (int i = m + threadIdx.x; i < keep; i += blockDim.x) out[(long long)blockIdx.x * keep + i] = -1;
}

// Radix-sort key of one ORDER BY / group-key column in row order idx (NULL =
// identity): an unsigned image whose ascending order is the column's order.
// Group keys: v - key_min (< key_card, so only the low bits are sorted); order
// columns: int64 with the sign bit flipped, fp64 by the IEEE total-order map,
// bitwise NOT for DESC.
__global__ void hq_sortkey_kernel(const long long* __restrict__ col, const int* __restrict__ idx, long long n,
                                  int mode, long long kmin, int desc, unsigned long long* __restrict__ out) {
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
    const long long v = col[idx ? idx[i] : i];
    unsigned long long t;
    if (mode == 0) t = (unsigned long long)(v - kmin);                 // group key
    else if (mode == 1) t = (unsigned long long)v ^ 0x8000000000000000ull;  // int64
    else t = v < 0 ? ~(unsigned long long)v : (unsigned long long)v ^ 0x8000000000000000ull;  // fp64 bits
    out[i] = desc ? ~t : t;
  }
}

__global__ void hq_iota_kernel(int* idx, long long n, long long valid) {
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
    idx[i] = i < valid ? (int)i : -1;
}
__global__ void hq_gather_kernel(const long long* src, const int* idx, long long n, long long* dst) {
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
    dst[i] = src[idx[i]];
}

// ---- top-k of a large group table (ORDER BY ... LIMIT k, k <= TOPK_MAX): the table
// is read once, no compaction.  Pass 1: every block sorts a chunk of table entries
// (live ones only) under the result order and keeps its first k entry indices, and
// sums the groups' counts; pass 2 (one block): sorts the blocks' candidates, keeps k,
// decodes those k rows and stages rows + statistics for ONE host copy.
constexpr int TOPK_MAX = 256;
struct KTopK {
  KCompact k;       // the group table and its decoding (k.out unused)
  KSort s;          // s.norder / ocol / odesc / nkeys (s.col unused)
  int keep;         // rows kept per chunk (= limit)
  int* cand;        // pass 1 output: gridDim x keep entry indices (-1 = none)
  unsigned long long* stats;  // [0] rows kept, [1] qualifying, [2] fault bits, [3] live groups, [4] pipeline faults
  long long* res[MAXRC];      // final columns (keep rows each)
  const int* pipe_err;
  const int* hash_err[8];
  int nhash;
};
__device__ __forceinline__ const long long* tk_entry(const KCompact& k, long long g) {
  return k.gtab + g * (k.vwords + (k.hash ? 1 : 0)) + (k.hash ? 1 : 0);
}
__device__ __forceinline__ bool tk_live(const KCompact& k, long long g) {
  const long long* e = k.gtab + g * (k.vwords + (k.hash ? 1 : 0));
  if (k.hash && (unsigned long long)e[0] == EMPTY_KEY) return false;
  return (k.hash ? e[1] : e[0]) != 0;
}
// result column c of the group at table entry g (keys decoded, AVG as fp64 bits)
__device__ __forceinline__ long long tk_col(const KCompact& k, long long g, int c) {
  const long long* e = tk_entry(k, g);
  if (c < k.nkeys) {
    const unsigned long long key = k.hash ? (unsigned long long)e[-1] : (unsigned long long)g;
    return k.key_min[c] + (long long)((key / (unsigned long long)k.key_stride[c]) % (unsigned long long)k.key_card[c]);
  }
  const int a = c - k.nkeys;
  const long long v = e[1 + a];
  if (k.agg_fn[a] == HQ_AGG_AVG) {
    const long long cnt = e[0];
    const double d = cnt ? (double)v / (double)cnt / k.agg_div[a] : __longlong_as_double(0x7ff8000000000000LL);
    return __double_as_longlong(d);
  }
  return v;
}
__device__ __forceinline__ int tk_cmp(const KCompact& k, const KSort& s, int c, long long a, long long b) {
  const long long x = tk_col(k, a, c), y = tk_col(k, b, c);
  if (s.isf[c]) {
    const double dx = __longlong_as_double(x), dy = __longlong_as_double(y);
    return dx < dy ? -1 : (dx > dy ? 1 : 0);
  }
  return x < y ? -1 : (x > y ? 1 : 0);
}
// the total order of hq_finalize (ORDER BY, then group keys, then entry index)
__device__ __forceinline__ bool tk_less(const KCompact& k, const KSort& s, long long a, long long b) {
  if (a < 0) return false;
  if (b < 0) return true;
  for (int i = 0; i < s.norder; ++i) {
    int c = tk_cmp(k, s, s.ocol[i], a, b);
    if (s.odesc[i]) c = -c;
    if (c) return c < 0;
  }
  for (int i = 0; i < s.nkeys; ++i) {
    const int c = tk_cmp(k, s, i, a, b);
    if (c) return c < 0;
  }
  return a < b;
}
// bitonic sort of idx[0..net) (entry indices, -1 sorts last) under tk_less; the first
// ORDER BY column travels as an order-preserving key so most comparisons stay in smem
__device__ void tk_sort(const KCompact& k, const KSort& s, long long* idx, unsigned long long* pk, int net) {
  const int c0 = s.norder > 0 ? s.ocol[0] : 0;
  const bool d0 = s.norder > 0 && s.odesc[0];
  for (int i = threadIdx.x; i < net; i += blockDim.x) {
    unsigned long long t = ~0ull;
    if (idx[i] >= 0) {
      const long long v = tk_col(k, idx[i], c0);
      t = s.isf[c0] ? (v < 0 ? ~(unsigned long long)v : (unsigned long long)v ^ 0x8000000000000000ull)
                    : (unsigned long long)v ^ 0x8000000000000000ull;
      if (d0) t = ~t;
      if (s.norder == 0 && s.nkeys == 0) t = 0;
    }
    pk[i] = t;
  }
  __syncthreads();
  for (int kk = 2; kk <= net; kk <<= 1) {
    for (int j = kk >> 1; j > 0; j >>= 1) {
      for (int i = threadIdx.x; i < net; i += blockDim.x) {
        const int l = i ^ j;
        if (l > i) {
          const long long a = idx[i], b = idx[l];
          const unsigned long long ka = pk[i], kb = pk[l];
          const bool up = (i & kk) == 0;
          const bool b_lt_a = kb != ka ? kb < ka : tk_less(k, s, b, a);
          const bool a_lt_b = kb != ka ? ka < kb : tk_less(k, s, a, b);
          if (up ? b_lt_a : a_lt_b) { idx[i] = b; idx[l] = a; pk[i] = kb; pk[l] = ka; }
        }
      }
      __syncthreads();
    }
  }
}
// primary sort key of a live entry: order-preserving image of the first ORDER BY column
// (or the first group key), ascending = the result order
__device__ __forceinline__ unsigned long long tk_pk(const KCompact& k, const KSort& s, long long g) {
  if (s.norder == 0 && s.nkeys == 0) return 0;
  const int c0 = s.norder > 0 ? s.ocol[0] : 0;
  const long long v = tk_col(k, g, c0);
  unsigned long long t = s.isf[c0] ? (v < 0 ? ~(unsigned long long)v : (unsigned long long)v ^ 0x8000000000000000ull)
                                   : (unsigned long long)v ^ 0x8000000000000000ull;
  return (s.norder > 0 && s.odesc[0]) ? ~t : t;
}
// radix-select state: [0] min pk, [1] max pk, [2] shift, [3] selected bin, [4] candidates, [5] overflow
constexpr int TK_BINS = 4096;
constexpr int TK_CAND = 16384;
constexpr int TK_U = 4;  // table entries per thread and round in the full-table passes
// pass 1: min / max primary key, qualifying rows, live groups
__global__ void __launch_bounds__(256) hq_topk_minmax_kernel(const __grid_constant__ KTopK q, unsigned long long* sel,
                                                             unsigned long long* bmin) {
  const KCompact& k = q.k;
  unsigned long long mn = ~0ull, mx = 0, qs = 0, ls = 0;
  // TK_U entries per thread and round, their loads issued together (one entry at a time
  // left each thread waiting on two dependent loads per entry: ~1 TB/s over the table)
  const long long st = (long long)gridDim.x * blockDim.x;
  for (long long g0 = blockIdx.x * (long long)blockDim.x + threadIdx.x; g0 < k.ngroups; g0 += TK_U * st) {
    bool live[TK_U];
#pragma unroll
    for (int u = 0; u < TK_U; ++u) live[u] = g0 + u * st < k.ngroups && tk_live(k, g0 + u * st);
#pragma unroll
    for (int u = 0; u < TK_U; ++u) {
      if (!live[u]) continue;
      const long long g = g0 + u * st;
      const unsigned long long pk = tk_pk(k, q.s, g);
      mn = pk < mn ? pk : mn;
      mx = pk > mx ? pk : mx;
      qs += (unsigned long long)tk_entry(k, g)[0];
      ++ls;
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const unsigned long long a = __shfl_xor_sync(0xffffffffu, mn, o), b = __shfl_xor_sync(0xffffffffu, mx, o);
    mn = a < mn ? a : mn;
    mx = b > mx ? b : mx;
    qs += __shfl_xor_sync(0xffffffffu, qs, o);
    ls += __shfl_xor_sync(0xffffffffu, ls, o);
  }
  // one set of atomics per block, not per warp (same-address atomics serialise: ~9 K
  // warps on four words took most of the kernel's 24 us at TPC-H Q3 SF30)
  __shared__ unsigned long long red[4][8];
  const int w = threadIdx.x >> 5;
  if ((threadIdx.x & 31) == 0) {
    red[0][w] = mn;
    red[1][w] = mx;
    red[2][w] = qs;
    red[3][w] = ls;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    for (int i = 1; i < (int)(blockDim.x >> 5); ++i) {
      mn = red[0][i] < mn ? red[0][i] : mn;
      mx = red[1][i] > mx ? red[1][i] : mx;
      qs += red[2][i];
      ls += red[3][i];
    }
    if (bmin) bmin[blockIdx.x] = ls ? mn : ~0ull;  // the block's smallest key (threshold select)
    if (ls) {
      atomicMin(sel + 0, mn);
      atomicMax(sel + 1, mx);
      atomicAdd(q.stats + 1, qs);
      atomicAdd(q.stats + 3, ls);
    }
  }
}
// threshold select (one block, replaces the histogram pass when every block's share of
// the table times k fits the candidate buffer): a 2,048-bin histogram of the blocks'
// smallest keys over their own [min, max] and a scan give the bin b of the k-th smallest
// minimum; tau = b's upper edge.  At least k entries have a key <= tau (k blocks' minima),
// so the top k all do; entries <= tau come only from blocks whose minimum is <= tau -- the
// k - 1 below b's and those in b (the candidate buffer's overflow flag sends a crowded bin
// the long way).
constexpr int TK_TAU_MAX = TK_BINS * 4 / 8;  // block minima held in the histogram's space
__global__ void __launch_bounds__(1024) hq_topk_tau_kernel(const unsigned long long* bmin, int n, int keep,
                                                          unsigned long long* sel) {
  __shared__ unsigned h[TK_TAU_MAX];
  __shared__ unsigned long long rmn[32], rmx[32];
  __shared__ unsigned part[32];
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  unsigned long long v[2], mn = ~0ull, mx = 0;
  for (int i = 0; i < 2; ++i) {
    const int x = tid * 2 + i;
    v[i] = x < n ? bmin[x] : ~0ull;
    h[x] = 0;
    if (v[i] != ~0ull) { mn = v[i] < mn ? v[i] : mn; mx = v[i] > mx ? v[i] : mx; }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const unsigned long long a = __shfl_xor_sync(0xffffffffu, mn, o), b = __shfl_xor_sync(0xffffffffu, mx, o);
    mn = a < mn ? a : mn;
    mx = b > mx ? b : mx;
  }
  if (lane == 0) { rmn[w] = mn; rmx[w] = mx; }
  __syncthreads();
  mn = rmn[lane];
  mx = rmx[lane];
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const unsigned long long a = __shfl_xor_sync(0xffffffffu, mn, o), b = __shfl_xor_sync(0xffffffffu, mx, o);
    mn = a < mn ? a : mn;
    mx = b > mx ? b : mx;
  }
  if (mn > mx) {  // no live entry
    if (tid == 0) { sel[6] = 0; sel[7] = 1; }
    return;
  }
  int sh = 0;
  while (sh < 63 && ((mx - mn) >> sh) >= (unsigned long long)TK_TAU_MAX) ++sh;
  for (int i = 0; i < 2; ++i)
    if (v[i] != ~0ull) atomicAdd(&h[(v[i] - mn) >> sh], 1u);
  __syncthreads();
  const unsigned c0 = h[tid * 2], c1 = h[tid * 2 + 1], t = c0 + c1;
  unsigned incl = t;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const unsigned x = __shfl_up_sync(0xffffffffu, incl, o);
    if (lane >= o) incl += x;
  }
  if (lane == 31) part[w] = incl;
  __syncthreads();
  if (w == 0) {
    const unsigned pv = part[lane];
    unsigned iv = pv;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const unsigned x = __shfl_up_sync(0xffffffffu, iv, o);
      if (lane >= o) iv += x;
    }
    part[lane] = iv - pv;
  }
  __syncthreads();
  const unsigned before = part[w] + incl - t;  // minima in the bins below this thread's two
  int b = -1;
  if (before < (unsigned)keep && before + c0 >= (unsigned)keep) b = tid * 2;
  else if (before + c0 < (unsigned)keep && before + t >= (unsigned)keep) b = tid * 2 + 1;
  if (tid == blockDim.x - 1 && before + t < (unsigned)keep) {  // fewer than k blocks hold entries: all of them
    sel[6] = ~0ull;
    sel[7] = 1;
  }
  if (b >= 0) {  // the bin of the k-th smallest minimum
    const unsigned long long top = mn + ((((unsigned long long)b + 1) << sh) - 1);
    sel[6] = top < mx && top >= mn ? top : mx;
    sel[7] = 1;  // collect takes key <= sel[6]
  }
}
__device__ __forceinline__ int tk_bin(unsigned long long pk, const unsigned long long* sel) {
  return (int)((pk - sel[0]) >> sel[2]);
}
// pass 2: histogram of the primary keys over TK_BINS bins spanning [min, max]
__global__ void __launch_bounds__(256) hq_topk_hist_kernel(const __grid_constant__ KTopK q, const unsigned long long* sel,
                                                           unsigned* hist) {
  __shared__ unsigned h[TK_BINS];
  for (int i = threadIdx.x; i < TK_BINS; i += blockDim.x) h[i] = 0;
  __syncthreads();
  const KCompact& k = q.k;
  const long long st = (long long)gridDim.x * blockDim.x;
  if (sel[0] <= sel[1])
    for (long long g0 = blockIdx.x * (long long)blockDim.x + threadIdx.x; g0 < k.ngroups; g0 += TK_U * st) {
      bool live[TK_U];
#pragma unroll
      for (int u = 0; u < TK_U; ++u) live[u] = g0 + u * st < k.ngroups && tk_live(k, g0 + u * st);
#pragma unroll
      for (int u = 0; u < TK_U; ++u)
        if (live[u]) atomicAdd(&h[tk_bin(tk_pk(k, q.s, g0 + u * st), sel)], 1u);
    }
  __syncthreads();
  for (int i = threadIdx.x; i < TK_BINS; i += blockDim.x)
    if (h[i]) atomicAdd(hist + i, h[i]);
}
// bins of 2^shift keys: TK_BINS bins cover [min, max]
__global__ void hq_topk_shift_kernel(unsigned long long* sel) {
  const unsigned long long span = sel[0] <= sel[1] ? sel[1] - sel[0] : 0;
  int sh = 0;
  while (sh < 63 && (span >> sh) >= (unsigned long long)TK_BINS) ++sh;
  sel[2] = (unsigned long long)sh;
}
// pass 3 (one block): the bin holding the k-th smallest key; every entry of a lower bin
// is in the top k, the k-th one's bin supplies the rest
__global__ void hq_topk_select_kernel(const unsigned* hist, int keep, unsigned long long* sel) {
  __shared__ unsigned part[32];
  const int tid = threadIdx.x;  // 1024 threads x 4 bins
  unsigned c[4], t = 0;
  for (int i = 0; i < 4; ++i) { c[i] = hist[tid * 4 + i]; t += c[i]; }
  unsigned incl = t;
  const int lane = tid & 31, w = tid >> 5;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const unsigned x = __shfl_up_sync(0xffffffffu, incl, o);
    if (lane >= o) incl += x;
  }
  if (lane == 31) part[w] = incl;
  __syncthreads();
  if (w == 0) {
    unsigned v = part[lane], iv = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const unsigned x = __shfl_up_sync(0xffffffffu, iv, o);
      if (lane >= o) iv += x;
    }
    part[lane] = iv - v;
  }
  __syncthreads();
  unsigned before = part[w] + incl - t;
  for (int i = 0; i < 4; ++i) {
    if (before < (unsigned)keep && before + c[i] >= (unsigned)keep) sel[3] = (unsigned long long)(tid * 4 + i);
    before += c[i];
  }
  if (tid == blockDim.x - 1 && before < (unsigned)keep) sel[3] = TK_BINS - 1;  // fewer live groups than k: all
}
// pass 4: the candidates -- every live entry in the selected bin or below
__global__ void __launch_bounds__(256) hq_topk_collect_kernel(const __grid_constant__ KTopK q, unsigned long long* sel) {
  const KCompact& k = q.k;
  if (sel[0] > sel[1]) return;
  const int bstar = (int)sel[3];
  const bool tau = sel[7] != 0;
  const unsigned long long tv = sel[6];
  const int lane = threadIdx.x & 31;
  // warp-uniform trip count: one atomic per warp and round claims the warp's candidates
  for (long long b0 = (blockIdx.x * (long long)blockDim.x + threadIdx.x) & ~31ll; b0 < k.ngroups;
       b0 += (long long)gridDim.x * blockDim.x) {
    const long long g = b0 + lane;
    bool take = g < k.ngroups && tk_live(k, g);
    if (take) {
      const unsigned long long pk = tk_pk(k, q.s, g);
      take = tau ? pk <= tv : tk_bin(pk, sel) <= bstar;
    }
    const unsigned bal = __ballot_sync(0xffffffffu, take);
    if (!bal) continue;
    unsigned long long base = 0;
    if (lane == 0) base = atomicAdd(sel + 4, (unsigned long long)__popc(bal));
    base = __shfl_sync(0xffffffffu, base, 0);
    if (!take) continue;
    const unsigned long long i = base + __popc(bal & ((1u << lane) - 1u));
    if (i < (unsigned long long)TK_CAND) q.cand[i] = (int)g;
    else sel[5] = 1;  // overflow: the host finalizes the long way
  }
}
__global__ void __launch_bounds__(1024) hq_topk2_kernel(const __grid_constant__ KTopK q, const unsigned long long* sel) {
  const int ncand = sel[5] ? 0 : (int)(sel[4] < (unsigned long long)TK_CAND ? sel[4] : (unsigned long long)TK_CAND);
  __shared__ long long idx[SORT_CHUNK];
  __shared__ unsigned long long pk[SORT_CHUNK];
  __shared__ int err_s;
  const KCompact& k = q.k;
  if (threadIdx.x == 0) err_s = 0;
  // candidates in rounds of SORT_CHUNK - keep, the running top-k in idx[0..keep)
  const int chunk = SORT_CHUNK - q.keep;
  for (int i = threadIdx.x; i < q.keep; i += blockDim.x) idx[i] = -1;
  for (int c0 = 0; c0 < ncand; c0 += chunk) {
    // the smallest network that holds the running top-k and this round's candidates
    const int m = q.keep + (ncand - c0 < chunk ? ncand - c0 : chunk);
    int net = 32;
    while (net < m) net <<= 1;
    __syncthreads();
    for (int i = threadIdx.x; i < net - q.keep; i += blockDim.x) idx[q.keep + i] = c0 + i < ncand ? q.cand[c0 + i] : -1;
    __syncthreads();
    tk_sort(k, q.s, idx, pk, net);
  }
  __syncthreads();
  const int nc = k.nkeys + k.naggs;
  for (int i = threadIdx.x; i < q.keep; i += blockDim.x) {
    const long long g = idx[i];
    if (g < 0) continue;
    for (int c = 0; c < nc; ++c) q.res[c][i] = tk_col(k, g, c);
    for (int a = 0; a < k.naggs; ++a) {
      const long long v = tk_entry(k, g)[1 + a];
      if ((k.agg_fn[a] == HQ_AGG_SUM || k.agg_fn[a] == HQ_AGG_AVG) && (v >= (1LL << 62) || v <= -(1LL << 62)))
        atomicOr(&err_s, HQF_OVERFLOW);
    }
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    const unsigned long long live = q.stats[3];
    q.stats[0] = live < (unsigned long long)q.keep ? live : (unsigned long long)q.keep;
    q.stats[2] = (unsigned long long)err_s;
    q.stats[5] = sel[5];  // candidate overflow
    int e_ = *q.pipe_err;
    for (int i = 0; i < q.nhash; ++i) e_ |= *(volatile const int*)q.hash_err[i];
    q.stats[4] = (unsigned long long)(unsigned)e_;
  }
}

// ---- small dense results (SSB/TPC-H aggregates: <= 4,375 groups): compaction,
// AVG, ORDER BY and LIMIT in ONE block, rows staged to the host with the fault
// bits in the same copy -- one launch and one host sync per finalize.
constexpr int SMALL_FIN = 8192;  // (SSB Q3.1 declares 4,375 groups)
constexpr int FIN_THREADS = 1024;
struct KSmall {
  KCompact k;                 // k.out: row-major-by-column scratch, capacity ngroups
  KSort s;                    // over k.out
  long long limit;            // <= 0: all rows
  long long* res[MAXRC];      // final columns
  unsigned long long* stats;  // [0] rows kept, [1] qualifying, [2] fault bits, [3] rows before LIMIT, [4] pipeline faults
  const int* pipe_err;        // the pipeline's fault word (copied into stats[4])
  const int* hash_err[8];     // fault words of the probed tables' builds (ORed into stats[4])
  int nhash;
};
constexpr int SMALL_STAGE = 1792;  // int64 cells of shared result columns (48-KB static limit)
__global__ void __launch_bounds__(FIN_THREADS) hq_finalize_small_kernel(const __grid_constant__ KSmall q) {
  __shared__ int idx[SMALL_FIN];
  __shared__ long long sstage[SMALL_STAGE];
  __shared__ long long* scol[MAXRC];
  __shared__ int wsum[32];
  __shared__ int base, tot;
  __shared__ unsigned long long qual_s;
  __shared__ int err_s;
  const KCompact& k = q.k;
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  if (tid == 0) { base = 0; qual_s = 0; err_s = 0; }
  __syncthreads();
  // 1. ordered compaction of the non-empty groups (block scan of ballots)
  for (long long g0 = 0; g0 < k.ngroups; g0 += FIN_THREADS) {
    const long long g = g0 + tid;
    const bool ne = g < k.ngroups && (k.scalar || k.gtab[g * k.vwords] != 0);
    const unsigned bal = __ballot_sync(0xffffffffu, ne);
    if (lane == 0) wsum[w] = __popc(bal);
    __syncthreads();
    if (w == 0) {
      const int v = wsum[lane];
      int incl = v;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const int t = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += t;
      }
      wsum[lane] = incl - v;
      if (lane == 31) tot = incl;
    }
    __syncthreads();
    if (ne) idx[base + wsum[w] + __popc(bal & ((1u << lane) - 1u))] = (int)g;
    __syncthreads();
    if (tid == 0) base += tot;
    __syncthreads();
  }
  const int n = base;
  // result columns in shared memory when they fit (SSB / TPC-H aggregates: tens to
  // hundreds of rows): the sort's comparisons then read shared memory, not the scratch
  // columns in global memory -- a round trip per network step (SSB Q4.1: 20 -> ~5 us)
  const int ncol = k.nkeys + k.naggs;
  const bool stg = (long long)n * ncol <= SMALL_STAGE;
  if (tid < MAXRC) scol[tid] = tid < ncol ? (stg ? sstage + (long long)tid * n : k.out[tid]) : nullptr;
  __syncthreads();
  // 2. one row per group: decoded keys, aggregates, AVG, int64 guard
  unsigned long long qsum = 0;
  bool big = false;
  for (int i = tid; i < n; i += FIN_THREADS) {
    const long long g = idx[i];
    const long long* e = k.gtab + g * k.vwords;
    const long long cnt = e[0];
    qsum += (unsigned long long)cnt;
    if (k.ngroups <= 0xFFFFFFFFll) {  // 32-bit division (a 64-bit one is a long software sequence)
      for (int c = 0; c < k.nkeys; ++c)
        scol[c][i] = k.key_min[c] + (long long)(((unsigned)g / (unsigned)k.key_stride[c]) % (unsigned)k.key_card[c]);
    } else {
      for (int c = 0; c < k.nkeys; ++c)
        scol[c][i] = k.key_min[c] + (long long)(((unsigned long long)g / (unsigned long long)k.key_stride[c]) % (unsigned long long)k.key_card[c]);
    }
    for (int a = 0; a < k.naggs; ++a) {
      const long long v = e[1 + a];
      long long* o = scol[k.nkeys + a];
      if (k.agg_fn[a] == HQ_AGG_AVG) {
        const double d = cnt ? (double)v / (double)cnt / k.agg_div[a] : __longlong_as_double(0x7ff8000000000000LL);
        o[i] = __double_as_longlong(d);
      } else {
        o[i] = v;
      }
      if ((k.agg_fn[a] == HQ_AGG_SUM || k.agg_fn[a] == HQ_AGG_AVG) && (v >= (1LL << 62) || v <= -(1LL << 62))) big = true;
    }
  }
  if (qsum) atomicAdd(&qual_s, qsum);
  if (big) atomicOr(&err_s, HQF_OVERFLOW);
  __syncthreads();
  // 3. ORDER BY (+ group keys, row id: a total order) -- bitonic network in shared memory;
  // staged columns are compared through a register copy of the comparison program (column,
  // direction, float flag per step) with shared-memory loads
  __shared__ int ord[HQ_MAX_ORDER + HQ_MAX_KEYS];
  const int nord = q.s.norder + q.s.nkeys;
  if (tid < q.s.norder) {
    const int c = q.s.ocol[tid];
    ord[tid] = c | (q.s.odesc[tid] ? 0x100 : 0) | (q.s.isf[c] ? 0x200 : 0);
  } else if (tid < nord) {
    const int c = tid - q.s.norder;
    ord[tid] = c | (q.s.isf[c] ? 0x200 : 0);
  }
  int net = 32;
  while (net < n) net <<= 1;
  for (int i = tid; i < net; i += FIN_THREADS) idx[i] = i < n ? i : -1;
  __syncthreads();
  // only the warps the network needs take part (a named barrier of net threads per step, a
  // warp barrier for 32): a 1,024-thread barrier per step cost ~1,300 cycles (SSB Q4.1)
  const int sT = net < FIN_THREADS ? net : FIN_THREADS;
  // up to 64 staged rows: rank by counting -- row i's position is the number of rows
  // before it in the total order (distinct: the row id breaks ties), n comparisons per
  // thread and one barrier instead of log^2 network steps (SSB Q4.1: 35 rows, 17.9 -> 15.9 us;
  // at 150 rows the network is faster: SSB Q3.1 34.7 vs 59.1 us, measured)
  const bool rank_sort = stg && n <= 64 && n > 1 && (q.s.norder > 0 || k.nkeys > 0);
  if (rank_sort) {
    __syncthreads();
    if (tid < n) {
      int r = 0;
      for (int j = 0; j < n; ++j) r += row_less_st(sstage, n, ord, nord, j, tid) ? 1 : 0;
      idx[r] = tid;
    }
  } else if (n > 1 && (q.s.norder > 0 || k.nkeys > 0) && tid < sT) {
    for (int kk = 2; kk <= net; kk <<= 1) {
      for (int j = kk >> 1; j > 0; j >>= 1) {
        for (int i = tid; i < net; i += sT) {
          const int l = i ^ j;
          if (l > i) {
            const int a = idx[i], b = idx[l];
            const bool up = (i & kk) == 0;
            const bool sw = stg ? (up ? row_less_st(sstage, n, ord, nord, b, a) : row_less_st(sstage, n, ord, nord, a, b))
                                : (up ? row_less_at(q.s, scol, b, a) : row_less_at(q.s, scol, a, b));
            if (sw) { idx[i] = b; idx[l] = a; }
          }
        }
        if (sT > 32) asm volatile("bar.sync 1, %0;" ::"r"(sT) : "memory");
        else __syncwarp();
      }
    }
  }
  __syncthreads();
  // 4. LIMIT + gather into the result columns
  const int nf = q.limit > 0 && q.limit < n ? (int)q.limit : n;
  for (int c = 0; c < k.nkeys + k.naggs; ++c)
    for (int i = tid; i < nf; i += FIN_THREADS) q.res[c][i] = scol[c][idx[i]];
  if (tid == 0) {
    q.stats[0] = (unsigned long long)nf;
    q.stats[1] = qual_s;
    q.stats[2] = (unsigned long long)err_s;
    q.stats[3] = (unsigned long long)n;
    int e_ = *q.pipe_err;
    for (int i = 0; i < q.nhash; ++i) e_ |= *(volatile const int*)q.hash_err[i];
    q.stats[4] = (unsigned long long)(unsigned)e_;
  }
}

// smallest power-of-two bitonic network (>= 32) that holds n rows
int net_for(long long n) {
  int v = 32;
  while (v < n && v < SORT_CHUNK) v <<= 1;
  return v;
}

int grid_for(hq_ctx* ctx, long long n) {
  return (int)std::max<long long>(1, std::min<long long>((n + 255) / 256, (long long)ctx->num_sms * 8));
}

}  // namespace

// per-context pinned host staging (small results, column statistics)
void* pinned_staging(hq_ctx* ctx, size_t bytes) {
  if (ctx->pinned_bytes < bytes) {
    if (ctx->pinned) HQ_CUDA(cudaFreeHost(ctx->pinned));
    ctx->pinned = nullptr;
    ctx->pinned_bytes = 0;
    const size_t want = std::max<size_t>(bytes, 1 << 20);
    HQ_CUDA(cudaHostAlloc(&ctx->pinned, want, cudaHostAllocDefault));
    ctx->pinned_bytes = want;
  }
  return ctx->pinned;
}

static bool decode_small(hq_result* r, const char* h, int64_t rcap, int nc);
namespace {
// one launch, one sync: fault bits + finalized rows come back together
bool finalize_small(hq_ctx* ctx, hq_result* r) {
  const hq_plan& P = r->plan;
  {  // more probed tables than the kernel reads fault words of: the syncing check first
    int nh = 0;
    for (hq_hash* hh : r->hashes) nh += (hh->dstate.p && !hh->checked) ? 1 : 0;
    if (nh > 8) hq_check_result_faults(ctx, r);
  }
  const int nk = P.nkeys, na = P.naggs, nc = nk + na;
  if (P.norder < 0 || P.norder > HQ_MAX_ORDER) HQ_THROW(HQ_ERR_UNSUPPORTED, "plan: 0..4 ORDER BY columns");
  for (int i = 0; i < P.norder; ++i)
    if (P.order_col[i] < 0 || P.order_col[i] >= nc) HQ_THROW(HQ_ERR_ARG, "plan: ORDER BY column out of range");
  const int64_t ng = std::max<int64_t>(r->ngroups, 1);
  // columns start 16-B aligned (an even row count): the result may become the fact
  // table of a later pipeline (hq_result_as_table), whose stage loads need it
  const int64_t rcap = ((P.limit > 0 ? std::min<int64_t>(ng, P.limit) : ng) + 1) / 2 * 2;
  std::vector<DevBuf> cols;
  for (int c = 0; c < nc; ++c) cols.emplace_back(ctx, (size_t)ng * 8);
  // [stats: 64 B][column 0: rcap rows][column 1]... -- one D2H copy brings it all back
  const size_t body = (size_t)nc * rcap * 8;
  DevBuf pack(ctx, 64 + body);
  KSmall q{};
  KCompact& k = q.k;
  k.gtab = r->gtab.as<long long>();
  k.ngroups = r->ngroups;
  k.vwords = r->vwords;
  k.nkeys = nk;
  k.naggs = na;
  k.scalar = nk == 0;
  int64_t st = 1;
  for (int i = nk - 1; i >= 0; --i) {
    k.key_stride[i] = st;
    st *= P.key_card[i];
  }
  for (int i = 0; i < nk; ++i) {
    k.key_min[i] = P.key_min[i];
    k.key_card[i] = P.key_card[i];
    r->types[i] = HQ_I64;
  }
  for (int a = 0; a < na; ++a) {
    k.agg_fn[a] = (uint8_t)P.agg_fn[a];
    double d = 1.0;
    for (int s2 = 0; s2 < P.agg_scale[a]; ++s2) d *= 10.0;
    k.agg_div[a] = d;
    r->types[nk + a] = P.agg_fn[a] == HQ_AGG_AVG ? HQ_F64 : HQ_I64;
  }
  for (int c = 0; c < nc; ++c) {
    k.out[c] = cols[c].as<long long>();
    q.s.col[c] = cols[c].as<long long>();
    q.s.isf[c] = r->types[c] == HQ_F64;
    q.res[c] = (long long*)(pack.as<char>() + 64 + (size_t)c * rcap * 8);
  }
  q.s.norder = P.norder;
  for (int i = 0; i < P.norder; ++i) {
    q.s.ocol[i] = P.order_col[i];
    q.s.odesc[i] = P.order_desc[i];
  }
  q.s.nkeys = nk;
  q.limit = P.limit;
  q.stats = pack.as<unsigned long long>();
  q.pipe_err = (const int*)(r->dstate.as<char>() + 8);
  q.nhash = 0;
  for (hq_hash* hh : r->hashes)
    if (hh->dstate.p && !hh->checked && q.nhash < 8) q.hash_err[q.nhash++] = hh->dstate.as<int>();
  ctx->launches++;
  hq_finalize_small_kernel<<<1, FIN_THREADS, 0, ctx->stream>>>(q);
  HQ_CUDA(cudaGetLastError());
  if (ctx->capturing) {
    // graph capture: the rows land in the result's own pinned staging at every launch
    // and are decoded on the host after it (hq_graph_launch -> hq_decode_captured)
    if (r->stage_host) HQ_THROW(HQ_ERR_STATE, "result finalized twice in one capture");
    HQ_CUDA(cudaHostAlloc(&r->stage_host, 64 + body, cudaHostAllocDefault));
    HQ_CUDA(cudaMemcpyAsync(r->stage_host, pack.p, 64 + body, cudaMemcpyDeviceToHost, ctx->stream));
    r->stage_rcap = rcap;
    r->ncols = nc;
    r->rescol.assign((size_t)nc, nullptr);
    for (int c = 0; c < nc; ++c) r->rescol[c] = pack.as<char>() + 64 + (size_t)c * rcap * 8;
    r->respack = std::move(pack);
    r->capture_retain(ctx);
    ctx->cap_results.push_back(r);
    r->finalized = true;  // for this capture; hq_graph_launch re-opens it
    return true;
  }
  char* h = (char*)pinned_staging(ctx, 64 + body);
  HQ_CUDA(cudaMemcpyAsync(h, pack.p, 64 + body, cudaMemcpyDeviceToHost, ctx->stream));
  HQ_CUDA(cudaStreamSynchronize(ctx->stream));
  if (!decode_small(r, h, rcap, nc)) return false;  // faults: the caller checks (and may re-run), then retries
  r->rescol.assign((size_t)nc, nullptr);
  for (int c = 0; c < nc; ++c) r->rescol[c] = pack.as<char>() + 64 + (size_t)c * rcap * 8;
  r->respack = std::move(pack);
  return true;
}
}  // namespace

// finalize_small's host part: stats + rows staged in h (layout of KSmall)
static bool decode_small(hq_result* r, const char* h, int64_t rcap, int nc) {
  const unsigned long long* sv = (const unsigned long long*)h;
  if (!r->checked && sv[4]) return false;
  r->checked = true;
  if (sv[2] & HQF_OVERFLOW) HQ_THROW(HQ_ERR_OVERFLOW, "aggregate exceeds the int64 guard (|v| >= 2^62)");
  const int64_t nf = (int64_t)sv[0];
  r->qualifying = (int64_t)sv[1];
  r->ncols = nc;
  r->host_rows.assign((size_t)nc * nf, 0);
  for (int c = 0; c < nc; ++c)
    std::memcpy(r->host_rows.data() + (size_t)c * nf, h + 64 + (size_t)c * rcap * 8, (size_t)nf * 8);
  r->host_ready = true;
  r->nrows = nf;
  r->finalized = true;
  return true;
}

void hq_decode_captured(hq_ctx* ctx, hq_result* r) {
  if (!r->stage_host) HQ_THROW(HQ_ERR_STATE, "result has no capture staging");
  if (r->stage_topk && ((const unsigned long long*)r->stage_host)[5])
    HQ_THROW(HQ_ERR_STATE, "captured query: more ties at the LIMIT boundary than the top-k selection holds "
                           "(run the query eagerly)");
  if (decode_small(r, (const char*)r->stage_host, r->stage_rcap, r->ncols)) return;
  // a fault (pipeline, or a probed table's build): raised by the syncing check; the
  // re-runnable ones cannot occur in a dense small result
  r->checked = false;
  hq_check_result_faults(ctx, r);
  HQ_THROW(HQ_ERR_STATE, "captured query: unexpected re-runnable fault");
}

// ORDER BY ... LIMIT k (k <= TOPK_MAX) of a large group table: two launches, one host
// copy (rows + statistics), no compaction of the whole table (hq_topk1/2_kernel).
static bool finalize_topk(hq_ctx* ctx, hq_result* r) {
  const hq_plan& P = r->plan;
  const int nk = P.nkeys, na = P.naggs, nc = nk + na;
  if (P.norder < 0 || P.norder > HQ_MAX_ORDER) HQ_THROW(HQ_ERR_UNSUPPORTED, "plan: 0..4 ORDER BY columns");
  for (int i = 0; i < P.norder; ++i)
    if (P.order_col[i] < 0 || P.order_col[i] >= nc) HQ_THROW(HQ_ERR_ARG, "plan: ORDER BY column out of range");
  KTopK q{};
  KCompact& k = q.k;
  k.gtab = r->gtab.as<long long>();
  k.ngroups = r->ngroups;
  k.vwords = r->vwords;
  k.hash = r->gmode == GM_HASH;
  k.nkeys = nk;
  k.naggs = na;
  int64_t st = 1;
  for (int i = nk - 1; i >= 0; --i) {
    k.key_stride[i] = st;
    st *= P.key_card[i];
  }
  for (int i = 0; i < nk; ++i) {
    k.key_min[i] = P.key_min[i];
    k.key_card[i] = P.key_card[i];
    r->types[i] = HQ_I64;
  }
  for (int a = 0; a < na; ++a) {
    k.agg_fn[a] = (uint8_t)P.agg_fn[a];
    double d = 1.0;
    for (int s2 = 0; s2 < P.agg_scale[a]; ++s2) d *= 10.0;
    k.agg_div[a] = d;
    r->types[nk + a] = P.agg_fn[a] == HQ_AGG_AVG ? HQ_F64 : HQ_I64;
  }
  for (int c = 0; c < nc; ++c) q.s.isf[c] = r->types[c] == HQ_F64;
  q.s.norder = P.norder;
  for (int i = 0; i < P.norder; ++i) {
    q.s.ocol[i] = P.order_col[i];
    q.s.odesc[i] = P.order_desc[i];
  }
  q.s.nkeys = nk;
  q.keep = (int)P.limit;
  const int64_t rcap = (P.limit + 1) / 2 * 2;
  const size_t body = (size_t)nc * rcap * 8;
  DevBuf pack(ctx, 64 + body);
  HQ_CUDA(cudaMemsetAsync(pack.p, 0, 64, ctx->stream));
  q.stats = pack.as<unsigned long long>();
  for (int c = 0; c < nc; ++c) q.res[c] = (long long*)(pack.as<char>() + 64 + (size_t)c * rcap * 8);
  DevBuf cand(ctx, (size_t)TK_CAND * 4 + 16);
  q.cand = cand.as<int>();
  // selection state + histogram: [0] min (all ones) [1] max [2] shift [3] bin [4] count [5] overflow, then the bins
  DevBuf selb(ctx, 64 + (size_t)TK_BINS * 4);
  unsigned long long* sel = selb.as<unsigned long long>();
  HQ_CUDA(cudaMemsetAsync(selb.p, 0, 64 + (size_t)TK_BINS * 4, ctx->stream));
  HQ_CUDA(cudaMemsetAsync(selb.p, 0xFF, 8, ctx->stream));
  q.pipe_err = (const int*)(r->dstate.as<char>() + 8);
  for (hq_hash* hh : r->hashes)
    if (hh->dstate.p && !hh->checked && q.nhash < 8) q.hash_err[q.nhash++] = hh->dstate.as<int>();
  const int grid = grid_for(ctx, r->ngroups);
  // threshold select (one table pass less) when k x a block's share of the table fits the
  // candidate buffer: TPC-H Q3 SF30, k = 10 over 2^20 entries; HQ_TOPK_RADIX=1 forces the
  // histogram select (A/B)
  const int64_t per_block = (r->ngroups + (int64_t)grid * 256 - 1) / ((int64_t)grid * 256) * 256;  // minmax's share
  const bool tau = grid <= TK_TAU_MAX && q.keep <= grid && (int64_t)q.keep * per_block <= TK_CAND && !getenv("HQ_TOPK_RADIX");
  unsigned long long* bmin = tau ? (unsigned long long*)(selb.as<char>() + 64) : nullptr;
  ctx->launches += tau ? 4 : 6;
  hq_topk_minmax_kernel<<<grid, 256, 0, ctx->stream>>>(q, sel, bmin);
  if (tau) {
    hq_topk_tau_kernel<<<1, 1024, 0, ctx->stream>>>(bmin, grid, q.keep, sel);
  } else {
    hq_topk_shift_kernel<<<1, 1, 0, ctx->stream>>>(sel);
    hq_topk_hist_kernel<<<grid, 256, 0, ctx->stream>>>(q, sel, (unsigned*)(selb.as<char>() + 64));
    hq_topk_select_kernel<<<1, 1024, 0, ctx->stream>>>((const unsigned*)(selb.as<char>() + 64), q.keep, sel);
  }
  hq_topk_collect_kernel<<<grid, 256, 0, ctx->stream>>>(q, sel);
  hq_topk2_kernel<<<1, 1024, 0, ctx->stream>>>(q, sel);
  HQ_CUDA(cudaGetLastError());
  if (ctx->capturing) {  // as finalize_small: the rows land in the result's pinned staging per launch
    if (r->stage_host) HQ_THROW(HQ_ERR_STATE, "result finalized twice in one capture");
    HQ_CUDA(cudaHostAlloc(&r->stage_host, 64 + body, cudaHostAllocDefault));
    HQ_CUDA(cudaMemcpyAsync(r->stage_host, pack.p, 64 + body, cudaMemcpyDeviceToHost, ctx->stream));
    r->stage_rcap = rcap;
    r->stage_topk = true;
    r->ncols = nc;
    r->rescol.assign((size_t)nc, nullptr);
    for (int c = 0; c < nc; ++c) r->rescol[c] = pack.as<char>() + 64 + (size_t)c * rcap * 8;
    r->respack = std::move(pack);
    r->capture_retain(ctx);
    ctx->cap_results.push_back(r);
    r->finalized = true;  // for this capture; hq_graph_launch re-opens it
    return true;
  }
  char* h = (char*)pinned_staging(ctx, 64 + body);
  HQ_CUDA(cudaMemcpyAsync(h, pack.p, 64 + body, cudaMemcpyDeviceToHost, ctx->stream));
  hq_sync(ctx, "a top-k finalize");
  if (((const unsigned long long*)h)[5]) return false;  // the k-th key's bin held too many ties
  if (!decode_small(r, h, rcap, nc)) return false;
  r->rescol.assign((size_t)nc, nullptr);
  for (int c = 0; c < nc; ++c) r->rescol[c] = pack.as<char>() + 64 + (size_t)c * rcap * 8;
  r->respack = std::move(pack);
  return true;
}

// Stable LSD radix sort of the rows by (ORDER BY columns, then the group keys
// ascending): one CUB radix pass per column, least significant first; returns
// the sorted row order in `idx` (n entries).
static void radix_order(hq_ctx* ctx, const hq_plan& P, const std::vector<DevBuf>& cols, const int* types, int64_t n,
                        DevBuf& idx) {
  DevBuf kb[2] = {DevBuf(ctx, (size_t)n * 8), DevBuf(ctx, (size_t)n * 8)};
  DevBuf ib(ctx, (size_t)n * 4);
  idx = DevBuf(ctx, (size_t)n * 4);
  size_t tmp_bytes = 0;
  cub::DeviceRadixSort::SortPairs(nullptr, tmp_bytes, kb[0].as<unsigned long long>(), kb[1].as<unsigned long long>(),
                                  ib.as<int>(), idx.as<int>(), (int)n, 0, 64, ctx->stream);
  DevBuf tmp(ctx, tmp_bytes + 16);
  bool first = true;
  auto pass = [&](int c, int mode, long long kmin, int desc, int bits) {
    ctx->launches++;
    hq_sortkey_kernel<<<grid_for(ctx, n), 256, 0, ctx->stream>>>(cols[c].as<long long>(), first ? nullptr : idx.as<int>(), n,
                                                                 mode, kmin, desc, kb[0].as<unsigned long long>());
    if (first) {
      ctx->launches++;
      hq_iota_kernel<<<grid_for(ctx, n), 256, 0, ctx->stream>>>(ib.as<int>(), n, n);
    } else {
      HQ_CUDA(cudaMemcpyAsync(ib.p, idx.p, (size_t)n * 4, cudaMemcpyDeviceToDevice, ctx->stream));
    }
    size_t tb = tmp_bytes;
    ctx->launches++;
    HQ_CUDA(cub::DeviceRadixSort::SortPairs(tmp.p, tb, kb[0].as<unsigned long long>(), kb[1].as<unsigned long long>(),
                                            ib.as<int>(), idx.as<int>(), (int)n, 0, bits, ctx->stream));
    first = false;
  };
  for (int i = P.nkeys - 1; i >= 0; --i) {  // tie-break: group keys ascending (R7)
    int bits = 1;
    while (bits < 64 && (1ull << bits) < (unsigned long long)P.key_card[i]) ++bits;
    pass(i, 0, P.key_min[i], 0, bits);
  }
  for (int i = P.norder - 1; i >= 0; --i) {
    const int c = P.order_col[i];
    pass(c, types[c] == HQ_F64 ? 2 : 1, 0, P.order_desc[i] ? 1 : 0, 64);
  }
  if (first) {  // no sort column: identity order
    ctx->launches++;
    hq_iota_kernel<<<grid_for(ctx, n), 256, 0, ctx->stream>>>(idx.as<int>(), n, n);
  }
}

void hq_finalize_impl(hq_ctx* ctx, hq_result* r, bool unordered) {
  if (r->finalized) return;
  if (r->sink == HQ_SINK_AGG && r->gmode != GM_HASH && r->ngroups <= SMALL_FIN) {
    if (finalize_small(ctx, r)) return;
    hq_check_result_faults(ctx, r);  // throws, or re-runs the pipeline with more room
    if (finalize_small(ctx, r)) return;
  }
  if (r->sink == HQ_SINK_AGG && r->plan.limit > 0 && r->plan.limit <= TOPK_MAX && r->plan.nkeys > 0 &&
      !getenv("HQ_NO_TOPK")) {
    if (finalize_topk(ctx, r)) return;  // (capturable: rows staged per launch)
    hq_check_result_faults(ctx, r);  // throws, or re-runs the pipeline with a larger group table
    if (finalize_topk(ctx, r)) return;  // (else: too many ties at the k-th key -- the full sort below)
  }
  hq_require_eager(ctx, "the finalize of a large, hash-grouped or materialised result");
  hq_check_result_faults(ctx, r);
  const hq_plan& P = r->plan;
  if (r->sink == HQ_SINK_MATERIALISE) {
    unsigned long long cnt = (unsigned long long)r->checked_counter;  // read by the fault check
    if (r->checked_counter < 0) {
      HQ_CUDA(cudaMemcpyAsync(&cnt, r->dstate.p, 8, cudaMemcpyDeviceToHost, ctx->stream));
      HQ_CUDA(cudaStreamSynchronize(ctx->stream));
    }
    r->qualifying = (int64_t)cnt;
    r->nrows = std::min<int64_t>((int64_t)cnt, r->capacity);
    r->ncols = P.nout;
    for (int j = 0; j < P.nout; ++j) r->types[j] = P.out_type[j];
    r->finalized = true;
    return;
  }
  // ---- AGG: compact
  const int nk = P.nkeys, na = P.naggs, nc = nk + na;
  r->ncols = nc;
  const int64_t cap = std::max<int64_t>(r->ngroups, 1);
  std::vector<DevBuf> cols;
  for (int c = 0; c < nc; ++c) cols.emplace_back(ctx, (size_t)cap * 8);
  DevBuf scratch(ctx, 64);
  HQ_CUDA(cudaMemsetAsync(scratch.p, 0, 64, ctx->stream));
  KCompact k{};
  k.gtab = r->gtab.as<long long>();
  k.ngroups = r->ngroups;
  k.vwords = r->vwords;
  k.hash = r->gmode == GM_HASH;
  k.nkeys = nk;
  k.naggs = na;
  int64_t st = 1;
  for (int i = nk - 1; i >= 0; --i) {
    k.key_stride[i] = st;
    st *= P.key_card[i];
  }
  for (int i = 0; i < nk; ++i) {
    k.key_min[i] = P.key_min[i];
    k.key_card[i] = P.key_card[i];
    r->types[i] = HQ_I64;
  }
  for (int a = 0; a < na; ++a) {
    k.agg_fn[a] = (uint8_t)P.agg_fn[a];
    double d = 1.0;
    for (int s = 0; s < P.agg_scale[a]; ++s) d *= 10.0;
    k.agg_div[a] = d;
    r->types[nk + a] = P.agg_fn[a] == HQ_AGG_AVG ? HQ_F64 : HQ_I64;
  }
  for (int c = 0; c < nc; ++c) k.out[c] = cols[c].as<long long>();
  k.nout = scratch.as<unsigned long long>();
  k.err = (int*)(scratch.as<char>() + 16);
  k.scalar = nk == 0;
  ctx->launches++;
  hq_compact_kernel<<<grid_for(ctx, r->ngroups), 256, 0, ctx->stream>>>(k);
  HQ_CUDA(cudaGetLastError());
  struct { unsigned long long rows, qual; int err; int pad; } st2{};
  HQ_CUDA(cudaMemcpyAsync(&st2, scratch.p, sizeof(st2), cudaMemcpyDeviceToHost, ctx->stream));
  HQ_CUDA(cudaStreamSynchronize(ctx->stream));
  if (st2.err & HQF_OVERFLOW) HQ_THROW(HQ_ERR_OVERFLOW, "aggregate exceeds the int64 guard (|v| >= 2^62)");
  const int64_t n = (int64_t)st2.rows;
  r->qualifying = (int64_t)st2.qual;
  int64_t nfinal = n;
  if (P.limit > 0) nfinal = std::min<int64_t>(nfinal, P.limit);
  // ---- ORDER BY (+ LIMIT)
  // a pure GROUP BY (no ORDER BY, no LIMIT) viewed as a table keeps the group-table order
  const bool sort = (P.norder > 0 || nk > 0) && n > 1 && !(unordered && P.norder == 0 && P.limit <= 0);
  if (sort) {
    KSort s{};
    for (int c = 0; c < nc; ++c) {
      s.col[c] = cols[c].as<long long>();
      s.isf[c] = r->types[c] == HQ_F64;
    }
    if (P.norder < 0 || P.norder > HQ_MAX_ORDER) HQ_THROW(HQ_ERR_UNSUPPORTED, "plan: 0..4 ORDER BY columns");
    s.norder = P.norder;
    for (int i = 0; i < P.norder; ++i) {
      if (P.order_col[i] < 0 || P.order_col[i] >= nc) HQ_THROW(HQ_ERR_ARG, "plan: ORDER BY column out of range");
      s.ocol[i] = P.order_col[i];
      s.odesc[i] = P.order_desc[i];
    }
    s.nkeys = nk;
    DevBuf ia(ctx, (size_t)std::max<int64_t>(n, SORT_CHUNK) * 4 + 16), ib;
    const int* cur = nullptr;  // NULL = identity
    int64_t cur_n = n;
    int* sorted = nullptr;
    if (P.limit > 0 && P.limit <= SORT_CHUNK / 2) {
      // top-k: chunk sorts keep `limit` rows each until one chunk remains
      const int keep = (int)P.limit;
      ib = DevBuf(ctx, (size_t)((n + SORT_CHUNK - 1) / SORT_CHUNK) * keep * 4 + 16);
      int* bufs[2] = {ia.as<int>(), ib.as<int>()};
      int which = 1;
      while (true) {
        const int64_t chunks = (cur_n + SORT_CHUNK - 1) / SORT_CHUNK;
        const int kp = chunks == 1 ? (int)std::min<int64_t>(cur_n, SORT_CHUNK) : keep;
        const int net = chunks == 1 ? net_for(cur_n) : SORT_CHUNK;
        int* dst = bufs[which];
        ctx->launches++;
        hq_chunk_sort_kernel<<<(unsigned)chunks, std::min(1024, net), 0, ctx->stream>>>(s, cur, cur_n, dst, kp, net);
        HQ_CUDA(cudaGetLastError());
        cur = dst;
        cur_n = chunks * kp;
        which ^= 1;
        if (chunks == 1) break;
      }
      sorted = (int*)cur;
    } else if (n <= SORT_CHUNK) {
      ctx->launches++;
      const int net = net_for(n);
      hq_chunk_sort_kernel<<<1, std::min(1024, net), 0, ctx->stream>>>(s, nullptr, n, ia.as<int>(), SORT_CHUNK, net);
      HQ_CUDA(cudaGetLastError());
      sorted = ia.as<int>();
    } else {  // large results: stable LSD radix sort, one CUB pass per sort column
      radix_order(ctx, P, cols, r->types, n, ia);
      HQ_CUDA(cudaGetLastError());
      sorted = ia.as<int>();
    }
    std::vector<DevBuf> out;
    for (int c = 0; c < nc; ++c) {
      out.emplace_back(ctx, (size_t)std::max<int64_t>(nfinal, 1) * 8);
      ctx->launches++;
      hq_gather_kernel<<<grid_for(ctx, nfinal), 256, 0, ctx->stream>>>(cols[c].as<long long>(), sorted, nfinal,
                                                                      out.back().as<long long>());
    }
    HQ_CUDA(cudaGetLastError());
    HQ_CUDA(cudaStreamSynchronize(ctx->stream));  // scratch index buffers are released below
    cols = std::move(out);
  }
  r->rescols = std::move(cols);
  r->rescol.clear();
  for (auto& c : r->rescols) r->rescol.push_back(c.p);
  r->nrows = nfinal;
  r->finalized = true;
}

// ------------------------------------------------------------- fault words
namespace {
constexpr int GF_MAX = 256;
struct KGather {
  const int* w[GF_MAX];
  int nh, nr;
  long long* out;
};
// word k < 16: bit k of any hash's build fault word; word 16 + k: bit k of any
// result's pipeline fault word (hq.h hq_gather_faults)
__global__ void hq_gather_faults_kernel(const __grid_constant__ KGather g) {
  const int k = threadIdx.x;
  int hb = 0, rb = 0;
  for (int i = 0; i < g.nh; ++i) hb |= *(volatile const int*)g.w[i];
  for (int i = 0; i < g.nr; ++i) rb |= *(volatile const int*)g.w[g.nh + i];
  if (k < 16) g.out[k] = (hb >> k) & 1;
  else if (k < 32) g.out[k] = (rb >> (k - 16)) & 1;
}
}  // namespace

void hq_launch_gather_faults(hq_ctx* ctx, const std::vector<const int*>& hw, const std::vector<const int*>& rw,
                             long long* out) {
  if (hw.size() + rw.size() > (size_t)GF_MAX) HQ_THROW(HQ_ERR_UNSUPPORTED, "hq_gather_faults: more than 256 handles");
  KGather g{};
  g.nh = (int)hw.size();
  g.nr = (int)rw.size();
  for (size_t i = 0; i < hw.size(); ++i) g.w[i] = hw[i];
  for (size_t i = 0; i < rw.size(); ++i) g.w[hw.size() + i] = rw[i];
  g.out = out;
  ctx->launches++;
  hq_gather_faults_kernel<<<1, 32, 0, ctx->stream>>>(g);
  HQ_CUDA(cudaGetLastError());
}
