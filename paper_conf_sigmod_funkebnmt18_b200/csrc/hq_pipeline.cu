// hq_pipeline.cu -- the fused pipeline ("compound") kernel of HorseQC on sm_100a.
//
// PAPER.md §5.2 / Fig 12: all phases of a fusion operator -- select,
// join probe, (prefix sum | reduction), project/write -- run in ONE kernel; flags,
// probe payloads and write offsets stay on chip (registers / shared memory).
// §6.1: write offsets and aggregates use *local resolution, global
// propagation* (LRGP): resolve inside the thread group first (warp ballots /
// shuffles, block scan, shared-memory tables), then one global atomic per group.
//
// B200 design:
//  * persistent grid, one CTA per SM, 16 consumer warps + 1 TMA producer warp;
//  * the producer streams the referenced fact columns tile by tile with 1-D TMA
//    bulk copies (cp.async.bulk, L2 evict_first) into an S-stage shared-memory
//    ring guarded by mbarriers (full: tx bytes, empty: one arrive per consumer
//    warp), so HBM reads run ahead of the processing;
//  * each consumer warp owns 32*R consecutive rows of a tile (lane + 32 r) and
//    walks the plan's ops over them: predicates -> per-thread live bit masks,
//    probes -> open-addressing lookups with R independent loads in flight,
//    expressions -> int64 accumulator machine; temporaries live in a per-lane
//    shared-memory region;
//  * sinks: scalar aggregates in registers (B3), grouped aggregates combined per
//    warp (match_any + shuffle reduction) into a shared-memory dense or hash
//    table and merged with global atomics at the end (C3, overflow -> C2),
//    materialisation with a ballot/popc warp scan, a block scan and ONE atomicAdd
//    per block and tile (A3, Fig 25 P:2064-2092 / P:1069-1072).
#include <climits>
#include <cstring>

#include "hq_internal.h"
#include "hq_device.cuh"

namespace hqk {

#define FULLMASK 0xffffffffu

// ----------------------------------------------------------- PTX helpers
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* b, uint32_t tx) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(tx) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n"
      "HQ_WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra HQ_WAIT_%=;\n}\n" ::"r"(smem_u32(b)),
      "r"(parity)  // no suspend-time hint: a long hint let a warp oversleep the phase flip
      : "memory");
}
__device__ __forceinline__ uint64_t policy_evict_first() {
  uint64_t pol;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  return pol;
}
__device__ __forceinline__ void tma_load_1d(void* dst, const void* src, uint32_t bytes, uint64_t* bar,
                                            uint64_t pol) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(pol)
      : "memory");
}
__device__ __forceinline__ void fence_proxy_async() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void consumer_bar(int nw) {  // all consumer warps (not the producer)
  asm volatile("bar.sync 1, %0;" ::"r"(nw * 32) : "memory");
}
__device__ __forceinline__ uint32_t lanemask_lt() {
  uint32_t m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

// ------------------------------------------------------------ reg access
template <int R>
__device__ __forceinline__ void load_rows(const KPlan& p, int reg, const char* stage, const char* tmp,
                                          int row0, long long (&v)[R]) {
  const KReg d = p.regs[reg];
  const char* base = (d.in_stage ? stage : tmp) + d.off;
  if (d.width == 4) {
    const int* b = (const int*)base + row0;
#pragma unroll
    for (int r = 0; r < R; ++r) v[r] = b[r * 32];
  } else if (d.width == 8) {
    const long long* b = (const long long*)base + row0;
#pragma unroll
    for (int r = 0; r < R; ++r) v[r] = b[r * 32];
  } else {
    const signed char* b = (const signed char*)base + row0;
#pragma unroll
    for (int r = 0; r < R; ++r) v[r] = b[r * 32];
  }
}
__device__ __forceinline__ long long load_one(const KPlan& p, int reg, const char* stage, const char* tmp,
                                              int row) {
  const KReg d = p.regs[reg];
  const char* base = (d.in_stage ? stage : tmp) + d.off;
  if (d.width == 4) return ((const int*)base)[row];
  if (d.width == 8) return ((const long long*)base)[row];
  return ((const signed char*)base)[row];
}
template <int R>
__device__ __forceinline__ void store_tmp(const KPlan& p, int reg, char* tmp, int row0, const long long (&v)[R]) {
  const KReg d = p.regs[reg];
  if (d.width == 8) {
    long long* b = (long long*)(tmp + d.off) + row0;
#pragma unroll
    for (int r = 0; r < R; ++r) b[r * 32] = v[r];
  } else {
    int* b = (int*)(tmp + d.off) + row0;
#pragma unroll
    for (int r = 0; r < R; ++r) b[r * 32] = (int)v[r];
  }
}

// ------------------------------------------------------------------ ops
// Selection (Fig 8 count kernel "select"): conjunction of
// range / bitmap predicates folded into the per-thread live mask.
template <int R>
__device__ __forceinline__ uint32_t op_filter(const KPlan& p, int idx, const char* stage, const char* tmp,
                                              int row0, uint32_t mask) {
  const KPred& f = p.preds[idx];
  const KReg d = p.regs[f.reg];
  const char* base = (d.in_stage ? stage : tmp) + d.off;
  if (f.kind == 0 && d.width == 4) {
    const int* b = (const int*)base + row0;
    const int lo = f.lo32, hi = f.hi32;
    const bool neg = f.neg;
#pragma unroll
    for (int r = 0; r < R; ++r) {
      const int v = b[r * 32];
      const bool ok = (v >= lo && v <= hi) != neg;
      if (!ok) mask &= ~(1u << r);
    }
    return mask;
  }
  long long v[R];
  load_rows<R>(p, f.reg, stage, tmp, row0, v);
  if (f.kind == 0) {
    const long long lo = f.lo, hi = f.hi;
    const bool neg = f.neg;
#pragma unroll
    for (int r = 0; r < R; ++r) {
      const bool ok = (v[r] >= lo && v[r] <= hi) != neg;
      if (!ok) mask &= ~(1u << r);
    }
  } else {
#pragma unroll
    for (int r = 0; r < R; ++r) {
      const unsigned long long x = (unsigned long long)v[r];
      const bool ok = x < 256 && ((f.bm[x >> 6] >> (x & 63)) & 1ull);
      if (!ok) mask &= ~(1u << r);
    }
  }
  return mask;
}

// Join probe (Fig 8 "check match" + "build tuple"): in the
// compound kernel the probe runs once and the payload stays on chip
// (P:947-953).  Slots are {key, payload...} of W words.  Direct-mapped tables
// (dense keys) resolve every probe with one load; linear-probing tables load a
// whole aligned 16-B group (4, 2 or 1 slots) per round and scan it in probe
// order, so a warp's round count is rarely more than one.
template <int R, int W>
__device__ __forceinline__ uint32_t probe_rows(const KPlan& p, const KProbe& pr, const long long (&kv)[R],
                                               const long long (&kv2)[R], char* tmp, int row0, uint32_t mask) {
  uint32_t pending = mask, found = 0;
  uint32_t pos[R];
#pragma unroll
  for (int r = 0; r < R; ++r) {
    const bool ok = kv[r] > (long long)INT_MIN && kv[r] <= (long long)INT_MAX;
    if (!ok) pending &= ~(1u << r);
    if (pr.direct) {
      pos[r] = (uint32_t)((int)kv[r] - pr.dmin);
      if (pos[r] >= pr.mask) pending &= ~(1u << r);  // outside the key range: miss
    } else {
      pos[r] = ((uint32_t)(int)kv[r] * 0x9E3779B1u) >> (32u - pr.log2cap);
    }
  }
  const bool inner = hq_probe_has_payload(pr.mode);
  int* dst0 = (int*)(tmp + p.regs[pr.dst[0]].off) + row0;
  int* dst1 = (int*)(tmp + p.regs[pr.dst[W > 2 ? 1 : 0]].off) + row0;
  int* dst2 = (int*)(tmp + p.regs[pr.dst[W > 2 ? 2 : 0]].off) + row0;
  if (W > 1 && pr.mode == HQ_PROBE_OUTER) {  // LEFT OUTER: a miss leaves payload 0
#pragma unroll
    for (int r = 0; r < R; ++r) {
      if (pr.npay > 0) dst0[r * 32] = 0;
      if (W > 2 && pr.npay > 1) dst1[r * 32] = 0;
      if (W > 2 && pr.npay > 2) dst2[r * 32] = 0;
    }
  }
  constexpr int G = W == 1 ? 4 : (W == 2 ? 2 : 1);  // slots per 16-B group
  while (pending) {
    int4 sl[R];
#pragma unroll
    for (int r = 0; r < R; ++r) {  // R independent loads in flight
      if (pending & (1u << r)) {
        if (pr.direct) {
          if (W == 1) sl[r].x = __ldg((const int*)pr.slots + pos[r]);
          else if (W == 2) { const int2 t = __ldg((const int2*)pr.slots + pos[r]); sl[r].x = t.x; sl[r].y = t.y; }
          else sl[r] = __ldg((const int4*)pr.slots + pos[r]);
        } else {
          sl[r] = __ldg((const int4*)pr.slots + pos[r] / G);
        }
      }
    }
#pragma unroll
    for (int r = 0; r < R; ++r) {
      if (pending & (1u << r)) {
        const int key = (int)kv[r];
        int sk[G], sp0[G], sp1 = sl[r].z, sp2 = sl[r].w;
        if (G == 4) { sk[0] = sl[r].x; sk[G > 1 ? 1 : 0] = sl[r].y; sk[G > 2 ? 2 : 0] = sl[r].z; sk[G > 3 ? 3 : 0] = sl[r].w; }
        else if (G == 2) { sk[0] = sl[r].x; sp0[0] = sl[r].y; sk[G > 1 ? 1 : 0] = sl[r].z; sp0[G > 1 ? 1 : 0] = sl[r].w; }
        else { sk[0] = sl[r].x; sp0[0] = sl[r].y; }
        const int first = pr.direct ? 0 : (int)(pos[r] % G);
        int hit = -1;
        bool stop = pr.direct;
#pragma unroll
        for (int j = 0; j < G; ++j) {
          if (!stop && j >= first) {
            if (sk[j] == key && (!pr.composite || (G == 1 ? sl[r].y : sp0[j]) == (int)kv2[r])) { hit = j; stop = true; }
            else if (sk[j] == INT_MIN) stop = true;
          }
        }
        if (pr.direct && sk[0] == key) hit = 0;
        if (hit >= 0) {
          found |= 1u << r;
          pending &= ~(1u << r);
          if (W > 1 && inner) {  // payload stays on chip
            int v0 = sp0[0];
#pragma unroll
            for (int j = 1; j < G; ++j)
              if (hit == j) v0 = sp0[j];
            if (pr.composite) {  // word 1 is the second key: payloads are words 2, 3
              if (W > 2 && pr.npay > 0) dst0[r * 32] = sp1;
              if (W > 2 && pr.npay > 1) dst1[r * 32] = sp2;
            } else {
              if (pr.npay > 0) dst0[r * 32] = v0;
              if (W > 2 && pr.npay > 1) dst1[r * 32] = sp1;
              if (W > 2 && pr.npay > 2) dst2[r * 32] = sp2;
            }
          }
        } else if (stop) {
          pending &= ~(1u << r);
        } else {
          pos[r] = ((pos[r] / G + 1) * G) & pr.mask;  // next group
        }
      }
    }
  }
  if (pr.mode == HQ_PROBE_ANTI) return mask & ~found;
  if (pr.mode == HQ_PROBE_OUTER) return mask;
  return mask & found;
}

template <int R>
__device__ __forceinline__ uint32_t op_probe(const KPlan& p, int idx, const char* stage, char* tmp, int row0,
                                             uint32_t mask) {
  const KProbe& pr = p.probes[idx];
  long long kv[R], kv2[R];
  load_rows<R>(p, pr.key_reg, stage, tmp, row0, kv);
  if (pr.composite) load_rows<R>(p, pr.key2_reg, stage, tmp, row0, kv2);
  if (pr.words == 1) return probe_rows<R, 1>(p, pr, kv, kv2, tmp, row0, mask);
  if (pr.words == 2) return probe_rows<R, 2>(p, pr, kv, kv2, tmp, row0, mask);
  return probe_rows<R, 4>(p, pr, kv, kv2, tmp, row0, mask);
}

// Projection / arithmetic (revenue[wp] = price[tid]*discount[tid]):
// an int64 accumulator machine, one instruction stream per plan, evaluated for
// the lane's R rows at once.
template <int R>
__device__ __forceinline__ void op_compute(const KPlan& p, int idx, const char* stage, char* tmp, int row0,
                                           uint32_t mask) {
  const KCompute c = p.comps[idx];
  long long acc[R];
#pragma unroll
  for (int r = 0; r < R; ++r) acc[r] = 0;
  for (int i = c.first; i < c.first + c.n; ++i) {
    const KInsn in = p.insns[i];
    long long o[R];
    if (in.reg < 0) {
#pragma unroll
      for (int r = 0; r < R; ++r) o[r] = in.imm;
    } else {
      load_rows<R>(p, in.reg, stage, tmp, row0, o);
    }
    switch (in.opc) {
      case HQ_I_LOAD:
#pragma unroll
        for (int r = 0; r < R; ++r) acc[r] = o[r];
        break;
      case HQ_I_ADD:
#pragma unroll
        for (int r = 0; r < R; ++r) acc[r] += o[r];
        break;
      case HQ_I_SUB:
#pragma unroll
        for (int r = 0; r < R; ++r) acc[r] -= o[r];
        break;
      case HQ_I_RSUB:
#pragma unroll
        for (int r = 0; r < R; ++r) acc[r] = o[r] - acc[r];
        break;
      case HQ_I_MUL:
#pragma unroll
        for (int r = 0; r < R; ++r) acc[r] *= o[r];
        break;
      case HQ_I_AND_EQ: case HQ_I_AND_NE: case HQ_I_AND_LT: case HQ_I_AND_LE: case HQ_I_AND_GT: case HQ_I_AND_GE:
      case HQ_I_AND_IN: case HQ_I_OR:
#pragma unroll
        for (int r = 0; r < R; ++r) acc[r] = hq_pred_insn(in.opc, acc[r], o[r], in.imm);
        break;
      default: {  // DIV / MOD
        bool bad = false;
#pragma unroll
        for (int r = 0; r < R; ++r) {
          if (o[r] == 0) {
            bad |= (mask >> r) & 1u;
            acc[r] = 0;
          } else {
            acc[r] = in.opc == HQ_I_DIV ? acc[r] / o[r] : acc[r] % o[r];
          }
        }
        if (bad) atomicOr(p.err, HQF_DIV_ZERO);
      }
    }
  }
  store_tmp<R>(p, c.dst, tmp, row0, acc);
}

// Local resolution target: the shared address of the shared-memory dense or
// hash table entry, or 0 when the smem hash table is full -- the caller then
// propagates to the global table directly (C3 -> C2).
__device__ __forceinline__ uint32_t local_locate(const KPlan& p, char* sagg, unsigned long long key) {
  if (p.smode == SM_DENSE) return smem_u32((long long*)sagg + key * p.vwords);
  if (p.smode == SM_HASH) {
    unsigned long long* keys = (unsigned long long*)sagg;
    long long* ent = (long long*)sagg + p.smem_cap;
    const uint32_t m = p.smem_cap - 1;
    uint32_t h = hash64(key, p.slog2);
#pragma unroll 1
    for (int i = 0; i < 32; ++i) {
      const unsigned long long k = keys[h];
      bool hit = k == key;
      if (!hit && k == EMPTY_KEY) {
        const unsigned long long old = atomicCAS(keys + h, EMPTY_KEY, key);
        hit = old == EMPTY_KEY || old == key;
      }
      if (hit) return smem_u32(ent + (size_t)h * p.vwords);
      h = (h + 1) & m;
    }
  }
  return 0u;
}
// Update one group entry -- shared (split 32-bit atomics) when the local table
// holds it, else global (red) -- with `cnt` rows whose aggregate values come
// from val(a).
template <class Val>
__device__ __forceinline__ void group_update(const KPlan& p, char* sagg, unsigned long long key, bool local,
                                             unsigned long long cnt, Val val) {
  const uint32_t sa = local ? local_locate(p, sagg, key) : 0u;
  if (sa) {
    s_add64(sa, (long long)cnt);
#pragma unroll
    for (int a = 0; a < HQ_MAX_AGGS; ++a)
      if (a < p.naggs) s_agg(p.agg_fn[a], sa + 8u * (1 + a), val(a), cnt);
    return;
  }
  long long* e = global_locate(p, key);
  if (!e) return;
  g_add64(e, (long long)cnt);
#pragma unroll
  for (int a = 0; a < HQ_MAX_AGGS; ++a)
    if (a < p.naggs) g_agg(p.agg_fn[a], e + 1 + a, val(a), cnt);
}

// ------------------------------------------------------------------- sinks
// Grouped aggregation with local resolution (C3-style, P:1211-1220,
// P:2040-2057): per row slot, lanes with equal keys are combined with
// match_any + shuffle reductions so each distinct key of a warp costs one
// shared-memory update; singletons update directly.
template <int R>
__device__ __forceinline__ void sink_group(const KPlan& p, const char* stage, const char* tmp, char* sagg,
                                           int row0, uint32_t mask, int lane) {
  unsigned long long gk[R];
#pragma unroll
  for (int r = 0; r < R; ++r) gk[r] = 0;
  for (int i = 0; i < p.nkeys; ++i) {
    long long v[R];
    load_rows<R>(p, p.key_reg[i], stage, tmp, row0, v);
    const long long mn = p.key_min[i], card = p.key_card[i], st = p.key_stride[i];
    bool bad = false;
#pragma unroll
    for (int r = 0; r < R; ++r) {
      const long long d = v[r] - mn;
      if (d < 0 || d >= card) {
        bad |= (mask >> r) & 1u;
        mask &= ~(1u << r);
      }
      gk[r] += (unsigned long long)d * (unsigned long long)st;
    }
    if (bad) atomicOr(p.err, HQF_KEY_DOMAIN);
  }
  if (p.smode == SM_LANE) {
    // tiny dense group domain: every lane owns a private accumulator table in
    // shared memory ([entry][lane] layout), updated with plain read-modify-write
    long long* lt = (long long*)sagg + threadIdx.x;
    const int nl = p.nw * 32;
#pragma unroll
    for (int r = 0; r < R; ++r) {
      if ((mask >> r) & 1u) {
        const int row = row0 + r * 32;
        long long* e = lt + (size_t)gk[r] * p.nacc * nl;
        e[0] += 1;
        for (int a = 1; a < p.nacc; ++a) {
          const long long v = load_one(p, p.acc_reg[a], stage, tmp, row);
          e[a * nl] = agg_combine(p.acc_fn[a], e[a * nl], v);
        }
      }
    }
    return;
  }
  const bool c2 = p.resolution == HQ_RES_ATOMIC;
#pragma unroll
  for (int r = 0; r < R; ++r) {
    const bool live = (mask >> r) & 1u;
    const uint32_t act = __ballot_sync(FULLMASK, live);
    if (!act) continue;
    const int row = row0 + r * 32;
    const unsigned long long mk = live ? gk[r] : EMPTY_KEY;
    // few live lanes (selective pipelines): each updates directly; match_any
    // only pays when many lanes may share a key
    const bool sparse = c2 || __popc(act) <= 4;
    const uint32_t peers = sparse ? (1u << lane) & act : __match_any_sync(FULLMASK, mk) & act;
    const bool single = live && __popc(peers) == 1;
    if (single) {  // C2 rows, and keys unique within the warp: direct update
      group_update(p, sagg, gk[r], !c2, 1ull, [&](int a) {
        return p.agg_fn[a] == HQ_AGG_COUNT ? 1ll : load_one(p, p.agg_reg[a], stage, tmp, row);
      });
    }
    uint32_t multi = act & ~__ballot_sync(FULLMASK, single);
    while (multi) {  // one warp-wide reduction per distinct key, leader updates
      const int leader = __ffs(multi) - 1;
      const uint32_t grp = __shfl_sync(FULLMASK, peers, leader);
      const bool mine = (grp >> lane) & 1u;
      long long vals[HQ_MAX_AGGS];
#pragma unroll
      for (int a = 0; a < HQ_MAX_AGGS; ++a) {
        if (a < p.naggs) {
          const uint8_t fn = p.agg_fn[a];
          long long v = agg_identity(fn);
          if (mine) v = fn == HQ_AGG_COUNT ? 1 : load_one(p, p.agg_reg[a], stage, tmp, row);
          vals[a] = warp_reduce(fn, v);
        }
      }
      if (lane == leader)
        group_update(p, sagg, gk[r], true, (unsigned long long)__popc(grp), [&](int a) { return vals[a]; });
      multi &= ~grp;
    }
  }
}

// Materialisation with LRGP (A3; Fig 25): warp
// ballot/popc prefix, block scan over the warps, one atomicAdd per block and
// tile, write at local offset + global offset.  Rows stay in order inside the
// block's segment; segments are permuted.
template <int R>
__device__ __forceinline__ void sink_materialise(const KPlan& p, const char* stage, const char* tmp, int row0,
                                                 uint32_t mask, int warp, int lane, int* s_wtot,
                                                 unsigned long long* s_base) {
  uint32_t b[R];
  int wtot = 0;
#pragma unroll
  for (int r = 0; r < R; ++r) {
    b[r] = __ballot_sync(FULLMASK, (mask >> r) & 1u);
    wtot += __popc(b[r]);
  }
  unsigned long long base;
  if (p.resolution == HQ_RES_ATOMIC) {
    base = 0;  // per-row atomics below (A2)
  } else {
    if (lane == 0) s_wtot[warp] = wtot;
    consumer_bar(p.nw);
    if (warp == 0) {
      int v = lane < p.nw ? s_wtot[lane] : 0;
      int incl = v;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const int t = __shfl_up_sync(FULLMASK, incl, o);
        if (lane >= o) incl += t;
      }
      const int total = __shfl_sync(FULLMASK, incl, 31);
      unsigned long long g = 0;
      if (lane == 0 && total > 0) g = atomicAdd(p.counter, (unsigned long long)total);  // global propagation
      g = __shfl_sync(FULLMASK, g, 0);
      if (lane < p.nw) s_base[lane] = g + (unsigned long long)(incl - v);
    }
    consumer_bar(p.nw);
    base = s_base[warp];
  }
  const uint32_t lt = lanemask_lt();
  unsigned long long run = 0;
#pragma unroll
  for (int r = 0; r < R; ++r) {
    if ((mask >> r) & 1u) {
      unsigned long long pos;
      if (p.resolution == HQ_RES_ATOMIC) pos = atomicAdd(p.counter, 1ull);
      else pos = base + run + __popc(b[r] & lt);
      if ((long long)pos < p.capacity) {
        const int row = row0 + r * 32;
        for (int j = 0; j < p.nout; ++j) {
          const long long v = load_one(p, p.out_reg[j], stage, tmp, row);
          const uint8_t w = p.out_width[j];
          if (w == 8) ((long long*)p.out_ptr[j])[pos] = v;
          else if (w == 4) ((int*)p.out_ptr[j])[pos] = (int)v;
          else ((signed char*)p.out_ptr[j])[pos] = (signed char)v;
        }
      } else {
        atomicOr(p.err, HQF_CAPACITY);
      }
    }
    run += __popc(b[r]);
  }
}

// ------------------------------------------------------------------ kernel
// SK: sink kind, a template parameter so each instantiation only carries the
// registers of its own sink (0 = scalar aggregate, 1 = grouped, 2 = materialise).
enum { SK_SCALAR = 0, SK_GROUP = 1, SK_MAT = 2 };
template <int R, int SK>
__global__ void __launch_bounds__(NTHREADS, 1) hq_fused_pipeline_kernel(const __grid_constant__ KPlan p) {
  extern __shared__ __align__(128) char smem[];
  uint64_t* full = (uint64_t*)smem;
  uint64_t* empty = full + MAX_STAGES;
  unsigned long long* s_base = (unsigned long long*)(empty + MAX_STAGES);  // [NW max]
  int* s_wtot = (int*)(s_base + NW);                                         // [NW max]
  long long* s_red = (long long*)(s_wtot + NW);                              // [NW max][1+MAX_AGGS]
  const int nw = p.nw;
  char* tmp = smem + p.off_tmp;
  char* sagg = smem + p.off_agg;
  char* stages = smem + p.off_stage;

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int T = p.tile_rows, S = p.nstages;
  const long long first_tile = p.row_begin / T;
  const long long ntiles = p.row_end > p.row_begin ? (p.row_end + T - 1) / T - first_tile : 0;
  const long long nj = ntiles > blockIdx.x ? (ntiles - blockIdx.x + gridDim.x - 1) / gridDim.x : 0;

  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], nw);
    }
    fence_mbar_init();
  }
  // smem pre-aggregation table: identities
  if (SK == SK_GROUP && warp < nw && p.smode != SM_NONE) {
    if (p.smode == SM_LANE) {
      long long* t = (long long*)sagg;
      const uint32_t nl = nw * 32, n = p.smem_cap * p.nacc * nl;
      for (uint32_t i = threadIdx.x; i < n; i += nl) {
        const uint32_t a = (i / nl) % p.nacc;
        t[i] = a == 0 ? 0 : agg_identity(p.acc_fn[a]);
      }
    } else if (p.smode == SM_DENSE) {
      long long* t = (long long*)sagg;
      for (uint32_t i = threadIdx.x; i < p.smem_cap * p.vwords; i += nw * 32) {
        const uint32_t c = i % p.vwords;
        t[i] = c == 0 ? 0 : agg_identity(p.agg_fn[c - 1]);
      }
    } else {
      unsigned long long* keys = (unsigned long long*)sagg;
      long long* ent = (long long*)sagg + p.smem_cap;
      for (uint32_t i = threadIdx.x; i < p.smem_cap; i += nw * 32) keys[i] = EMPTY_KEY;
      for (uint32_t i = threadIdx.x; i < p.smem_cap * p.vwords; i += nw * 32) {
        const uint32_t c = i % p.vwords;
        ent[i] = c == 0 ? 0 : agg_identity(p.agg_fn[c - 1]);
      }
    }
  }
  __syncthreads();

  if (warp == nw) {
    // ------------------------------------------------ TMA producer warp
    if (lane == 0) {
      const uint64_t pol = policy_evict_first();
      for (long long j = 0; j < nj; ++j) {
        const int s = (int)(j % S);
        if (j >= S) mbar_wait(&empty[s], (uint32_t)(((j / S) - 1) & 1));
        const long long t0 = (first_tile + blockIdx.x + j * gridDim.x) * (long long)T;
        char* st = stages + (size_t)s * p.stage_stride;
        if (t0 >= p.row_begin && t0 + T <= p.row_end) {
          mbar_expect_tx(&full[s], p.stage_bytes);
          for (int c = 0; c < p.ncols; ++c) {
            const KCol col = p.cols[c];
            tma_load_1d(st + col.soff, col.ptr + t0 * col.width, (uint32_t)T * col.width, &full[s], pol);
          }
        } else {
          mbar_arrive(&full[s]);  // ragged head/tail tile: consumers load it themselves
        }
      }
    }
    return;
  }

  // ------------------------------------------------------ consumer warps
  const int row0 = warp * 32 * R + lane;
  long long sacc[SK == SK_SCALAR ? HQ_MAX_AGGS : 1];
  unsigned long long scount = 0;
  if constexpr (SK == SK_SCALAR) {
#pragma unroll
    for (int a = 0; a < HQ_MAX_AGGS; ++a) sacc[a] = a < p.naggs ? agg_identity(p.agg_fn[a]) : 0;
  }

  for (long long j = 0; j < nj; ++j) {
    const int s = (int)(j % S);
    mbar_wait(&full[s], (uint32_t)((j / S) & 1));
    const long long t0 = (first_tile + blockIdx.x + j * gridDim.x) * (long long)T;
    const int lo = (int)(p.row_begin > t0 ? p.row_begin - t0 : 0);
    const int hi = (int)(p.row_end - t0 < T ? p.row_end - t0 : T);
    char* stage = stages + (size_t)s * p.stage_stride;
    uint32_t mask = 0;
#pragma unroll
    for (int r = 0; r < R; ++r) {
      const int row = row0 + r * 32;
      if (row >= lo && row < hi) mask |= 1u << r;
    }
    if (lo > 0 || hi < T) {  // ragged tile: each lane copies its own rows
      for (int c = 0; c < p.ncols; ++c) {
        const KCol col = p.cols[c];
#pragma unroll
        for (int r = 0; r < R; ++r) {
          if (mask & (1u << r)) {
            const int row = row0 + r * 32;
            const long long g = t0 + row;
            char* dst = stage + col.soff;
            if (col.width == 4) ((int*)dst)[row] = ((const int*)col.ptr)[g];
            else if (col.width == 8) ((long long*)dst)[row] = ((const long long*)col.ptr)[g];
            else ((signed char*)dst)[row] = ((const signed char*)col.ptr)[g];
          }
        }
      }
      fence_proxy_async();
      __syncwarp();
    }
    // ---- the plan's operators, in order
    for (int o = 0; o < p.nops; ++o) {
      if (!__any_sync(FULLMASK, mask)) break;
      const KOp op = p.ops[o];
      if (op.kind == OP_FILTER) mask = op_filter<R>(p, op.idx, stage, tmp, row0, mask);
      else if (op.kind == OP_PROBE) mask = op_probe<R>(p, op.idx, stage, tmp, row0, mask);
      else op_compute<R>(p, op.idx, stage, tmp, row0, mask);
    }
    // ---- sink
    if constexpr (SK == SK_MAT) {
      sink_materialise<R>(p, stage, tmp, row0, mask, warp, lane, s_wtot, s_base);
    } else if constexpr (SK == SK_SCALAR) {
      if (p.resolution == HQ_RES_ATOMIC) {  // B2: per-row atomic reduce
#pragma unroll
        for (int r = 0; r < R; ++r) {
          if (mask & (1u << r)) {
            long long vals[HQ_MAX_AGGS];
#pragma unroll
            for (int a = 0; a < HQ_MAX_AGGS; ++a)
              if (a < p.naggs)
                vals[a] = p.agg_fn[a] == HQ_AGG_COUNT ? 1 : load_one(p, p.agg_reg[a], stage, tmp, row0 + r * 32);
            entry_update(p, p.gtab, 1, vals);
          }
        }
      } else {  // B3: register partials, reduced once at the end
        scount += __popc(mask);
#pragma unroll
        for (int a = 0; a < HQ_MAX_AGGS; ++a) {
          if (a < p.naggs && p.agg_fn[a] != HQ_AGG_COUNT) {
            long long v[R];
            load_rows<R>(p, p.agg_reg[a], stage, tmp, row0, v);
            const uint8_t fn = p.agg_fn[a];
#pragma unroll
            for (int r = 0; r < R; ++r)
              if (mask & (1u << r)) sacc[SK == SK_SCALAR ? a : 0] = agg_combine(fn, sacc[SK == SK_SCALAR ? a : 0], v[r]);
          }
        }
      }
    } else {
      sink_group<R>(p, stage, tmp, sagg, row0, mask, lane);
    }
    __syncwarp();
    if (lane == 0) mbar_arrive(&empty[s]);
  }

  // ---------------------------------------------- global propagation (end)
  {
    if (SK == SK_SCALAR && p.resolution != HQ_RES_ATOMIC) {
      // B3: warp reduction -> block reduction in smem -> one atomic per aggregate
      unsigned long long c = scount;
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) c += __shfl_xor_sync(FULLMASK, c, o);
      long long red[HQ_MAX_AGGS];
#pragma unroll
      for (int a = 0; a < HQ_MAX_AGGS; ++a) red[a] = a < p.naggs ? warp_reduce(p.agg_fn[a], sacc[SK == SK_SCALAR ? a : 0]) : 0;
      if (lane == 0) {
        s_red[warp * (1 + HQ_MAX_AGGS)] = (long long)c;
#pragma unroll
        for (int a = 0; a < HQ_MAX_AGGS; ++a) s_red[warp * (1 + HQ_MAX_AGGS) + 1 + a] = red[a];
      }
      consumer_bar(nw);
      if (threadIdx.x == 0) {
        unsigned long long cnt = 0;
        long long vals[HQ_MAX_AGGS];
#pragma unroll
        for (int a = 0; a < HQ_MAX_AGGS; ++a) vals[a] = a < p.naggs ? agg_identity(p.agg_fn[a]) : 0;
        for (int w = 0; w < nw; ++w) {
          cnt += (unsigned long long)s_red[w * (1 + HQ_MAX_AGGS)];
#pragma unroll
          for (int a = 0; a < HQ_MAX_AGGS; ++a)
            if (a < p.naggs) vals[a] = agg_combine(p.agg_fn[a], vals[a], s_red[w * (1 + HQ_MAX_AGGS) + 1 + a]);
        }
        if (cnt) entry_update(p, p.gtab, cnt, vals);
      }
    } else if (SK == SK_GROUP && p.smode != SM_NONE) {
      // C3: merge the block's pre-aggregates into the global table
      consumer_bar(nw);
      if (p.smode == SM_LANE) {
        const int nl = nw * 32;
        const long long* t = (const long long*)sagg;
        for (uint32_t g = threadIdx.x; g < p.smem_cap; g += nl) {
          const long long* e = t + (size_t)g * p.nacc * nl;
          unsigned long long cnt = 0;
          for (int l = 0; l < nl; ++l) cnt += (unsigned long long)e[l];
          if (!cnt) continue;
          long long acc[HQ_MAX_AGGS + 1];
          for (int a = 1; a < p.nacc; ++a) {
            long long v = agg_identity(p.acc_fn[a]);
            for (int l = 0; l < nl; ++l) v = agg_combine(p.acc_fn[a], v, e[a * nl + l]);
            acc[a] = v;
          }
          long long vals[HQ_MAX_AGGS];
          for (int k = 0; k < p.naggs; ++k) vals[k] = p.acc_of[k] ? acc[p.acc_of[k]] : (long long)cnt;
          global_update(p, g, cnt, vals);
        }
      } else if (p.smode == SM_DENSE) {
        const long long* t = (const long long*)sagg;
        for (uint32_t g = threadIdx.x; g < p.smem_cap; g += nw * 32) {
          const long long* e = t + (size_t)g * p.vwords;
          if (e[0] != 0) global_update(p, g, (unsigned long long)e[0], e + 1);
        }
      } else {
        const unsigned long long* keys = (const unsigned long long*)sagg;
        const long long* ent = (const long long*)sagg + p.smem_cap;
        for (uint32_t h = threadIdx.x; h < p.smem_cap; h += nw * 32) {
          if (keys[h] != EMPTY_KEY) {
            const long long* e = ent + (size_t)h * p.vwords;
            global_update(p, keys[h], (unsigned long long)e[0], e + 1);
          }
        }
      }
    }
  }
}

// group table initialisation (identities; hash keys EMPTY)
__global__ void hq_init_groups_kernel(long long* tab, long long n, uint32_t vwords, int hash, uint64_t fns_lo) {
  const uint32_t stride = vwords + (hash ? 1 : 0);
  const long long total = n * stride;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total;
       i += (long long)gridDim.x * blockDim.x) {
    // (a 32-bit remainder where the table allows: the 64-bit one is a long software sequence)
    const uint32_t c = total <= 0xFFFFFFFFll ? (uint32_t)i % stride : (uint32_t)(i % stride);
    long long v;
    if (hash && c == 0) v = (long long)EMPTY_KEY;
    else {
      const uint32_t k = c - (hash ? 1 : 0);
      v = k == 0 ? 0 : agg_identity((uint8_t)((fns_lo >> (8 * (k - 1))) & 0xff));
    }
    tab[i] = v;
  }
}

int64_t fused_smem_bytes(const KPlan& kp) {
  return (int64_t)kp.off_stage + (int64_t)kp.nstages * kp.stage_stride;
}

template <int R, int SK>
static void launch_one(hq_ctx* ctx, const KPlan& kp, int grid, size_t smem) {
  HQ_CUDA(cudaFuncSetAttribute(hq_fused_pipeline_kernel<R, SK>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  ctx->launches++;
  hq_fused_pipeline_kernel<R, SK><<<grid, (kp.nw + 1) * 32, smem, ctx->stream>>>(kp);
}

void launch_fused(hq_ctx* ctx, const KPlan& kp, int grid, size_t smem) {
  const int sk = kp.sink == HQ_SINK_MATERIALISE ? SK_MAT : (kp.nkeys == 0 ? SK_SCALAR : SK_GROUP);
  if (kp.R == 4) {
    if (sk == SK_SCALAR) launch_one<4, SK_SCALAR>(ctx, kp, grid, smem);
    else if (sk == SK_GROUP) launch_one<4, SK_GROUP>(ctx, kp, grid, smem);
    else launch_one<4, SK_MAT>(ctx, kp, grid, smem);
  } else {
    if (sk == SK_SCALAR) launch_one<2, SK_SCALAR>(ctx, kp, grid, smem);
    else if (sk == SK_GROUP) launch_one<2, SK_GROUP>(ctx, kp, grid, smem);
    else launch_one<2, SK_MAT>(ctx, kp, grid, smem);
  }
  HQ_CUDA(cudaGetLastError());
}

void launch_init_groups(hq_ctx* ctx, long long* tab, int64_t ngroups, uint32_t vwords, bool hash,
                        const uint8_t* agg_fn, int naggs) {
  uint64_t fns = 0;
  for (int a = 0; a < naggs; ++a) fns |= (uint64_t)agg_fn[a] << (8 * a);
  const long long total = ngroups * (long long)(vwords + (hash ? 1 : 0));
  int grid = (int)std::min<long long>((total + 255) / 256, (long long)ctx->num_sms * 8);
  if (grid < 1) grid = 1;
  ctx->launches++;
  hq_init_groups_kernel<<<grid, 256, 0, ctx->stream>>>(tab, ngroups, vwords, hash ? 1 : 0, fns);
  HQ_CUDA(cudaGetLastError());
}

}  // namespace hqk
