// hq_device.cuh -- device helpers shared by the fused kernel (hq_pipeline.cu)
// and the operator-at-a-time baseline (hq_oaat.cu): aggregate identities and
// combination, atomics on group-table entries, the global group table (dense
// or atomicCAS hash).
//
// Atomics are written in PTX on purpose: sm_100a has no native 64-bit
// shared-memory atomic add (the compiler emits a CAS spin loop), so shared
// entries use two native 32-bit atom.shared.add with an explicit carry; global
// entries use red.global (no return value, no generic-address ATOM).
#pragma once
#include <climits>

#include "hq_internal.h"

namespace hqk {

#ifndef FULLMASK
#define FULLMASK 0xffffffffu
#endif

// --------------------------------------------------------------- agg tables
__device__ __forceinline__ long long agg_identity(uint8_t fn) {
  return fn == HQ_AGG_MIN ? LLONG_MAX : (fn == HQ_AGG_MAX ? LLONG_MIN : 0);
}
__device__ __forceinline__ long long agg_combine(uint8_t fn, long long a, long long b) {
  return fn == HQ_AGG_MIN ? (a < b ? a : b) : (fn == HQ_AGG_MAX ? (a > b ? a : b) : a + b);
}
__device__ __forceinline__ long long warp_reduce(uint8_t fn, long long v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = agg_combine(fn, v, __shfl_xor_sync(FULLMASK, v, o));
  return v;
}

// ---- global-memory entries (red: fire-and-forget)
__device__ __forceinline__ void g_add64(long long* p, long long v) {
  asm volatile("red.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void g_min64(long long* p, long long v) {
  asm volatile("red.global.min.s64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void g_max64(long long* p, long long v) {
  asm volatile("red.global.max.s64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void g_agg(uint8_t fn, long long* t, long long v, unsigned long long cnt) {
  if (fn == HQ_AGG_MIN) g_min64(t, v);
  else if (fn == HQ_AGG_MAX) g_max64(t, v);
  else g_add64(t, fn == HQ_AGG_COUNT ? (long long)cnt : v);
}
// accumulate (count, vals) into one global entry [count, agg...]
__device__ __forceinline__ void entry_update(const KPlan& p, long long* e, unsigned long long cnt,
                                             const long long* vals) {
  g_add64(e, (long long)cnt);
  for (int a = 0; a < p.naggs; ++a) g_agg(p.agg_fn[a], e + 1 + a, vals[a], cnt);
}

// ---- shared-memory entries (addresses are 32-bit shared-window offsets)
__device__ __forceinline__ void s_add64(uint32_t a, long long v) {
  const uint32_t lo = (uint32_t)v;
  uint32_t hi = (uint32_t)((unsigned long long)v >> 32);
  uint32_t old;
  asm volatile("atom.shared.add.u32 %0, [%1], %2;" : "=r"(old) : "r"(a), "r"(lo) : "memory");
  hi += (old + lo < old) ? 1u : 0u;  // carry out of the low word
  if (hi) asm volatile("red.shared.add.u32 [%0], %1;" ::"r"(a + 4), "r"(hi) : "memory");
}
__device__ __forceinline__ void s_minmax64(uint32_t a, long long v, bool is_min) {
  unsigned long long cur;
  asm volatile("ld.shared.u64 %0, [%1];" : "=l"(cur) : "r"(a) : "memory");
  while (is_min ? v < (long long)cur : v > (long long)cur) {
    unsigned long long prev;
    asm volatile("atom.shared.cas.b64 %0, [%1], %2, %3;" : "=l"(prev) : "r"(a), "l"(cur), "l"(v) : "memory");
    if (prev == cur) break;
    cur = prev;
  }
}
__device__ __forceinline__ void s_agg(uint8_t fn, uint32_t t, long long v, unsigned long long cnt) {
  if (fn == HQ_AGG_MIN) s_minmax64(t, v, true);
  else if (fn == HQ_AGG_MAX) s_minmax64(t, v, false);
  else s_add64(t, fn == HQ_AGG_COUNT ? (long long)cnt : v);
}

__device__ __forceinline__ uint32_t hash64(unsigned long long k, int log2) {
  return (uint32_t)((k * 0x9E3779B97F4A7C15ull) >> (64 - log2));
}
// Global propagation target: dense array slot, or the entry of `key` in the
// global hash table, claimed with atomicCAS ("atomic_hash_reduce", App C
// P:2049-2052).  NULL (fault raised) when the hash table is full.
__device__ __forceinline__ long long* global_locate(const KPlan& p, unsigned long long key) {
  if (p.gmode != GM_HASH) return p.gtab + key * p.vwords;
  const uint32_t vw1 = p.vwords + 1;
  uint64_t h = hash64(key, p.glog2);
  for (uint64_t i = 0; i <= p.gmask; ++i) {
    unsigned long long* kp = (unsigned long long*)(p.gtab + h * vw1);
    const unsigned long long k = *(volatile unsigned long long*)kp;
    if (k == key) return p.gtab + h * vw1 + 1;
    if (k == EMPTY_KEY) {
      const unsigned long long old = atomicCAS(kp, EMPTY_KEY, key);
      if (old == EMPTY_KEY || old == key) return p.gtab + h * vw1 + 1;
    }
    h = (h + 1) & p.gmask;
  }
  atomicOr(p.err, HQF_GROUP_FULL);
  return nullptr;
}
__device__ __forceinline__ void global_update(const KPlan& p, unsigned long long key, unsigned long long cnt,
                                              const long long* vals) {
  long long* e = global_locate(p, key);
  if (e) entry_update(p, e, cnt, vals);
}
}  // namespace hqk
