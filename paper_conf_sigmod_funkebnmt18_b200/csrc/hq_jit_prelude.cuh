// hq_jit_prelude.cuh -- fixed device code of the generated (NVRTC) pipeline
// kernels; hq_jit.cu embeds this file and prepends the plan's constants.
//
// Query compilation as in HorseQC (§4.3 / §5.2):
// each pipeline becomes one kernel whose operators are straight-line code with
// the plan's constants, columns and temporaries in registers.  This prelude
// holds what every generated kernel shares: PTX wrappers (mbarrier, 1-D TMA,
// fences), atomics on group-table entries, warp reductions, and the
// shared/global group-table lookups.  It expects these generated constants:
//   NW, R, T, S, STAGE_STRIDE, OFF_TMP, OFF_AGG, OFF_STAGE, STAGE_BYTES,
//   NAGGS, AGG_FN[], VWORDS, GMODE, SMODE, SMEM_CAP, SCOPIES, SLOG2, NACC, ACC_FN[].
typedef unsigned int u32;
typedef unsigned long long u64;
typedef long long i64;
#define HQ_FULL 0xffffffffu
#define HQ_INT_MIN (-2147483647 - 1)
#define HQ_INT_MAX 2147483647
#define HQ_LL_MAX 9223372036854775807LL
#define HQ_LL_MIN (-HQ_LL_MAX - 1LL)
#define HQ_EMPTY_KEY 0xffffffffffffffffULL
// aggregate functions (hq.h hq_agg_fn)
#define F_SUM 1
#define F_COUNT 2
#define F_MIN 3
#define F_MAX 4
#define F_AVG 5
// fault bits (hq_internal.h HQF_*)
#define F_KEY_DOMAIN 2
#define F_GROUP_FULL 4
#define F_DIV_ZERO 8
#define F_CAPACITY 1

__device__ __forceinline__ u32 smem_u32(const void* p) { return (u32)__cvta_generic_to_shared(p); }
// loads from read-only shared tables at 32-bit shared-window addresses
__device__ __forceinline__ u32 lds_u32(u32 a) {
  u32 v;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ u32 lds_u8(u32 a) {
  u32 v;
  asm volatile("ld.shared.u8 %0, [%1];" : "=r"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ void mbar_init(u64* b, u32 count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(u64* b, u32 tx) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(tx) : "memory");
}
__device__ __forceinline__ void mbar_arrive(u64* b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ bool mbar_try_wait(u64* b, u32 parity) {
  u32 ok;
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
      "selp.u32 %0, 1, 0, p;\n}\n"
      : "=r"(ok)
      : "r"(smem_u32(b)), "r"(parity)
      : "memory");
  return ok != 0;
}
__device__ __forceinline__ void mbar_wait(u64* b, u32 parity) {
  while (!mbar_try_wait(b, parity)) {
  }
}
// consumer-side wait: back off between polls so that warps waiting for a tile
// leave the issue slots to the warps still working on the previous one (all
// consumer warps must release a stage before it is refilled; a spinning warp
// set can starve the last one and lock the CTA into a slow steady state)
__device__ __forceinline__ void mbar_wait_sleep(u64* b, u32 parity) {
  while (!mbar_try_wait(b, parity)) __nanosleep(WAIT_NS);
}
// consumer-side wait with a suspend-time hint: the warp is parked by the
// hardware until the phase completes (or the hint expires) instead of issuing
// poll/sleep instructions that compete with the working warps
__device__ __forceinline__ void mbar_wait_suspend(u64* b, u32 parity) {
  u32 ok;
  do {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\t"
        "selp.u32 %0, 1, 0, p;\n}\n"
        : "=r"(ok)
        : "r"(smem_u32(b)), "r"(parity), "r"(1000000u)
        : "memory");
  } while (!ok);
}
// the same on a 32-bit shared-window address computed once (a generic pointer makes
// ptxas re-derive the window base from SR_CgaCtaId at every call)
__device__ __forceinline__ void mbar_wait_suspend_a(u32 a, u32 parity) {
  u32 ok;
  do {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\t"
        "selp.u32 %0, 1, 0, p;\n}\n"
        : "=r"(ok)
        : "r"(a), "r"(parity), "r"(1000000u)
        : "memory");
  } while (!ok);
}
__device__ __forceinline__ void mbar_arrive_a(u32 a) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(a) : "memory");
}
__device__ __forceinline__ u64 policy_evict_first() {
  u64 pol;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  return pol;
}
__device__ __forceinline__ void tma_load_1d(void* dst, const void* src, u32 bytes, u64* bar, u64 pol) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(pol)
      : "memory");
}
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void fence_mbar_init() { asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
__device__ __forceinline__ void consumer_bar() { asm volatile("bar.sync 1, %0;" ::"n"(NW * 32) : "memory"); }
__device__ __forceinline__ u32 lanemask_lt() {
  u32 m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

// ---- aggregates
__device__ __forceinline__ i64 agg_identity(int fn) {
  return fn == F_MIN ? HQ_LL_MAX : (fn == F_MAX ? HQ_LL_MIN : 0);
}
__device__ __forceinline__ i64 agg_combine(int fn, i64 a, i64 b) {
  return fn == F_MIN ? (a < b ? a : b) : (fn == F_MAX ? (a > b ? a : b) : a + b);
}
__device__ __forceinline__ i64 warp_reduce(int fn, i64 v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = agg_combine(fn, v, __shfl_xor_sync(HQ_FULL, v, o));
  return v;
}
__device__ __forceinline__ void g_add64(i64* p, i64 v) {
  asm volatile("red.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void g_agg(int fn, i64* t, i64 v, u64 cnt) {
  if (fn == F_MIN) asm volatile("red.global.min.s64 [%0], %1;" ::"l"(t), "l"(v) : "memory");
  else if (fn == F_MAX) asm volatile("red.global.max.s64 [%0], %1;" ::"l"(t), "l"(v) : "memory");
  else g_add64(t, fn == F_COUNT ? (i64)cnt : v);
}
// 64-bit add on shared memory as two native 32-bit atomics with carry
__device__ __forceinline__ void s_add64(u32 a, i64 v) {
  const u32 lo = (u32)v;
  u32 hi = (u32)((u64)v >> 32);
  u32 old;
  asm volatile("atom.shared.add.u32 %0, [%1], %2;" : "=r"(old) : "r"(a), "r"(lo) : "memory");
  hi += (old + lo < old) ? 1u : 0u;
  if (hi) asm volatile("red.shared.add.u32 [%0], %1;" ::"r"(a + 4), "r"(hi) : "memory");
}
__device__ __forceinline__ void s_minmax64(u32 a, i64 v, bool is_min) {
  u64 cur;
  asm volatile("ld.shared.u64 %0, [%1];" : "=l"(cur) : "r"(a) : "memory");
  while (is_min ? v < (i64)cur : v > (i64)cur) {
    u64 prev;
    asm volatile("atom.shared.cas.b64 %0, [%1], %2, %3;" : "=l"(prev) : "r"(a), "l"(cur), "l"(v) : "memory");
    if (prev == cur) break;
    cur = prev;
  }
}
__device__ __forceinline__ void s_agg(int fn, u32 t, i64 v, u64 cnt) {
  if (fn == F_MIN) s_minmax64(t, v, true);
  else if (fn == F_MAX) s_minmax64(t, v, false);
  else s_add64(t, fn == F_COUNT ? (i64)cnt : v);
}
__device__ __forceinline__ u32 hash64(u64 k, int log2) { return (u32)((k * 0x9E3779B97F4A7C15ull) >> (64 - log2)); }

// global group table: dense [count, agg...] rows, or hash entries [key, count, agg...]
__device__ __forceinline__ i64* global_locate(const JParams& p, u64 key) {
  if (GMODE != 2) return p.gtab + key * VWORDS;
  u64 h = hash64(key, p.glog2);
  for (u64 i = 0; i <= p.gmask; ++i) {
    u64* kp = (u64*)(p.gtab + h * (VWORDS + 1));
    const u64 k = *(volatile u64*)kp;
    if (k == key) return (i64*)kp + 1;
    if (k == HQ_EMPTY_KEY) {
      const u64 old = atomicCAS(kp, HQ_EMPTY_KEY, key);
      if (old == HQ_EMPTY_KEY || old == key) return (i64*)kp + 1;
    }
    h = (h + 1) & p.gmask;
  }
  atomicOr(p.err, F_GROUP_FULL);
  return 0;
}
// shared pre-aggregation table entry (dense or hash), 0 when the hash is full.
// sl0: the 32-bit shared address of this warp's copy of a dense table, taken once per
// kernel (recomputing it per update cost a generic->shared conversion, a thread-index
// read and a modulo by SCOPIES every time: ~8 % of SSB Q3.1's instructions)
__device__ __forceinline__ u32 local_locate(char* sagg, u32 sl0, u64 key) {
  if (SMODE == 1) return sl0 + (u32)key * (u32)(LVWORDS * 8);
  if (SMODE == 2) {
    u64* keys = (u64*)sagg;
    i64* ent = (i64*)sagg + SMEM_CAP;
    u32 h = hash64(key, SLOG2);
#pragma unroll 1
    for (int i = 0; i < 32; ++i) {
      const u64 k = keys[h];
      bool hit = k == key;
      if (!hit && k == HQ_EMPTY_KEY) {
        const u64 old = atomicCAS(keys + h, HQ_EMPTY_KEY, key);
        hit = old == HQ_EMPTY_KEY || old == key;
      }
      if (hit) return smem_u32(ent + (u64)h * LVWORDS);
      h = (h + 1) & (SMEM_CAP - 1);
    }
  }
  return 0u;
}
// add (cnt, vals) to the group entry: shared when the local table holds it, else global
__device__ __forceinline__ void group_update(const JParams& p, char* sagg, u32 sl0, u64 key, bool local, u64 cnt,
                                             const i64 (&vals)[NAGGS > 0 ? NAGGS : 1]) {
  const u32 sa = (local && SMODE != 0) ? local_locate(sagg, sl0, key) : 0u;
  if (sa) {
    // the per-CTA count of a group stays below 2^32: a return-less 32-bit red on
    // the low word; COUNT aggregates are read from it at the merge
    asm volatile("red.shared.add.u32 [%0], %1;" ::"r"(sa), "r"((u32)cnt) : "memory");
#pragma unroll
    for (int a = 0; a < NAGGS; ++a)
      if (AGG_FN[a] != F_COUNT) s_agg(AGG_FN[a], sa + 8u * LCOL[a], vals[a], cnt);
    return;
  }
  i64* e = global_locate(p, key);
  if (!e) return;
  g_add64(e, (i64)cnt);
#pragma unroll
  for (int a = 0; a < NAGGS; ++a) g_agg(AGG_FN[a], e + 1 + a, vals[a], cnt);
}
