// hq_plan.cu -- validation of an hq_plan and its translation into the fused
// kernel's device plan (KPlan): register map, TMA stage layout, shared-memory
// budget, sink tables.  One plan = one fusion operator (§4.1).
#include <algorithm>
#include <climits>
#include <cstring>

#include "hq_internal.h"

using namespace hqk;

namespace {

int64_t next_pow2(int64_t x) {
  int64_t c = 1;
  while (c < x) c <<= 1;
  return c;
}
uint32_t align_up(uint32_t x, uint32_t a) { return (x + a - 1) / a * a; }

// barriers, block-scan and reduction scratch: full/empty[10], base[32], wtot[32], red[32][9]

struct RegInfo {
  int width = 0;       // 0 = undefined
  bool is_col = false;
};

// external register id -> internal index (columns 0..15, temporaries 16..23)
int reg_index(int32_t reg, int ncols) {
  if (reg >= 0 && reg < ncols) return reg;
  if (reg >= HQ_TMP(0) && reg < HQ_TMP(HQ_MAX_TMP)) return HQ_MAX_COLS + (reg - HQ_TMP(0));
  return -1;
}

void fold_pred(const hq_pred& in, KPred& out, int16_t reg) {
  out.reg = reg;
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
    default: HQ_THROW(HQ_ERR_ARG, "unknown comparison in filter");
  }
  // int32 fast path bounds (an empty range stays empty after clamping)
  if (out.lo > out.hi || out.lo > INT_MAX || out.hi < INT_MIN) {
    out.lo32 = 1;
    out.hi32 = 0;
  } else {
    out.lo32 = (int32_t)std::max<int64_t>(out.lo, INT_MIN);
    out.hi32 = (int32_t)std::min<int64_t>(out.hi, INT_MAX);
  }
}

}  // namespace

int hq_type_width(int type) {
  switch (type) {
    case HQ_I8: return 1;
    case HQ_I32: return 4;
    case HQ_I64: return 8;
    case HQ_F64: return 8;
  }
  return 0;
}

// Build the device plan; allocates the result's sink buffers on first use.
void hq_build_kplan(hq_ctx* ctx, hq_result* r, KPlan& kp, int64_t group_cap, int64_t mat_cap, bool jit, int mp_pass) {
  const hq_plan& P = r->plan;
  const hq_table* F = r->fact;
  std::memset(&kp, 0, sizeof(kp));
  const int64_t rb = P.row_begin, re = P.row_end < 0 ? F->nrows : P.row_end;
  if (rb < 0 || re < rb || re > F->nrows) HQ_THROW(HQ_ERR_ARG, "plan: row range outside the fact table");
  kp.row_begin = rb;
  kp.row_end = re;
  if (P.nops < 0 || P.nops > HQ_MAX_OPS) HQ_THROW(HQ_ERR_UNSUPPORTED, "plan: too many ops");

  RegInfo regs[NREGS];
  bool col_used[HQ_MAX_COLS] = {false};
  for (int c = 0; c < F->ncols; ++c) {
    regs[c].width = F->cols[c].width;
    regs[c].is_col = true;
  }
  auto use = [&](int32_t reg, const char* what) -> int {
    const int i = reg_index(reg, F->ncols);
    if (i < 0 || regs[i].width == 0)
      HQ_THROW(HQ_ERR_ARG, std::string("plan: ") + what + " reads an undefined register " + std::to_string(reg));
    if (i < HQ_MAX_COLS) col_used[i] = true;
    return i;
  };
  auto def = [&](int32_t reg, int width, const char* what) -> int {
    const int i = reg_index(reg, F->ncols);
    if (i < HQ_MAX_COLS) HQ_THROW(HQ_ERR_ARG, std::string("plan: ") + what + " must write a temporary HQ_TMP(k)");
    if (regs[i].width != 0 && regs[i].width != width)
      HQ_THROW(HQ_ERR_ARG, std::string("plan: temporary redefined with another type by ") + what);
    regs[i].width = width;
    return i;
  };

  int npred = 0, nprobe = 0, ncomp = 0, ninsn = 0;
  kp.nops = P.nops;
  for (int o = 0; o < P.nops; ++o) {
    const hq_op& op = P.ops[o];
    if (op.kind == HQ_OP_FILTER) {
      if (npred >= MAX_PREDS) HQ_THROW(HQ_ERR_UNSUPPORTED, "plan: too many filters");
      const int i = use(op.filter.reg, "filter");
      fold_pred(op.filter, kp.preds[npred], (int16_t)i);
      kp.ops[o] = {OP_FILTER, (uint8_t)npred++};
    } else if (op.kind == HQ_OP_PROBE) {
      if (nprobe >= MAX_PROBES) HQ_THROW(HQ_ERR_UNSUPPORTED, "plan: too many probes");
      if (!op.ht) HQ_THROW(HQ_ERR_ARG, "plan: probe without hash table");
      if (op.mode < HQ_PROBE_INNER || op.mode > HQ_PROBE_OUTER) HQ_THROW(HQ_ERR_ARG, "plan: bad probe mode");
      KProbe& pr = kp.probes[nprobe];
      pr.key_reg = (int16_t)use(op.key_reg, "probe key");
      // generated kernels read a direct table's compact form; the other executions its slots
      pr.slots = jit ? op.ht->slots : hq_hash_slots(ctx, const_cast<hq_hash*>(op.ht));
      pr.direct = op.ht->meta.layout == HQ_HT_DIRECT;
      pr.mask = pr.direct ? (uint32_t)op.ht->meta.capacity : (uint32_t)(op.ht->meta.capacity - 1);
      pr.dmin = (int32_t)op.ht->meta.key_min;
      pr.log2cap = (uint8_t)op.ht->log2cap;
      // a ranked sparse-key table (hq_hash::ranked): generated kernels probe its bitmap,
      // directory and payload rows; the other executions its derived slot array
      const bool rk = op.ht->ranked();
      pr.ranked = (uint8_t)(jit && rk);
      pr.ckind = rk ? 0 : (uint8_t)op.ht->ckind;
      pr.crank = (uint8_t)op.ht->crank;
      pr.compact = rk ? nullptr : op.ht->compact_ptr();
      pr.rstride = (uint8_t)op.ht->rstride;
      pr.rpay = nullptr;
      pr.pay_min = op.ht->meta.pay_min;
      pr.pay_max = op.ht->meta.pay_max;
      for (int k = 0; k < 4; ++k) pr.pay_set[k] = op.ht->meta.pay_set[k];
      {  // uniform foreign keys over the key range: pass fraction = key density (anti: the rest);
         // pass_src: over the build side's source rows (star joins: qualifying / all dimension
         // rows -- SSB Q1.2's date table, 31 of 2,557 days, is dense over its own key range)
        const double range = (double)op.ht->meta.key_max - (double)op.ht->meta.key_min + 1.0;
        double est = (op.ht->meta.nkeys >= 0 && range >= 1.0) ? (double)op.ht->meta.nkeys / range : 1.0;
        est = est > 1.0 ? 1.0 : est;
        double src = est;
        if (op.ht->meta.nkeys >= 0 && op.ht->src_rows > 0)
          src = std::min(est, (double)op.ht->meta.nkeys / (double)op.ht->src_rows);
        pr.pass_est = (float)(op.mode == HQ_PROBE_ANTI ? 1.0 - est : (op.mode == HQ_PROBE_OUTER ? 1.0 : est));
        pr.pass_src = (float)(op.mode == HQ_PROBE_ANTI ? 1.0 - src : (op.mode == HQ_PROBE_OUTER ? 1.0 : src));
      }
      pr.cbytes = rk ? 0u : (uint32_t)op.ht->cbytes;
      pr.smem_off = 0;
      pr.pf = op.ht->pf_words ? op.ht->prefilter.as<uint32_t>() : nullptr;
      if (pr.ranked) {
        const char* base = (const char*)op.ht->compact_ptr();
        pr.pf = (const uint32_t*)base;  // bitmap words, or {bits, dir} pairs when the table has payloads
        if (pr.rstride) pr.rpay = (const int32_t*)(base + op.ht->roff_pay);
      }
      pr.pf_min = (int32_t)op.ht->meta.key_min;
      pr.pf_range = (uint32_t)((int64_t)op.ht->meta.key_max - op.ht->meta.key_min + 1);
      pr.words = (uint8_t)op.ht->meta.slot_words;
      pr.mode = (uint8_t)op.mode;
      const int npay = hq_probe_has_payload(op.mode) ? op.npayload : 0;
      pr.composite = op.ht->meta.composite ? 1 : 0;
      pr.key2_reg = 0;
      if (pr.composite) {  // two-column key: payload word 0 is the second key
        pr.key2_reg = (int16_t)use(op.key2_reg, "probe second key");
        pr.pay_min = 1;  // payload ranges of the count pass describe the second key, not the payloads
        pr.pay_max = 0;
        for (int k = 0; k < 4; ++k) pr.pay_set[k] = 0;
      }
      if (npay < 0 || npay > op.ht->meta.npayload - pr.composite)
        HQ_THROW(HQ_ERR_ARG, "plan: probe asks for more payload words than the table holds");
      pr.npay = (uint8_t)npay;
      for (int k = 0; k < npay; ++k) pr.dst[k] = (int16_t)def(op.payload_dst[k], 4, "probe payload");
      kp.ops[o] = {OP_PROBE, (uint8_t)nprobe++};
    } else if (op.kind == HQ_OP_COMPUTE) {
      if (ncomp >= MAX_COMPUTES) HQ_THROW(HQ_ERR_UNSUPPORTED, "plan: too many compute ops");
      if (op.ninsn < 1 || op.ninsn > HQ_MAX_INSN || ninsn + op.ninsn > MAX_INSNS)
        HQ_THROW(HQ_ERR_UNSUPPORTED, "plan: expression length");
      if (op.code[0].opc != HQ_I_LOAD) HQ_THROW(HQ_ERR_ARG, "plan: expression must start with HQ_I_LOAD");
      KCompute& c = kp.comps[ncomp];
      c.first = (uint8_t)ninsn;
      c.n = (uint8_t)op.ninsn;
      for (int k = 0; k < op.ninsn; ++k) {
        const hq_insn& in = op.code[k];
        if (in.opc < HQ_I_LOAD || in.opc > HQ_I_OR) HQ_THROW(HQ_ERR_ARG, "plan: bad opcode");
        if (in.opc >= HQ_I_AND_EQ && in.opc <= HQ_I_AND_IN && in.reg < 0)
          HQ_THROW(HQ_ERR_ARG, "plan: predicate instruction needs a register operand");
        KInsn& ki = kp.insns[ninsn++];
        ki.opc = (uint8_t)in.opc;
        ki.reg = in.reg < 0 ? (int16_t)-1 : (int16_t)use(in.reg, "expression");
        ki.imm = in.imm;
      }
      c.dst = (int16_t)def(op.dst, 8, "compute");
      kp.ops[o] = {OP_COMPUTE, (uint8_t)ncomp++};
    } else {
      HQ_THROW(HQ_ERR_ARG, "plan: unknown op kind");
    }
  }

  // ---- sink
  kp.sink = P.sink;
  kp.resolution = P.resolution;
  if (P.resolution != HQ_RES_LRGP && P.resolution != HQ_RES_ATOMIC && P.resolution != HQ_RES_WE)
    HQ_THROW(HQ_ERR_ARG, "plan: bad resolution");
  const bool we = P.resolution == HQ_RES_WE;
  if (we && (!jit || mp_pass))
    HQ_THROW(HQ_ERR_UNSUPPORTED, "Resolution:WE is implemented by the generated fused kernel only (HQ_EXEC_FUSED)");
  uint32_t agg_smem = 0;
  if (P.sink == HQ_SINK_AGG) {
    if (P.nkeys < 0 || P.nkeys > HQ_MAX_KEYS) HQ_THROW(HQ_ERR_UNSUPPORTED, "plan: 0..4 group keys");
    if (P.naggs < 0 || P.naggs > HQ_MAX_AGGS) HQ_THROW(HQ_ERR_UNSUPPORTED, "plan: 0..8 aggregates");
    kp.nkeys = P.nkeys;
    __int128 prod = 1;
    for (int i = 0; i < P.nkeys; ++i) {
      if (P.key_card[i] <= 0) HQ_THROW(HQ_ERR_ARG, "plan: key cardinality must be > 0");
      kp.key_reg[i] = (int16_t)use(P.key_reg[i], "group key");
      kp.key_min[i] = P.key_min[i];
      kp.key_card[i] = P.key_card[i];
      prod *= P.key_card[i];
      if (prod >= ((__int128)1 << 62)) HQ_THROW(HQ_ERR_UNSUPPORTED, "plan: packed group key exceeds 62 bits");
    }
    int64_t st = 1;
    for (int i = P.nkeys - 1; i >= 0; --i) {
      kp.key_stride[i] = st;
      st *= P.key_card[i];
    }
    const int64_t ngroups = (int64_t)prod;
    kp.naggs = P.naggs;
    for (int a = 0; a < P.naggs; ++a) {
      if (P.agg_fn[a] < HQ_AGG_SUM || P.agg_fn[a] > HQ_AGG_AVG) HQ_THROW(HQ_ERR_ARG, "plan: bad aggregate");
      kp.agg_fn[a] = (uint8_t)P.agg_fn[a];
      kp.agg_reg[a] = P.agg_fn[a] == HQ_AGG_COUNT ? (int16_t)0 : (int16_t)use(P.agg_reg[a], "aggregate");
    }
    kp.vwords = 1 + P.naggs;
    kp.lvwords = 1;
    for (int a = 0; a < P.naggs; ++a) {  // interpreter: the global layout; generated: COUNTs share word 0
      if (jit && P.agg_fn[a] == HQ_AGG_COUNT) kp.lcol[a] = 0;
      else kp.lcol[a] = (uint8_t)kp.lvwords++;
    }
    // a dense global table for a tight but large key domain (fused execution): no hash
    // claim round trip per group update, when it is at most twice the hash table's size
    auto dense_global = [&](int64_t ng) {
      if (P.exec != HQ_EXEC_FUSED && P.exec != HQ_EXEC_FUSED_INTERP) return false;
      if (ng > DENSE_GLOBAL_LIMIT) return false;
      int64_t hcap = group_cap > 0 ? group_cap : (P.group_capacity > 0 ? P.group_capacity : std::min<int64_t>(ng, 1 << 20));
      hcap = std::max<int64_t>(1024, next_pow2(hcap * 2));
      return (__int128)ng * kp.vwords <= (__int128)2 * hcap * (kp.vwords + 1);
    };
    if (P.nkeys == 0) {
      kp.gmode = GM_SCALAR;
      r->ngroups = 1;
    } else if (ngroups <= DENSE_LIMIT || dense_global(ngroups)) {
      kp.gmode = GM_DENSE;
      r->ngroups = ngroups;
    } else {
      kp.gmode = GM_HASH;
      int64_t cap = group_cap > 0 ? group_cap : (P.group_capacity > 0 ? P.group_capacity : std::min<int64_t>(ngroups, 1 << 20));
      cap = std::max<int64_t>(1024, next_pow2(cap * 2));
      r->ngroups = cap;
      kp.gmask = (uint64_t)(cap - 1);
      int l = 0;
      while ((1LL << l) < cap) ++l;
      kp.glog2 = l;
    }
    r->gmode = kp.gmode;
    r->vwords = kp.vwords;
    const size_t gbytes = (size_t)r->ngroups * (kp.vwords + (kp.gmode == GM_HASH ? 1 : 0)) * 8;
    if (!r->gtab.p || r->gtab.bytes < gbytes) r->gtab = DevBuf(ctx, gbytes);
    kp.gtab = r->gtab.as<long long>();
    // deduplicated accumulators for the lane-private mode: 0 = count,
    // SUM/AVG of one register share one sum, MIN/MAX get their own
    kp.nacc = 1;
    kp.acc_fn[0] = HQ_AGG_COUNT;
    kp.acc_reg[0] = 0;
    for (int a = 0; a < P.naggs; ++a) {
      const uint8_t cls = (P.agg_fn[a] == HQ_AGG_AVG) ? (uint8_t)HQ_AGG_SUM : (uint8_t)P.agg_fn[a];
      if (cls == HQ_AGG_COUNT) { kp.acc_of[a] = 0; continue; }
      int found = -1;
      for (int k = 1; k < kp.nacc; ++k)
        if (kp.acc_fn[k] == cls && kp.acc_reg[k] == kp.agg_reg[a]) found = k;
      if (found < 0) {
        found = kp.nacc++;
        kp.acc_fn[found] = cls;
        kp.acc_reg[found] = kp.agg_reg[a];
      }
      kp.acc_of[a] = (uint8_t)found;
    }
    // Generated kernels: a group key that is payload 0 of an inner probe only
    // takes the payload's value range (count pass), e.g. SSB Q3.1 c_nation of the
    // ASIA customers spans 14 of the declared 25 values -- the shared table can
    // be dense over the narrowed domain where the declared one needs a hash.
    int64_t lmin[HQ_MAX_KEYS], lcard[HQ_MAX_KEYS];
    __int128 lgroups = 1;
    for (int i = 0; i < P.nkeys; ++i) {
      lmin[i] = kp.key_min[i];
      lcard[i] = kp.key_card[i];
      for (int q = 0; jit && q < nprobe; ++q) {
        const KProbe& pr = kp.probes[q];
        if (pr.mode != HQ_PROBE_INNER || pr.npay < 1 || pr.dst[0] != kp.key_reg[i] || pr.pay_min > pr.pay_max) continue;
        if (pr.pay_min < kp.key_min[i] || (int64_t)pr.pay_max >= kp.key_min[i] + kp.key_card[i]) continue;
        lmin[i] = pr.pay_min;
        lcard[i] = (int64_t)pr.pay_max - pr.pay_min + 1;
        for (int k = 0; k < 4; ++k) kp.lkey_set[i][k] = 0;
        if (lcard[i] <= 256) {  // distinct payload values (count pass): index by rank
          int64_t n = 0;
          uint64_t rel[4] = {0, 0, 0, 0};
          for (int64_t d = 0; d < lcard[i]; ++d) {
            const uint32_t v = (uint32_t)(pr.pay_min + d) & 255u;
            if ((pr.pay_set[v >> 6] >> (v & 63)) & 1ull) {
              rel[d >> 6] |= 1ull << (d & 63);
              ++n;
            }
          }
          if (n > 0 && n < lcard[i]) {
            lcard[i] = n;
            for (int k = 0; k < 4; ++k) kp.lkey_set[i][k] = rel[k];
          }
        }
      }
      lgroups *= lcard[i];
    }
    // local-resolution table in shared memory: 32 KB, or for a probe-free generated
    // kernel (nothing else competes for shared memory) whatever the TMA ring leaves
    // with 3 stages of the 2-rows-per-lane tile (Exp 2: up to 8,192 groups
    // keep their pre-aggregation in shared memory)
    uint64_t agg_budget = SMEM_AGG_BYTES;
    if (jit && nprobe == 0 && !mp_pass) {
      uint32_t rb = 0;
      for (int c = 0; c < F->ncols; ++c) rb += col_used[c] ? (uint32_t)F->cols[c].width : 0u;
      const uint64_t stage = align_up(31u * 32u * 2u * std::max<uint32_t>(rb, 1u), 128);
      const uint64_t avail = ctx->max_smem > MISC_BYTES + 3 * stage + 1024 ? ctx->max_smem - MISC_BYTES - 3 * stage - 1024 : 0;
      agg_budget = std::max<uint64_t>(agg_budget, avail / 128 * 128);
    }
    const uint32_t lvw = kp.lvwords;
    // a group key narrowed to the rank of a rank-coded byte map (hq_build_compact) indexes
    // the shared table with the probe's byte itself: prefer the narrowed table then
    bool ranked_narrow = false;
    for (int i = 0; jit && i < P.nkeys; ++i) {
      if (!(kp.lkey_set[i][0] | kp.lkey_set[i][1] | kp.lkey_set[i][2] | kp.lkey_set[i][3])) continue;
      for (int q = 0; q < nprobe; ++q)
        if (kp.probes[q].dst[0] == kp.key_reg[i] && kp.probes[q].crank && kp.probes[q].ckind == 2 && kp.probes[q].npay > 0)
          ranked_narrow = true;
    }
    kp.smode = SM_NONE;
    if (P.nkeys > 0 && P.resolution == HQ_RES_LRGP) {
      // lane-private tables halve the warps, so only for probe-free pipelines
      // (no latency to hide) whose group domain is tiny
      if (kp.gmode == GM_DENSE && nprobe == 0 &&
          (uint64_t)ngroups * kp.nacc * LANE_NW * 32 * 8 <= (uint64_t)SMEM_LANE_BYTES) {
        kp.smode = SM_LANE;  // tiny domain (e.g. TPC-H Q1): contention-free lane-private tables
        kp.smem_cap = (uint32_t)ngroups;
        agg_smem = (uint32_t)(ngroups * kp.nacc * LANE_NW * 32 * 8);
      } else if (kp.gmode == GM_DENSE && (uint64_t)ngroups * lvw * 8 <= agg_budget && !(ranked_narrow && lgroups < (__int128)ngroups)) {
        kp.smode = SM_DENSE;
        kp.smem_cap = (uint32_t)ngroups;
        agg_smem = (uint32_t)(ngroups * lvw * 8);
      } else if (lgroups < (__int128)ngroups && lgroups * lvw * 8 <= (__int128)agg_budget) {
        kp.smode = SM_DENSE;  // dense over the narrowed domain; merged into the global table by key
        kp.local_keys = 1;
        kp.smem_cap = (uint32_t)lgroups;
        agg_smem = (uint32_t)(lgroups * lvw * 8);
        int64_t st2 = 1;
        for (int i = P.nkeys - 1; i >= 0; --i) {
          kp.lkey_min[i] = lmin[i];
          kp.lkey_stride[i] = st2;
          st2 *= lcard[i];
        }
      } else {
        uint32_t cap = agg_budget > SMEM_AGG_BYTES ? 16384 : 4096;
        while (cap > 64 && (uint64_t)cap * (lvw + 1) * 8 > agg_budget) cap >>= 1;
        // far more groups than the shared table holds (TPC-H Q3: ~10^5-10^6
        // orderkeys): it would fill up and every later row would scan it before
        // going to global memory -- update the global table directly (C2)
        // (a dense domain larger than the table: as many groups as the domain)
        const int64_t expect = kp.gmode == GM_DENSE ? ngroups : (group_cap > 0 ? group_cap : P.group_capacity);
        const char* nl = getenv("HQ_JIT_NOLOCAL");
        if (jit && expect > (kp.gmode == GM_DENSE ? 1 : 4) * (int64_t)cap && !(nl && nl[0] == '0')) {
          kp.smode = SM_NONE;
          // per-warp update queues in front of the global hash table (hq_jit.cu): 16 rows
          // per warp, for the 31 warps of the widest layout
          if (kp.gmode == GM_HASH && !mp_pass && P.resolution == HQ_RES_LRGP && !getenv("HQ_JIT_NOGQ")) {
            kp.gq_cap = 16;
            if (const char* e = getenv("HQ_JIT_GQ")) kp.gq_cap = (uint16_t)std::max(1, std::min(64, atoi(e)));  // A/B
            agg_smem = 31u * kp.gq_cap * (2u + (uint32_t)P.naggs) * 8u;
          }
        } else {
        kp.smode = SM_HASH;
        kp.smem_cap = cap;
        int l = 0;
        while ((1u << l) < cap) ++l;
        kp.slog2 = l;
        agg_smem = cap * (lvw + 1) * 8;
        }
      }
    }
  } else if (P.sink == HQ_SINK_MATERIALISE) {
    if (P.nout < 1 || P.nout > HQ_MAX_OUT) HQ_THROW(HQ_ERR_UNSUPPORTED, "plan: 1..8 output columns");
    const int64_t cap = mat_cap > 0 ? mat_cap : (P.capacity > 0 ? P.capacity : std::max<int64_t>(re - rb, 0));
    const bool realloc = (int)r->outcols.size() != P.nout || r->capacity < cap;
    if (realloc) r->outcols.clear();
    kp.nout = P.nout;
    for (int j = 0; j < P.nout; ++j) {
      kp.out_reg[j] = (int16_t)use(P.out_reg[j], "output column");
      const int w = hq_type_width(P.out_type[j]);
      if (w == 0 || P.out_type[j] == HQ_F64) HQ_THROW(HQ_ERR_ARG, "plan: output type must be HQ_I8/I32/I64");
      kp.out_width[j] = (uint8_t)w;
      if (realloc) r->outcols.emplace_back(ctx, (size_t)std::max<int64_t>(cap, 1) * w + 16);
      kp.out_ptr[j] = r->outcols[j].p;
    }
    r->capacity = std::max(r->capacity, cap);
    kp.capacity = r->capacity;
  } else {
    HQ_THROW(HQ_ERR_ARG, "plan: bad sink");
  }

  // Generated kernels: replicas of a small dense shared table, so that the 31
  // consumer warps do not serialise on the same few entries (Exp 2 with 32-512
  // groups: one table measured 6-9x slower than the tiny lane-private domains)
  kp.scopies = 1;
  if (jit && kp.smode == SM_DENSE && !mp_pass) {
    // every row updates a probe-free pipeline's table; behind selective probes
    // (star joins: 1-4 % of the rows) contention is low and the shared memory
    // is worth more to the staged probe tables and the TMA ring
    const uint64_t one = (uint64_t)kp.smem_cap * kp.lvwords * 8;
    const uint64_t budget = nprobe == 0 ? (uint64_t)SMEM_AGG_BYTES : 16384;
    uint32_t c = 1;
    // behind probes: up to 4 replicas within 16 KB (SSB Q4.1 SF100 7 replicas 2.197 ms, 4:
    // 2.167 ms; Q3.1 SF30 1 replica 0.485 ms, 4: 0.473 ms, 16: 0.529 ms, measured)
    while (c < (nprobe == 0 ? 31u : 4u) && one * (c + 1) <= budget) ++c;
    if (const char* e = getenv("HQ_JIT_SCOPIES")) c = std::max(1, std::min(31, atoi(e)));
    kp.scopies = c;
    agg_smem = (uint32_t)(one * c);
  }

  // Resolution:WE (hq_jit.cu gen_we_tile): 16 consumer warps (a power-of-two tree),
  // the tile's scratch in the aggregation region: B3 [1 + naggs][512] int64, A3 [512]
  // int32, C3 512 x (key, count, naggs values, head flag) at one row per lane
  if (we) {
    const uint32_t nt = (uint32_t)NW * 32;
    if (P.sink == HQ_SINK_MATERIALISE) agg_smem = nt * 4;
    else if (P.nkeys == 0) agg_smem = (1u + (uint32_t)P.naggs) * nt * 8;
    else agg_smem = nt * (8u + 8u + 8u * (uint32_t)std::max(P.naggs, 1) + 4u);
  }

  // ---- multi-pass (hq_multipass.cu): which ops a pass executes and which
  // columns it reads (backward liveness).  Count kernel: selections, probes and
  // the computes feeding them; write kernel: inner probes and computes whose
  // results reach the sink, plus the flag and position columns.
  kp.mp_pass = (uint8_t)mp_pass;
  kp.mp_flag_reg = kp.mp_pos_reg = -1;
  int ncols_all = F->ncols;
  const char* colptr[HQ_MAX_COLS];
  int colw[HQ_MAX_COLS];
  for (int c = 0; c < F->ncols; ++c) {
    colptr[c] = (const char*)F->cols[c].ptr;
    colw[c] = F->cols[c].width;
  }
  if (mp_pass) {
    if (!jit) HQ_THROW(HQ_ERR_UNSUPPORTED, "multi-pass execution needs generated kernels (HQ_JIT=0 is set)");
    bool need[NREGS] = {false};
    if (mp_pass == 2) {
      if (P.sink == HQ_SINK_MATERIALISE) {
        for (int j = 0; j < kp.nout; ++j) need[kp.out_reg[j]] = true;
      } else {
        for (int i = 0; i < kp.nkeys; ++i) need[kp.key_reg[i]] = true;
        for (int a = 0; a < kp.naggs; ++a)
          if (kp.agg_fn[a] != HQ_AGG_COUNT) need[kp.agg_reg[a]] = true;
      }
    }
    for (int o = kp.nops - 1; o >= 0; --o) {
      const KOp& op = kp.ops[o];
      bool exec = false;
      if (op.kind == OP_FILTER) {
        exec = mp_pass == 1;
        if (exec) need[kp.preds[op.idx].reg] = true;
      } else if (op.kind == OP_PROBE) {
        const KProbe& pr = kp.probes[op.idx];
        exec = mp_pass == 1;
        for (int k = 0; mp_pass == 2 && hq_probe_has_payload(pr.mode) && k < pr.npay; ++k) exec = exec || need[pr.dst[k]];
        if (exec) need[pr.key_reg] = true;
        if (exec && pr.composite) need[pr.key2_reg] = true;
      } else {
        const KCompute& c = kp.comps[op.idx];
        exec = need[c.dst];
        for (int k = 0; exec && k < c.n; ++k)
          if (kp.insns[c.first + k].reg >= 0) need[kp.insns[c.first + k].reg] = true;
      }
      kp.op_skip[o] = exec ? 0 : 1;
    }
    for (int c = 0; c < F->ncols; ++c) col_used[c] = need[c];
    if (mp_pass == 2) {
      if (F->ncols + 2 > HQ_MAX_COLS) HQ_THROW(HQ_ERR_UNSUPPORTED, "multi-pass: no column slots left for flags/positions");
      kp.mp_flag_reg = (int16_t)F->ncols;
      kp.mp_pos_reg = (int16_t)(F->ncols + 1);
      colptr[F->ncols] = r->mp_flags_col;
      colptr[F->ncols + 1] = r->mp_pos_col;
      colw[F->ncols] = colw[F->ncols + 1] = 4;
      col_used[F->ncols] = col_used[F->ncols + 1] = true;
      ncols_all = F->ncols + 2;
    }
    // both passes write plain arrays: no shared pre-aggregation table
    kp.smode = SM_NONE;
    kp.local_keys = 0;
    agg_smem = 0;
  }

  // ---- lazy columns (generated kernels): a fact column first read where only a few rows
  // are still expected to be live (the paper's lazy loading, Table 3) is not
  // streamed; the live rows read it from global memory at its first use.  Expected
  // survival before op i = product of the earlier ops' estimates (probe: build-side key
  // density; filter: 1/2; compute: 1); lazy when <= 15 %.
  bool lazy[HQ_MAX_COLS] = {false};
  if (jit && !mp_pass && !getenv("HQ_JIT_NOLAZY")) {
    int first[HQ_MAX_COLS];
    for (int c = 0; c < HQ_MAX_COLS; ++c) first[c] = -1;
    auto mark = [&](int reg, int at) {
      if (reg >= 0 && reg < F->ncols && first[reg] < 0) first[reg] = at;
    };
    for (int o = 0; o < kp.nops; ++o) {
      const KOp& op = kp.ops[o];
      if (op.kind == OP_FILTER) mark(kp.preds[op.idx].reg, o);
      else if (op.kind == OP_PROBE) {
        mark(kp.probes[op.idx].key_reg, o);
        if (kp.probes[op.idx].composite) mark(kp.probes[op.idx].key2_reg, o);
      } else {
        const KCompute& c = kp.comps[op.idx];
        for (int k = 0; k < c.n; ++k) mark(kp.insns[c.first + k].reg, o);
      }
    }
    for (int c = 0; c < F->ncols; ++c)
      if (col_used[c] && first[c] < 0) first[c] = kp.nops;  // read by the sink only
    double est[HQ_MAX_OPS + 1];
    est[0] = 1.0;
    for (int o = 0; o < kp.nops; ++o) {
      const KOp& op = kp.ops[o];
      const double e = op.kind == OP_FILTER ? 0.5 : (op.kind == OP_PROBE ? (double)kp.probes[op.idx].pass_src : 1.0);
      est[o + 1] = est[o] * e;
    }
    // only where the rows wait on no global-memory probe: a lazy load is one more
    // dependent DRAM round trip per tile, which HBM-bound pipelines hide (TPC-H Q6 SF10
    // 0.248 -> 0.196 ms) but latency-bound star joins do not (SSB Q3.1 SF30 0.56 -> 0.97,
    // Q4.1 SF100 2.48 -> 3.45 ms, measured)
    uint64_t ctab = 0;
    bool stageable = true;
    for (int q = 0; q < nprobe; ++q) {
      const KProbe& pr = kp.probes[q];
      stageable = stageable && pr.direct && pr.ckind;
      ctab += (pr.cbytes + 127) / 128 * 128;
    }
    stageable = stageable && ctab <= 64 * 1024;
    for (int c = 0; c < F->ncols; ++c)
      lazy[c] = stageable && col_used[c] && first[c] > 0 && est[first[c]] <= 0.15;
  }
  // ---- stage layout: only referenced columns are streamed
  kp.ncols = 0;
  uint32_t rowbytes = 0;
  for (int c = 0; c < ncols_all; ++c) {
    if (!col_used[c] || lazy[c]) continue;
    // (host-streamed columns are copied into 256-B aligned ring slots)
    if (!F->host_stream && ((uintptr_t)colptr[c] & 15) != 0) HQ_THROW(HQ_ERR_ARG, "column pointer not 16-byte aligned");
    rowbytes += (uint32_t)colw[c];
  }
  uint32_t tmp_row = 0;  // generated kernels keep temporaries in registers
  if (!jit)
    for (int k = 0; k < HQ_MAX_TMP; ++k) tmp_row += (uint32_t)regs[HQ_MAX_COLS + k].width;

  kp.nw = kp.smode == SM_LANE ? LANE_NW : NW;
  int force_R = 0;
  if (jit && kp.smode != SM_LANE) {
    // generated kernels need fewer registers: 31 consumer warps x 2 rows per lane
    // hides the probe/atomic latency best (sweep on B200, profiles/r01)
    kp.nw = 31;
    force_R = 2;
    if (const char* e = getenv("HQ_JIT_NW")) kp.nw = std::max(1, std::min(31, atoi(e)));
    if (const char* e = getenv("HQ_JIT_R")) force_R = atoi(e);
  }
  if (we) {  // the WE trees need a power-of-two thread count; C3-WE sorts one row per lane
    kp.nw = NW;
    force_R = (P.sink == HQ_SINK_AGG && P.nkeys > 0) ? 1 : 2;
  }
  // Generated kernels stage small compact probe tables (bitmaps / byte arrays of
  // direct tables) in shared memory, earliest probes first (they see the most
  // rows), as long as the TMA ring keeps >= 3 stages.
  int staged[MAX_PROBES];
  int nstaged = 0;
  const uint32_t stage_budget = 96 * 1024;
  if (jit) {
    uint32_t total = 0;
    for (int o = 0; o < kp.nops; ++o) {
      if (kp.ops[o].kind != OP_PROBE) continue;
      const KProbe& pr = kp.probes[kp.ops[o].idx];
      if (!pr.ckind || pr.cbytes == 0) continue;
      const uint32_t b = align_up(pr.cbytes, 128);
      if (total + b > stage_budget) continue;
      total += b;
      staged[nstaged++] = kp.ops[o].idx;
    }
  }
  // Generated kernels whose probes all read shared-memory-staged tables (or that
  // have none) wait on no global round trip per row: 4 rows per lane halve the
  // per-tile overhead (mbarrier waits, loop, votes) and stream faster (SSB Q1.1
  // SF30 0.428 -> 0.395 ms); probes that wait on global memory keep 2 rows per
  // lane, and R = 4 applies only when the ring still holds 3 stages with every
  // table staged (SSB Q3.1 at R = 4 lost its staged tables: 0.61 -> 1.85 ms).
  bool prefer4 = false;
  if (jit && force_R == 2 && !getenv("HQ_JIT_R") && !we && P.sink == HQ_SINK_MATERIALISE) {
    // A3 behind a global probe: its per-tile barriers wait for the slowest warp's probe,
    // so fewer, larger tiles pay (TPC-H Q3 SF30 orders side 0.367 -> 0.336 ms, SSB Q3.1
    // materialised 1.165 -> 0.98 ms at 4 rows per lane, measured)
    prefer4 = true;
  } else if (jit && force_R == 2 && !getenv("HQ_JIT_R") && !we && !(P.sink == HQ_SINK_AGG && P.nkeys > 0)) {
    // (not for group-by sinks: their R >= 4 path compacts the live rows of a warp
    // before the table updates, pure overhead when every row is live -- Exp 2 with
    // 32-512 groups 0.115 ms at R = 2 vs 1.1-1.25 ms at R = 4, measured)
    prefer4 = true;
    for (int o = 0; o < kp.nops; ++o) {
      if (kp.ops[o].kind != OP_PROBE) continue;
      bool st = false;
      for (int i = 0; i < nstaged; ++i) st = st || staged[i] == kp.ops[o].idx;
      prefer4 = prefer4 && st && kp.probes[kp.ops[o].idx].direct;
    }
  }
  int chosen_R = 0;
  // generated materialisation (A3): stage the tile's output rows in shared memory when
  // two tile buffers fit beside the ring (the global write-out moves to the next tile)
  uint32_t outbytes = 0;
  for (int j = 0; j < kp.nout; ++j) outbytes += kp.out_width[j];
  // opt-in (HQ_JIT_A3STAGE=1): measured on B200 it does not pay -- TPC-H Q3 SF30 orders side
  // 0.367 -> 0.377 ms, SSB Q3.1 materialised 1.165 -> 1.166 ms, Exp 1 Query 1 0.26 -> 0.32 ms:
  // the per-tile barriers, not the atomic's round trip, bound A3 behind a global probe
  const char* a3e = getenv("HQ_JIT_A3STAGE");
  bool a3try = jit && !mp_pass && P.sink == HQ_SINK_MATERIALISE && P.resolution == HQ_RES_LRGP && a3e && a3e[0] == '1';
  // warp-workgroup A3 (a3stage 2) behind a global probe: the per-tile block scan would make
  // every warp wait for the slowest warp's probe and for the tile's atomicAdd round trip
  bool a3w = false;
  if (jit && !mp_pass && !we && !a3try && P.sink == HQ_SINK_MATERIALISE && P.resolution == HQ_RES_LRGP &&
      !getenv("HQ_JIT_NOA3W")) {
    for (int o = 0; o < kp.nops; ++o) {
      if (kp.ops[o].kind != OP_PROBE) continue;
      const KProbe& pr = kp.probes[kp.ops[o].idx];
      bool st = false;
      for (int i = 0; i < nstaged; ++i) st = st || staged[i] == kp.ops[o].idx;
      a3w = a3w || !pr.direct || !st;
    }
  }
  kp.a3stage = 0;
  uint32_t a3w_tiles = 2;
  // The unified L1 / shared-memory array is 256 KB per SM and the driver carves the
  // shared part out of it in steps (.., 164, 196, 228 KB) by the kernel's request: a
  // ring that fills 228 KB leaves 28 KB of L1 for the probes that read global memory
  // (byte maps / bitmaps in L2), one that stays within 196 KB leaves 60 KB.  Generated
  // kernels with such probes therefore trade consumer warps for L1 (measured on B200,
  // SSB Q4.1 SF100: 31 warps / 228 KB 2.465 ms, 29 warps / 196 KB 2.19 ms -- the 175-KB
  // part bitmap's hits; SF30 already fit 196 KB).  HQ_JIT_CARVE=<KB> overrides (A/B).
  bool l1_probe = false;
  for (int o = 0; jit && o < kp.nops; ++o) {
    if (kp.ops[o].kind != OP_PROBE) continue;
    bool st = false;
    for (int i = 0; i < nstaged; ++i) st = st || staged[i] == kp.ops[o].idx;
    l1_probe = l1_probe || !st;
  }
  uint64_t carve_kb = l1_probe && !getenv("HQ_JIT_NW") ? 196 : 0;
  if (const char* e = getenv("HQ_JIT_CARVE")) carve_kb = jit ? (uint64_t)atoi(e) : 0;
  const int nstaged0 = nstaged, nw0 = kp.nw;
  const bool a3try0 = a3try, a3w0 = a3w;
  const uint64_t carve_cap = carve_kb ? std::min<uint64_t>(ctx->max_smem, carve_kb * 1024 - 1024) : ctx->max_smem;
  // warp update queues: the longest (16 .. 4 rows per warp) that keeps the ring's depth
  // (up to 4 stages) -- a stage less cost more than the queue saved (TPC-H Q3 SF30 lineitem:
  // no queue 0.752 ms, 6 rows at 4 stages 0.721 ms, 16 rows at 3 stages 0.777 ms; TPC-H Q10
  // SF10 0.397 / 0.281 / 0.255 ms, measured)
  if (kp.gq_cap && !getenv("HQ_JIT_GQ")) {
    uint32_t tab_total = 0;
    for (int i = 0; i < nstaged; ++i) tab_total += align_up(kp.probes[staged[i]].cbytes, 128);
    const uint32_t T = (uint32_t)kp.nw * 32u * 2u;
    const uint32_t stride = std::max<uint32_t>(128, align_up(T * rowbytes, 128));
    const uint32_t off_agg = align_up(MISC_BYTES + T * tmp_row, 128);
    const uint32_t per = 31u * (2u + (uint32_t)kp.naggs) * 8u;
    auto stages = [&](uint32_t q) -> int64_t {
      const uint32_t off_stage = align_up(align_up(off_agg + q * per, 128) + tab_total, 128);
      return off_stage >= carve_cap ? 0 : std::min<int64_t>(MAX_STAGES, (int64_t)(carve_cap - off_stage) / stride);
    };
    const int64_t want = std::min<int64_t>(stages(0), 4);
    uint32_t q = 16;
    while (q >= 4 && stages(q) < want) --q;
    kp.gq_cap = (uint16_t)(q >= 4 ? q : 0);
    agg_smem = kp.gq_cap * per;
  }
  // search: the most consumer warps (>= 16) whose ring keeps >= 3 stages and every staged
  // table within the carve-out; else the full shared memory with the default warps
  bool carve_ok = false;
  for (int nw = nw0; carve_cap < ctx->max_smem && !carve_ok && nw >= 16; --nw) {
    nstaged = nstaged0; a3try = a3try0; a3w = a3w0; a3w_tiles = 2; kp.nw = nw;
    const uint64_t smem_cap = carve_cap;
  for (;;) {
    uint32_t tab_total = 0;
    for (int i = 0; i < nstaged; ++i) tab_total += align_up(kp.probes[staged[i]].cbytes, 128);
    for (int R : {8, 4, 3, 2, 1}) {  // (3: only when forced, HQ_JIT_R=3 experiments)
      if (prefer4 ? (R != 4 && R != 2) : (force_R ? R != force_R : (R == 8 || R == 1 || R == 3))) continue;
      const uint32_t T = (uint32_t)(kp.nw * 32 * R);
      const uint32_t off_tmp = MISC_BYTES;
      const uint32_t off_agg = align_up(off_tmp + T * tmp_row, 128);
      // (a3w: one buffer per warp at off_agg of a3w_tiles x 32 R rows, i.e. that many of the
      // warp's tiles at full selectivity: 2, or 1 when two do not fit beside the ring)
      uint32_t a3wb = 0;
      for (int j = 0; a3w && j < kp.nout; ++j) a3wb += align_up(32u * a3w_tiles * (uint32_t)R * kp.out_width[j], 16);
      const uint32_t a3buf = a3try ? align_up(T * outbytes, 128) : (a3w ? (uint32_t)kp.nw * a3wb / 2 : 0);
      const uint32_t off_tab = align_up(off_agg + agg_smem + 2 * a3buf, 128);
      const uint32_t off_stage = align_up(off_tab + tab_total, 128);
      const uint32_t stride = std::max<uint32_t>(128, align_up(T * rowbytes, 128));
      if (off_stage >= smem_cap) continue;
      int S = (int)std::min<int64_t>(MAX_STAGES, (smem_cap - off_stage) / stride);
      if (const char* e = jit ? getenv("HQ_JIT_MAXS") : nullptr) S = std::min(S, std::max(2, atoi(e)));  // A/B
      if (S >= 3 || (R <= 2 && S >= 2 && nstaged == 0)) {
        chosen_R = R;
        kp.R = R;
        kp.tile_rows = (int32_t)T;
        kp.nstages = S;
        kp.stage_bytes = T * rowbytes;
        kp.stage_stride = stride;
        kp.off_tmp = off_tmp;
        kp.off_agg = off_agg;
        kp.off_tab = off_tab;
        kp.tab_bytes = tab_total;
        kp.off_stage = off_stage;
        kp.a3stage = a3try ? 1 : (a3w ? 2 : 0);
        kp.a3_buf = a3w ? a3wb : a3buf;
        kp.a3_rows = a3w ? 32u * a3w_tiles * (uint32_t)R : 0;
        break;
      }
    }
    if (chosen_R) break;
    if (a3w && a3w_tiles > 1) {  // a smaller warp buffer
      --a3w_tiles;
      continue;
    }
    if (a3try || a3w) {  // no room for the buffers: write rows straight to global memory
      a3try = a3w = false;
      continue;
    }
    if (nstaged == 0) break;
    --nstaged;  // give the last staged table back to the ring
  }
    carve_ok = chosen_R != 0 && nstaged == nstaged0 && kp.nstages >= 3 && a3w == a3w0 && a3try == a3try0;
    if (!carve_ok) chosen_R = 0;
  }
  if (!carve_ok) {
    nstaged = nstaged0; a3try = a3try0; a3w = a3w0; a3w_tiles = 2; kp.nw = nw0;
    const uint64_t smem_cap = ctx->max_smem;
  for (;;) {
    uint32_t tab_total = 0;
    for (int i = 0; i < nstaged; ++i) tab_total += align_up(kp.probes[staged[i]].cbytes, 128);
    for (int R : {8, 4, 3, 2, 1}) {  // (3: only when forced, HQ_JIT_R=3 experiments)
      if (prefer4 ? (R != 4 && R != 2) : (force_R ? R != force_R : (R == 8 || R == 1 || R == 3))) continue;
      const uint32_t T = (uint32_t)(kp.nw * 32 * R);
      const uint32_t off_tmp = MISC_BYTES;
      const uint32_t off_agg = align_up(off_tmp + T * tmp_row, 128);
      // (a3w: one buffer per warp at off_agg of a3w_tiles x 32 R rows, i.e. that many of the
      // warp's tiles at full selectivity: 2, or 1 when two do not fit beside the ring)
      uint32_t a3wb = 0;
      for (int j = 0; a3w && j < kp.nout; ++j) a3wb += align_up(32u * a3w_tiles * (uint32_t)R * kp.out_width[j], 16);
      const uint32_t a3buf = a3try ? align_up(T * outbytes, 128) : (a3w ? (uint32_t)kp.nw * a3wb / 2 : 0);
      const uint32_t off_tab = align_up(off_agg + agg_smem + 2 * a3buf, 128);
      const uint32_t off_stage = align_up(off_tab + tab_total, 128);
      const uint32_t stride = std::max<uint32_t>(128, align_up(T * rowbytes, 128));
      if (off_stage >= smem_cap) continue;
      int S = (int)std::min<int64_t>(MAX_STAGES, (smem_cap - off_stage) / stride);
      if (const char* e = jit ? getenv("HQ_JIT_MAXS") : nullptr) S = std::min(S, std::max(2, atoi(e)));  // A/B
      if (S >= 3 || (R <= 2 && S >= 2 && nstaged == 0)) {
        chosen_R = R;
        kp.R = R;
        kp.tile_rows = (int32_t)T;
        kp.nstages = S;
        kp.stage_bytes = T * rowbytes;
        kp.stage_stride = stride;
        kp.off_tmp = off_tmp;
        kp.off_agg = off_agg;
        kp.off_tab = off_tab;
        kp.tab_bytes = tab_total;
        kp.off_stage = off_stage;
        kp.a3stage = a3try ? 1 : (a3w ? 2 : 0);
        kp.a3_buf = a3w ? a3wb : a3buf;
        kp.a3_rows = a3w ? 32u * a3w_tiles * (uint32_t)R : 0;
        break;
      }
    }
    if (chosen_R) break;
    if (a3w && a3w_tiles > 1) {  // a smaller warp buffer
      --a3w_tiles;
      continue;
    }
    if (a3try || a3w) {  // no room for the buffers: write rows straight to global memory
      a3try = a3w = false;
      continue;
    }
    if (nstaged == 0) break;
    --nstaged;  // give the last staged table back to the ring
  }
  }
  if (kp.a3stage == 1) {
    uint32_t off = 0;
    for (int j = 0; j < kp.nout; ++j) {
      kp.a3_col[j] = off;
      off += (uint32_t)kp.tile_rows * kp.out_width[j];
    }
  } else if (kp.a3stage == 2) {
    uint32_t off = 0;
    for (int j = 0; j < kp.nout; ++j) {
      kp.a3_col[j] = off;
      off += align_up(kp.a3_rows * kp.out_width[j], 16);
    }
  }
  if (!chosen_R) HQ_THROW(HQ_ERR_UNSUPPORTED, "plan: rows too wide for the shared-memory stage ring");
  kp.early_release = 0;
  if (jit) {
    // early stage release when an operator waits on global memory: linear
    // probes, probes of tables not staged in shared memory, global hash groups
    bool slow = kp.sink == HQ_SINK_AGG && kp.gmode == GM_HASH && kp.smode == SM_NONE;
    for (int o = 0; o < kp.nops; ++o) {
      if (kp.ops[o].kind != OP_PROBE) continue;
      const KProbe& pr = kp.probes[kp.ops[o].idx];
      bool staged_here = false;
      for (int i = 0; i < nstaged; ++i) staged_here = staged_here || staged[i] == kp.ops[o].idx;
      if (!pr.direct || !staged_here) slow = true;
    }
    // (not for a one-probe warp-workgroup A3 pipeline: its warps hold the stage through
    // the probe and append straight from it -- TPC-H Q3 SF30 orders side 0.170 -> 0.157
    // ms, Q5 SF10 orders side 0.056 -> 0.053 ms; SSB Q3.1 materialised, three probes,
    // keeps it: 0.637 vs 0.652 ms, measured)
    int nprobe_ops = 0;
    for (int o = 0; o < kp.nops; ++o) nprobe_ops += kp.ops[o].kind == OP_PROBE ? 1 : 0;
    kp.early_release = slow && !(kp.a3stage == 2 && nprobe_ops == 1) ? 1 : 0;
    if (const char* e = getenv("HQ_JIT_EARLY")) kp.early_release = e[0] == '1' ? 1 : 0;
  }
  r->segment_rows = kp.a3stage == 2 ? 0 : kp.tile_rows;  // (warp workgroups: no tile segments)
  {
    uint32_t off = kp.off_tab;
    for (int i = 0; i < nstaged; ++i) {
      kp.probes[staged[i]].smem_off = off;
      off += align_up(kp.probes[staged[i]].cbytes, 128);
    }
  }
  const uint32_t T = (uint32_t)kp.tile_rows;
  uint32_t soff = 0;
  for (int c = 0; c < ncols_all; ++c) {
    if (!col_used[c]) continue;
    KCol& kc = kp.cols[kp.ncols++];
    kc.ptr = colptr[c];
    kc.width = (uint32_t)colw[c];
    if (lazy[c]) {  // read from global memory, not staged
      if (((uintptr_t)colptr[c] & 15) != 0 && !F->host_stream) HQ_THROW(HQ_ERR_ARG, "column pointer not 16-byte aligned");
      kc.soff = 0;
      kc.lazy = 1;
      kp.regs[c] = {0, (uint8_t)kc.width, 2, {0, 0}};
      continue;
    }
    kc.soff = soff;
    kp.regs[c] = {soff, (uint8_t)kc.width, 1, {0, 0}};
    soff += T * kc.width;
  }
  uint32_t toff = 0;
  for (int k = 0; k < HQ_MAX_TMP; ++k) {
    const int w = regs[HQ_MAX_COLS + k].width;
    if (!w) continue;
    kp.regs[HQ_MAX_COLS + k] = {toff, (uint8_t)w, 0, {0, 0}};
    toff += T * (uint32_t)w;
  }
  kp.counter = (unsigned long long*)r->dstate.p;
  kp.err = (int*)(r->dstate.as<char>() + 8);
}

// Batch processing (§3; Exp 5) of an HQ_HOST_STREAM
// fact table: block b's referenced columns are copied host -> device into ring slot
// b % 2 on ctx->copy_stream while the compound kernel of block b - 1 runs on the
// context stream (copy of b waits for the kernel of b - 2 to release the slot).  The
// kernels see block-local rows [0, rows of the block); the sink state (group table,
// output counter, fault bits) is initialised once by the caller and carries over.
static void launch_streamed(hq_ctx* ctx, hq_result* r, const KPlan& kp, bool jit, size_t smem) {
  const long long T = kp.tile_rows;
  const int64_t B = std::max<int64_t>(T, (r->stream_block + T - 1) / T * T);
  size_t slot_off[HQ_MAX_COLS + 1] = {0};
  for (int k = 0; k < kp.ncols; ++k) slot_off[k + 1] = slot_off[k] + ((size_t)B * kp.cols[k].width + 511) / 256 * 256;
  const size_t slot_bytes = std::max<size_t>(slot_off[kp.ncols], 256);
  if (!r->ring.p || r->ring.bytes < 2 * slot_bytes) r->ring = DevBuf(ctx, 2 * slot_bytes);
  if (!ctx->copy_stream) {
    HQ_CUDA(cudaStreamCreateWithFlags(&ctx->copy_stream, cudaStreamNonBlocking));
    for (int i = 0; i < 2; ++i) {
      HQ_CUDA(cudaEventCreateWithFlags(&ctx->ev_copied[i], cudaEventDisableTiming));
      HQ_CUDA(cudaEventCreateWithFlags(&ctx->ev_consumed[i], cudaEventDisableTiming));
    }
  }
  // the ring may still be read by earlier work on the context stream
  for (int i = 0; i < 2; ++i) HQ_CUDA(cudaEventRecord(ctx->ev_consumed[i], ctx->stream));
  int64_t b = 0;
  for (int64_t s = kp.row_begin; s < kp.row_end; s += B, ++b) {
    const int64_t e = std::min<int64_t>(s + B, kp.row_end);
    const int slot = (int)(b & 1);
    char* base = r->ring.as<char>() + (size_t)slot * slot_bytes;
    HQ_CUDA(cudaStreamWaitEvent(ctx->copy_stream, ctx->ev_consumed[slot], 0));
    KPlan kb = kp;
    kb.row_begin = 0;
    kb.row_end = e - s;
    for (int k = 0; k < kp.ncols; ++k) {
      const size_t w = kp.cols[k].width;
      HQ_CUDA(cudaMemcpyAsync(base + slot_off[k], (const char*)kp.cols[k].ptr + (size_t)s * w, (size_t)(e - s) * w,
                              cudaMemcpyHostToDevice, ctx->copy_stream));
      kb.cols[k].ptr = base + slot_off[k];
    }
    HQ_CUDA(cudaEventRecord(ctx->ev_copied[slot], ctx->copy_stream));
    HQ_CUDA(cudaStreamWaitEvent(ctx->stream, ctx->ev_copied[slot], 0));
    const int grid = (int)std::max<long long>(1, std::min<long long>((e - s + T - 1) / T, ctx->num_sms));
    if (jit) hq_jit_launch(ctx, kb, grid, smem);
    else launch_fused(ctx, kb, grid, smem);
    HQ_CUDA(cudaEventRecord(ctx->ev_consumed[slot], ctx->stream));
  }
}

static void launch_pipeline(hq_ctx* ctx, hq_result* r, int64_t group_cap, int64_t mat_cap) {
  const bool jit = r->plan.exec == HQ_EXEC_FUSED && hq_jit_enabled();
  KPlan kp;
  hq_build_kplan(ctx, r, kp, group_cap, mat_cap, jit);
  HQ_CUDA(cudaMemsetAsync(r->dstate.p, 0, r->dstate.bytes, ctx->stream));
  if (r->plan.sink == HQ_SINK_AGG)
    launch_init_groups(ctx, kp.gtab, r->ngroups, kp.vwords, kp.gmode == GM_HASH, kp.agg_fn, kp.naggs);
  const long long T = kp.tile_rows;
  const long long ntiles = kp.row_end > kp.row_begin ? (kp.row_end + T - 1) / T - kp.row_begin / T : 0;
  const int grid = (int)std::max<long long>(1, std::min<long long>(ntiles, ctx->num_sms));
  const size_t smem = (size_t)fused_smem_bytes(kp);
  cudaEvent_t e0 = nullptr, e1 = nullptr;
  const bool timing = ctx->timing && !ctx->capturing;
  if (timing) {
    for (cudaEvent_t* e : {&e0, &e1}) {
      if (!ctx->event_pool.empty()) { *e = ctx->event_pool.back(); ctx->event_pool.pop_back(); }
      else HQ_CUDA(cudaEventCreate(e));
    }
  }
  if (jit) hq_jit_prepare(ctx, kp, smem);  // compile (cached) outside the timed launch
  if (timing) HQ_CUDA(cudaEventRecord(e0, ctx->stream));
  if (r->stream_block > 0) launch_streamed(ctx, r, kp, jit, smem);
  else if (jit) hq_jit_launch(ctx, kp, grid, smem);
  else launch_fused(ctx, kp, grid, smem);
  if (timing) {
    HQ_CUDA(cudaEventRecord(e1, ctx->stream));
    ctx->events.emplace_back(e0, e1);
  }
}

void hq_prepare_result(hq_ctx* ctx, const hq_plan* plan, hq_result* r) {
  r->ctx = ctx;
  r->plan = *plan;
  r->sink = plan->sink;
  r->dstate = DevBuf(ctx, 32);
  if (r->fact->host_stream && plan->exec != HQ_EXEC_FUSED && plan->exec != HQ_EXEC_FUSED_INTERP)
    HQ_THROW(HQ_ERR_UNSUPPORTED, "HQ_HOST_STREAM fact tables stream through the fused kernel only");
  if (plan->exec == HQ_EXEC_OAAT) {
    hq_run_oaat(ctx, plan, r);
    return;
  }
  if (plan->exec == HQ_EXEC_MULTIPASS) {
    hq_run_multipass(ctx, plan, r);
    return;
  }
  if (plan->exec != HQ_EXEC_FUSED && plan->exec != HQ_EXEC_FUSED_INTERP) HQ_THROW(HQ_ERR_ARG, "plan: bad exec mode");
  launch_pipeline(ctx, r, 0, 0);
}

// Sync, read the device fault bits; re-run once with the exact size when an
// output capacity or group table overflowed (SURVEY.md §5 failure handling).
// Faults of a result: the build faults of the hash tables it probed (duplicate keys,
// stale cached statistics, ...; gathered on the device) and its own pipeline's fault
// word and output counter, read back together with ONE host synchronisation; a build
// fault is raised through hq_hash_check (which names it).  Capacity faults re-run the
// pipeline with larger outputs and read again.
void hq_check_result_faults(hq_ctx* ctx, hq_result* r) {
  if (r->checked) return;
  hq_require_eager(ctx, "a result's fault check");
  std::vector<const int*> hw;
  for (hq_hash* h : r->hashes)
    if (h->dstate.p && !h->checked) hw.push_back(h->dstate.as<int>());
  for (int attempt = 0;; ++attempt) {
    struct St {
      unsigned long long counter;
      int err;
      int pad;
      long long hw[32];
    };
    St* st = (St*)pinned_staging(ctx, sizeof(St));
    DevBuf out;
    const bool gather = attempt == 0 && !hw.empty();
    if (gather) {
      out = DevBuf(ctx, 32 * 8);
      hq_launch_gather_faults(ctx, hw, {}, out.as<long long>());
      HQ_CUDA(cudaMemcpyAsync(st->hw, out.p, 32 * 8, cudaMemcpyDeviceToHost, ctx->stream));
    }
    HQ_CUDA(cudaMemcpyAsync(st, r->dstate.p, 16, cudaMemcpyDeviceToHost, ctx->stream));
    HQ_CUDA(cudaStreamSynchronize(ctx->stream));
    if (gather) {
      bool any = false;
      for (int k = 0; k < 16; ++k) any = any || st->hw[k] != 0;
      if (any)
        for (hq_hash* h : r->hashes)
          if (h->dstate.p) hq_hash_check(ctx, h);
    }
    const int err = st->err;
    const unsigned long long counter = st->counter;
    if (err & HQF_DIV_ZERO) HQ_THROW(HQ_ERR_ARG, "pipeline: division by zero");
    if (err & HQF_KEY_DOMAIN) HQ_THROW(HQ_ERR_ARG, "pipeline: group key outside its declared [min, min+card)");
    const bool fixable = (err & (HQF_CAPACITY | HQF_GROUP_FULL)) != 0;
    if (!fixable) {
      r->checked_counter = (int64_t)counter;
      break;
    }
    if (attempt >= 3 || r->plan.exec == HQ_EXEC_OAAT) HQ_THROW(HQ_ERR_OVERFLOW, "pipeline: capacity exceeded");
    if (r->plan.exec == HQ_EXEC_MULTIPASS) hq_run_multipass(ctx, &r->plan, r, r->ngroups * 4);
    else if (err & HQF_CAPACITY) launch_pipeline(ctx, r, 0, (int64_t)counter);
    else launch_pipeline(ctx, r, r->ngroups * 4, 0);
  }
  r->checked = true;
}
