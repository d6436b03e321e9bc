// hq_oaat.cu -- operator-at-a-time execution of an hq_plan: the baseline the
// fused kernel is measured against (DRAM-bytes ratio, BASELINE.json metric).
//
// PAPER.md §4.2, Fig 6, after He et al.: every relational operator
// runs as separate primitives with global-memory intermediates -- (1) the
// relational primitive writes one flag per input row, (2) a prefix sum gives
// unique write positions, (3) an aligned write compacts the survivors.  The
// current selection is a TID list (row ids) as in CoGaDB; a later operator
// fetches its input column through the TID list (gather).  Probe payloads and
// expression results are materialised intermediate columns that follow the TID
// list through every compaction.  The aggregation operator reads its dense
// inputs and updates the same global group table as the fused kernel (per-row
// global atomics, i.e. a hash/dense group-by operator), so finalisation is
// shared.  The prefix sum is CUB DeviceScan (the paper used boost::compute,
// P:1398-1399).
#include <cub/device/device_scan.cuh>

#include <map>

#include "hq_device.cuh"
#include "hq_internal.h"

using namespace hqk;

namespace {

__device__ __forceinline__ long long ldw(const char* p, int w, long long i) {
  if (w == 4) return ((const int*)p)[i];
  if (w == 8) return ((const long long*)p)[i];
  return ((const signed char*)p)[i];
}
__device__ __forceinline__ void stw(char* p, int w, long long i, long long v) {
  if (w == 4) ((int*)p)[i] = (int)v;
  else if (w == 8) ((long long*)p)[i] = v;
  else ((signed char*)p)[i] = (signed char)v;
}
#define GRID_STRIDE(i, n) \
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < (n); i += (long long)gridDim.x * blockDim.x)

// fetch a column through the TID list
__global__ void hq_oaat_gather(const char* col, int w, const int* rid, long long n, char* out) {
  GRID_STRIDE(i, n) stw(out, w, i, ldw(col, w, rid[i]));
}
// selection primitive: flag per row
__global__ void hq_oaat_filter(const char* in, int w, KPred f, long long n, int* flags) {
  GRID_STRIDE(i, n) {
    const long long v = ldw(in, w, i);
    bool ok;
    if (f.kind == 0) ok = (v >= f.lo && v <= f.hi) != (bool)f.neg;
    else ok = (unsigned long long)v < 256 && ((f.bm[v >> 6] >> (v & 63)) & 1ull);
    flags[i] = ok;
  }
}
// join probe primitive: flag + payload per row
__global__ void hq_oaat_probe(const char* key, int w, const char* key2, int w2, KProbe pr, long long n, int* flags,
                              int* p0, int* p1, int* p2) {
  GRID_STRIDE(i, n) {
    const long long kv = ldw(key, w, i);
    const int k2 = pr.composite ? (int)ldw(key2, w2, i) : 0;  // composite: slot word 1 = second key
    int hit = 0, pay[3] = {0, 0, 0};
    if (kv > (long long)INT_MIN && kv <= (long long)INT_MAX) {
      const int k = (int)kv;
      if (pr.direct) {
        const uint32_t d = (uint32_t)(k - pr.dmin);
        if (d < pr.mask) {
          const uint32_t* s = pr.slots + (size_t)d * pr.words;
          if ((int)s[0] == k) {
            hit = 1;
            for (int j = 0; j < pr.npay; ++j) pay[j] = (int)s[1 + j];
          }
        }
      } else {
        uint32_t pos = ((uint32_t)k * 0x9E3779B1u) >> (32u - pr.log2cap);
        for (uint32_t t = 0; t <= pr.mask; ++t) {
          const uint32_t* s = pr.slots + (size_t)pos * pr.words;
          if ((int)s[0] == k && (!pr.composite || (int)s[1] == k2)) {
            hit = 1;
            for (int j = 0; j < pr.npay; ++j) pay[j] = (int)s[1 + pr.composite + j];
            break;
          }
          if ((int)s[0] == INT_MIN) break;
          pos = (pos + 1) & pr.mask;
        }
      }
    }
    flags[i] = pr.mode == HQ_PROBE_ANTI ? !hit : (pr.mode == HQ_PROBE_OUTER ? 1 : hit);  // OUTER: payload 0 on a miss
    if (pr.npay > 0) p0[i] = pay[0];
    if (pr.npay > 1) p1[i] = pay[1];
    if (pr.npay > 2) p2[i] = pay[2];
  }
}
// aligned write: compact a column by flags / positions
__global__ void hq_oaat_compact(const int* flags, const int* pos, long long n, const char* in, int w, char* out) {
  GRID_STRIDE(i, n) if (flags[i]) stw(out, w, pos[i], ldw(in, w, i));
}
__global__ void hq_oaat_compact_rid(const int* flags, const int* pos, long long n, const int* rid, long long base,
                                    int* out) {
  GRID_STRIDE(i, n) if (flags[i]) out[pos[i]] = rid ? rid[i] : (int)(base + i);
}
__global__ void hq_oaat_cast(const char* in, int wi, long long n, char* out, int wo) {
  GRID_STRIDE(i, n) stw(out, wo, i, ldw(in, wi, i));
}
struct KIn {
  const char* p[HQ_MAX_INSN];
  int w[HQ_MAX_INSN];
};
// projection primitive: one expression over dense inputs
__global__ void hq_oaat_compute(KInsn const* __restrict__ code, int ninsn, KIn in, long long n, long long* out,
                                int* err) {
  __shared__ KInsn c[HQ_MAX_INSN];
  if (threadIdx.x < ninsn) c[threadIdx.x] = code[threadIdx.x];
  __syncthreads();
  GRID_STRIDE(i, n) {
    long long acc = 0;
    for (int k = 0; k < ninsn; ++k) {
      const long long o = c[k].reg < 0 ? c[k].imm : ldw(in.p[k], in.w[k], i);
      switch (c[k].opc) {
        case HQ_I_LOAD: acc = o; break;
        case HQ_I_ADD: acc += o; break;
        case HQ_I_SUB: acc -= o; break;
        case HQ_I_RSUB: acc = o - acc; break;
        case HQ_I_MUL: acc *= o; break;
        case HQ_I_AND_EQ: case HQ_I_AND_NE: case HQ_I_AND_LT: case HQ_I_AND_LE: case HQ_I_AND_GT: case HQ_I_AND_GE:
        case HQ_I_AND_IN: case HQ_I_OR: acc = hq_pred_insn(c[k].opc, acc, o, c[k].imm); break;
        default:
          if (o == 0) { atomicOr(err, HQF_DIV_ZERO); acc = 0; }
          else acc = c[k].opc == HQ_I_DIV ? acc / o : acc % o;
      }
    }
    out[i] = acc;
  }
}
struct KAggIn {
  const char* key[HQ_MAX_KEYS];
  int kw[HQ_MAX_KEYS];
  const char* val[HQ_MAX_AGGS];
  int vw[HQ_MAX_AGGS];
};
// aggregation operator over dense inputs: a hash/dense group-by operator with
// the usual per-block pre-aggregation in shared memory when the dense group
// domain fits (sgroups > 0), else per-row global atomics (scalar: block reduce
// first).  Pre-aggregation only changes on-chip traffic, not the DRAM bytes the
// ratio compares; without it a tiny domain (TPC-H Q1: 4 groups) serialises on
// global atomics and the kernel-time ratio would measure contention.
__global__ void hq_oaat_agg(const __grid_constant__ KPlan p, KAggIn in, long long n, int sgroups) {
  extern __shared__ long long stab[];
  const bool scalar = p.nkeys == 0;
  long long acc[HQ_MAX_AGGS];
  unsigned long long cnt = 0;
  for (int a = 0; a < p.naggs; ++a) acc[a] = agg_identity(p.agg_fn[a]);
  if (sgroups > 0) {
    for (int i = threadIdx.x; i < sgroups * (int)p.vwords; i += blockDim.x) {
      const int c = i % (int)p.vwords;
      stab[i] = c == 0 ? 0 : agg_identity(p.agg_fn[c - 1]);
    }
    __syncthreads();
  }
  GRID_STRIDE(i, n) {
    long long vals[HQ_MAX_AGGS];
    for (int a = 0; a < p.naggs; ++a) vals[a] = p.agg_fn[a] == HQ_AGG_COUNT ? 1 : ldw(in.val[a], in.vw[a], i);
    if (scalar) {
      ++cnt;
      for (int a = 0; a < p.naggs; ++a) acc[a] = agg_combine(p.agg_fn[a], acc[a], vals[a]);
      continue;
    }
    unsigned long long key = 0;
    bool bad = false;
    for (int k = 0; k < p.nkeys; ++k) {
      const long long d = ldw(in.key[k], in.kw[k], i) - p.key_min[k];
      if (d < 0 || d >= p.key_card[k]) bad = true;
      key += (unsigned long long)d * (unsigned long long)p.key_stride[k];
    }
    if (bad) {
      atomicOr(p.err, HQF_KEY_DOMAIN);
      continue;
    }
    if (sgroups > 0) {
      const uint32_t e = (uint32_t)__cvta_generic_to_shared(stab + key * p.vwords);
      s_add64(e, 1);
      for (int a = 0; a < p.naggs; ++a) s_agg(p.agg_fn[a], e + 8u * (1 + a), vals[a], 1);
      continue;
    }
    long long* e = global_locate(p, key);
    if (e) entry_update(p, e, 1, vals);
  }
  if (sgroups > 0) {  // merge the block's groups into the global table
    __syncthreads();
    for (int g = threadIdx.x; g < sgroups; g += blockDim.x) {
      const long long* t = stab + (long long)g * p.vwords;
      if (t[0] == 0) continue;
      long long vals[HQ_MAX_AGGS];
      for (int a = 0; a < p.naggs; ++a) vals[a] = t[1 + a];
      entry_update(p, p.gtab + (long long)g * p.vwords, (unsigned long long)t[0], vals);
    }
  }
  if (scalar) {
    for (int o = 16; o > 0; o >>= 1) cnt += __shfl_xor_sync(FULLMASK, cnt, o);
    for (int a = 0; a < p.naggs; ++a) acc[a] = warp_reduce(p.agg_fn[a], acc[a]);
    if ((threadIdx.x & 31) == 0 && cnt) entry_update(p, p.gtab, cnt, acc);
  }
}

struct Mat {
  const char* p = nullptr;
  int w = 0;
  DevBuf own;
};

int grid_for(hq_ctx* ctx, long long n) {
  return (int)std::max<long long>(1, std::min<long long>((n + 255) / 256, (long long)ctx->num_sms * 16));
}

}  // namespace

void hq_run_oaat(hq_ctx* ctx, const hq_plan* plan, hq_result* r) {
  KPlan kp;
  hq_build_kplan(ctx, r, kp, 0, 0);  // validation + sink buffers (same layouts as fused)
  cudaStream_t st = ctx->stream;
  HQ_CUDA(cudaMemsetAsync(r->dstate.p, 0, r->dstate.bytes, st));
  if (plan->sink == HQ_SINK_AGG)
    launch_init_groups(ctx, kp.gtab, r->ngroups, kp.vwords, kp.gmode == GM_HASH, kp.agg_fn, kp.naggs);
  const hq_table* F = r->fact;
  const long long base = kp.row_begin;
  long long n = kp.row_end - kp.row_begin;
  DevBuf rid;  // TID list (empty = identity over [row_begin, row_end))
  std::map<int, Mat> mats;
  auto width_of = [&](int reg) { return reg < HQ_MAX_COLS ? F->cols[reg].width : (int)kp.regs[reg].width; };
  auto get = [&](int reg) -> Mat& {
    auto it = mats.find(reg);
    if (it != mats.end()) return it->second;
    if (reg >= HQ_MAX_COLS) HQ_THROW(HQ_ERR_ARG, "oaat: temporary read before written");
    Mat& m = mats[reg];
    m.w = F->cols[reg].width;
    if (!rid.p) {
      m.p = (const char*)F->cols[reg].ptr + base * m.w;  // the scan itself: no copy
    } else {
      m.own = DevBuf(ctx, (size_t)std::max<long long>(n, 1) * m.w);
      ctx->launches++;
      hq_oaat_gather<<<grid_for(ctx, n), 256, 0, st>>>((const char*)F->cols[reg].ptr, m.w, rid.as<int>(), n,
                                                        m.own.as<char>());
      m.p = m.own.as<char>();
    }
    return m;
  };
  // prefix sum + aligned writes of the TID list and of every materialised temporary
  auto compact = [&](DevBuf& flags) {
    DevBuf pos(ctx, (size_t)std::max<long long>(n, 1) * 4 + 16);
    size_t tmp_bytes = 0;
    if (n > 0) {
      HQ_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tmp_bytes, flags.as<int>(), pos.as<int>(), (int)n, st));
      DevBuf tmp(ctx, tmp_bytes + 16);
      ctx->launches += 2;
      HQ_CUDA(cub::DeviceScan::ExclusiveSum(tmp.p, tmp_bytes, flags.as<int>(), pos.as<int>(), (int)n, st));
    }
    int last[2] = {0, 0};
    if (n > 0) {
      HQ_CUDA(cudaMemcpyAsync(&last[0], pos.as<int>() + n - 1, 4, cudaMemcpyDeviceToHost, st));
      HQ_CUDA(cudaMemcpyAsync(&last[1], flags.as<int>() + n - 1, 4, cudaMemcpyDeviceToHost, st));
      HQ_CUDA(cudaStreamSynchronize(st));
    }
    const long long m = (long long)last[0] + last[1];
    DevBuf nrid(ctx, (size_t)std::max<long long>(m, 1) * 4);
    ctx->launches++;
    hq_oaat_compact_rid<<<grid_for(ctx, n), 256, 0, st>>>(flags.as<int>(), pos.as<int>(), n,
                                                          rid.p ? rid.as<int>() : nullptr, base, nrid.as<int>());
    std::map<int, Mat> next;
    for (auto& kv : mats) {
      if (kv.first < HQ_MAX_COLS) continue;  // base columns are re-fetched through the TID list
      Mat& o = next[kv.first];
      o.w = kv.second.w;
      o.own = DevBuf(ctx, (size_t)std::max<long long>(m, 1) * o.w);
      ctx->launches++;
      hq_oaat_compact<<<grid_for(ctx, n), 256, 0, st>>>(flags.as<int>(), pos.as<int>(), n, kv.second.p, o.w,
                                                        o.own.as<char>());
      o.p = o.own.as<char>();
    }
    HQ_CUDA(cudaGetLastError());
    mats = std::move(next);
    rid = std::move(nrid);
    n = m;
  };

  for (int o = 0; o < kp.nops; ++o) {
    const KOp op = kp.ops[o];
    if (op.kind == OP_FILTER) {
      const KPred& f = kp.preds[op.idx];
      Mat& in = get(f.reg);
      DevBuf flags(ctx, (size_t)std::max<long long>(n, 1) * 4);
      ctx->launches++;
      hq_oaat_filter<<<grid_for(ctx, n), 256, 0, st>>>(in.p, in.w, f, n, flags.as<int>());
      compact(flags);
    } else if (op.kind == OP_PROBE) {
      const KProbe& pr = kp.probes[op.idx];
      Mat& in = get(pr.key_reg);
      const Mat* in2 = pr.composite ? &get(pr.key2_reg) : nullptr;
      DevBuf flags(ctx, (size_t)std::max<long long>(n, 1) * 4);
      DevBuf pay[3];
      for (int j = 0; j < pr.npay; ++j) pay[j] = DevBuf(ctx, (size_t)std::max<long long>(n, 1) * 4);
      ctx->launches++;
      hq_oaat_probe<<<grid_for(ctx, n), 256, 0, st>>>(in.p, in.w, in2 ? in2->p : nullptr, in2 ? in2->w : 4, pr, n,
                                                      flags.as<int>(), pay[0].as<int>(),
                                                      pay[1].as<int>(), pay[2].as<int>());
      for (int j = 0; j < pr.npay; ++j) {
        Mat& m = mats[pr.dst[j]];
        m.w = 4;
        m.own = std::move(pay[j]);
        m.p = m.own.as<char>();
      }
      compact(flags);
    } else {
      const KCompute& c = kp.comps[op.idx];
      KIn in{};
      for (int k = 0; k < c.n; ++k) {
        const KInsn& ki = kp.insns[c.first + k];
        if (ki.reg >= 0) {
          Mat& m = get(ki.reg);
          in.p[k] = m.p;
          in.w[k] = m.w;
        }
      }
      DevBuf code(ctx, sizeof(KInsn) * c.n);
      HQ_CUDA(cudaMemcpyAsync(code.p, kp.insns + c.first, sizeof(KInsn) * c.n, cudaMemcpyHostToDevice, st));
      Mat out;
      out.w = 8;
      out.own = DevBuf(ctx, (size_t)std::max<long long>(n, 1) * 8);
      out.p = out.own.as<char>();
      ctx->launches++;
      hq_oaat_compute<<<grid_for(ctx, n), 256, 0, st>>>(code.as<KInsn>(), c.n, in, n, out.own.as<long long>(),
                                                        kp.err);
      HQ_CUDA(cudaStreamSynchronize(st));  // `code` is released at scope end
      mats[c.dst] = std::move(out);
    }
    HQ_CUDA(cudaGetLastError());
  }

  if (plan->sink == HQ_SINK_AGG) {
    KAggIn in{};
    for (int k = 0; k < kp.nkeys; ++k) {
      Mat& m = get(kp.key_reg[k]);
      in.key[k] = m.p;
      in.kw[k] = m.w;
    }
    for (int a = 0; a < kp.naggs; ++a) {
      if (kp.agg_fn[a] == HQ_AGG_COUNT) continue;
      Mat& m = get(kp.agg_reg[a]);
      in.val[a] = m.p;
      in.vw[a] = m.w;
    }
    if (n > 0) {
      ctx->launches++;
      const long long sg = (kp.gmode == GM_DENSE && r->ngroups * kp.vwords * 8 <= SMEM_AGG_BYTES) ? r->ngroups : 0;
      hq_oaat_agg<<<grid_for(ctx, n), 256, (size_t)sg * kp.vwords * 8, st>>>(kp, in, n, (int)sg);
    }
  } else {
    const long long m = std::min<long long>(n, kp.capacity);
    for (int j = 0; j < kp.nout; ++j) {
      Mat& src = get(kp.out_reg[j]);  // fetched through the final TID list
      if (m > 0) {                    // cast-copy into the result column
        ctx->launches++;
        hq_oaat_cast<<<grid_for(ctx, m), 256, 0, st>>>(src.p, src.w, m, (char*)kp.out_ptr[j], kp.out_width[j]);
      }
    }
    const unsigned long long cnt = (unsigned long long)n;
    HQ_CUDA(cudaMemcpyAsync(r->dstate.p, &cnt, 8, cudaMemcpyHostToDevice, st));
    if (n > kp.capacity) {
      const int flag = HQF_CAPACITY;
      HQ_CUDA(cudaMemcpyAsync(r->dstate.as<char>() + 8, &flag, 4, cudaMemcpyHostToDevice, st));
    }
  }
  HQ_CUDA(cudaGetLastError());
  HQ_CUDA(cudaStreamSynchronize(st));  // intermediates are released on return
}
