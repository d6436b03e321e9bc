// hq_multipass.cu -- multi-pass query compilation of an hq_plan, the paper's
// middle execution model (§4 "Multi-Pass Query Compilation",
// P:544-649, Fig 7-9; Table 4 techniques A1/B1/C1).
//
// The prefix sum is extracted from the operators and run once between two
// generated kernels (Fig 7): the COUNT kernel runs the relational primitives
// (selections, join probes) and writes one int32 flag per row; an exclusive
// prefix sum over the flags gives every selected row its write position; the
// WRITE kernel is entered by the flagged rows and performs the projections
// (re-probing the joins whose payloads it needs), writing at the positions
// (Fig 8).  Reductions run on the materialised data with library calls, as the
// paper's Multi-pass used boost::compute: B1 = a device reduce
// per aggregate, C1 = radix sort of the packed group keys + reduce-by-key.
// Both generated kernels are the same code frame as the fused kernel
// (hq_jit.cu, KPlan::mp_pass); the prefix sum, sort and reductions are CUB.
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_reduce.cuh>
#include <cub/device/device_run_length_encode.cuh>
#include <cub/device/device_scan.cuh>

#include <climits>
#include <cstdio>
#include <vector>

#include "hq_device.cuh"
#include "hq_internal.h"

using namespace hqk;

namespace {

struct AggOp {
  uint8_t fn;
  __device__ __forceinline__ long long operator()(long long a, long long b) const {
    return fn == HQ_AGG_MIN ? (a < b ? a : b) : (fn == HQ_AGG_MAX ? (a > b ? a : b) : a + b);
  }
};

__global__ void mp_iota(unsigned* p, long long n) {
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
    p[i] = (unsigned)i;
}
__global__ void mp_gather(const long long* v, const unsigned* idx, long long n, long long* out) {
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
    out[i] = v[idx[i]];
}
// C1: one thread per distinct key: its group entry (dense slot or hash entry)
// receives the reduced count and aggregates
__global__ void mp_scatter_groups(const __grid_constant__ KPlan p, const unsigned long long* uniq, const int* counts,
                                  const long long* aggs, long long stride, const int* nruns, long long n) {
  const long long m = *nruns;
  for (long long g = blockIdx.x * (long long)blockDim.x + threadIdx.x; g < m && g < n;
       g += (long long)gridDim.x * blockDim.x) {
    long long vals[HQ_MAX_AGGS];
    int k = 0;
    for (int a = 0; a < p.naggs; ++a) vals[a] = p.agg_fn[a] == HQ_AGG_COUNT ? 0 : aggs[(long long)(k++) * stride + g];
    long long* e = global_locate(p, uniq[g]);
    if (e) entry_update(p, e, (unsigned long long)counts[g], vals);
  }
}
// B1: the single group
__global__ void mp_scalar_entry(const __grid_constant__ KPlan p, const long long* red, unsigned long long cnt) {
  long long vals[HQ_MAX_AGGS];
  int k = 0;
  for (int a = 0; a < p.naggs; ++a) vals[a] = p.agg_fn[a] == HQ_AGG_COUNT ? 0 : red[k++];
  entry_update(p, p.gtab, cnt, vals);
}

int grid_for(hq_ctx* ctx, long long n) {
  return (int)std::max<long long>(1, std::min<long long>((n + 255) / 256, (long long)ctx->num_sms * 16));
}

void launch_generated(hq_ctx* ctx, const KPlan& kp) {
  const long long T = kp.tile_rows;
  const long long ntiles = kp.row_end > kp.row_begin ? (kp.row_end + T - 1) / T - kp.row_begin / T : 0;
  if (ntiles == 0) return;
  const int grid = (int)std::max<long long>(1, std::min<long long>(ntiles, ctx->num_sms));
  const size_t smem = (size_t)fused_smem_bytes(kp);
  hq_jit_prepare(ctx, kp, smem);
  hq_jit_launch(ctx, kp, grid, smem);
}

void* scratch(hq_ctx* ctx, hq_result* r, size_t bytes) {
  if (r->mp_scratch.bytes < bytes) r->mp_scratch = DevBuf(ctx, bytes);
  return r->mp_scratch.p;
}

}  // namespace

void hq_run_multipass(hq_ctx* ctx, const hq_plan* plan, hq_result* r, int64_t group_cap) {
  if (!hq_jit_enabled()) HQ_THROW(HQ_ERR_UNSUPPORTED, "multi-pass execution needs generated kernels (HQ_JIT=0 is set)");
  const hq_table* F = r->fact;
  const int64_t rb = plan->row_begin, re = plan->row_end < 0 ? F->nrows : plan->row_end;
  if (rb < 0 || re < rb || re > F->nrows) HQ_THROW(HQ_ERR_ARG, "plan: row range outside the fact table");
  const int64_t n = re - rb;
  if (n >= (1LL << 31)) HQ_THROW(HQ_ERR_UNSUPPORTED, "multi-pass: more than 2^31 - 1 rows in one range");
  cudaStream_t st = ctx->stream;
  HQ_CUDA(cudaMemsetAsync(r->dstate.p, 0, r->dstate.bytes, st));
  cudaEvent_t e0 = nullptr, e1 = nullptr;
  if (ctx->timing) {
    for (cudaEvent_t* e : {&e0, &e1}) {
      if (!ctx->event_pool.empty()) { *e = ctx->event_pool.back(); ctx->event_pool.pop_back(); }
      else HQ_CUDA(cudaEventCreate(e));
    }
  }
  // flag and position columns indexed by absolute row; the base is placed so
  // that base + row_begin * 4 keeps the 16-B alignment the TMA copies need
  const size_t pad = (size_t)((rb * 4) % 16);
  r->mp_flags = DevBuf(ctx, (size_t)n * 4 + 32);
  r->mp_pos = DevBuf(ctx, (size_t)n * 4 + 32);
  int* flags = (int*)(r->mp_flags.as<char>() + pad);  // flags[i] = row rb + i
  int* pos = (int*)(r->mp_pos.as<char>() + pad);
  r->mp_flags_col = (const char*)flags - rb * 4;
  r->mp_pos_col = (const char*)pos - rb * 4;

  // pass 1: count kernel
  KPlan k1;
  hq_build_kplan(ctx, r, k1, 0, 1, true, 1);
  k1.nout = 1;
  k1.out_ptr[0] = (void*)r->mp_flags_col;
  if (ctx->timing) HQ_CUDA(cudaEventRecord(e0, st));
  launch_generated(ctx, k1);
  // prefix sum over the flags (exclusive: write positions), total selected rows
  size_t tb = 0;
  HQ_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tb, flags, pos, (int)n, st));
  HQ_CUDA(cub::DeviceScan::ExclusiveSum(scratch(ctx, r, tb), tb, flags, pos, (int)n, st));
  long long nq = 0;
  if (n > 0) {
    int last[2];
    HQ_CUDA(cudaMemcpyAsync(&last[0], pos + n - 1, 4, cudaMemcpyDeviceToHost, st));
    HQ_CUDA(cudaMemcpyAsync(&last[1], flags + n - 1, 4, cudaMemcpyDeviceToHost, st));
    HQ_CUDA(cudaStreamSynchronize(st));  // the count sizes the outputs (the one host sync)
    nq = (long long)last[0] + last[1];
  }

  // pass 2: write kernel
  KPlan k2;
  hq_build_kplan(ctx, r, k2, group_cap, std::max<long long>(nq, 1), true, 2);
  const bool agg = plan->sink == HQ_SINK_AGG;
  int nvals = 0;
  for (int a = 0; a < k2.naggs; ++a) nvals += k2.agg_fn[a] != HQ_AGG_COUNT;
  if (agg) {
    launch_init_groups(ctx, k2.gtab, r->ngroups, k2.vwords, k2.gmode == GM_HASH, k2.agg_fn, k2.naggs);
    const size_t m = (size_t)std::max<long long>(nq, 1);
    r->mp_keys = DevBuf(ctx, k2.nkeys > 0 ? m * 8 * 2 : 16);           // keys, sorted keys
    r->mp_vals = DevBuf(ctx, m * 8 * (size_t)(nvals > 0 ? 2 * nvals : 1));  // values, reduced/gathered
    int oc = 0;
    if (k2.nkeys > 0) k2.out_ptr[oc++] = r->mp_keys.p;
    for (int a = 0; a < nvals; ++a) k2.out_ptr[oc++] = r->mp_vals.as<long long>() + (size_t)a * m;
    k2.nout = oc;
  }
  const bool dbg = getenv("HQ_MP_DEBUG") != nullptr;
  if (dbg && agg && k2.nkeys > 0 && nq > 0) HQ_CUDA(cudaMemsetAsync(r->mp_keys.p, 0xFF, (size_t)nq * 8, st));
  if (nq > 0) launch_generated(ctx, k2);
  if (dbg && agg && k2.nkeys > 0 && nq > 0) {  // every position written exactly once, keys in the domain
    std::vector<unsigned long long> hk((size_t)nq);
    HQ_CUDA(cudaMemcpyAsync(hk.data(), r->mp_keys.p, (size_t)nq * 8, cudaMemcpyDeviceToHost, st));
    HQ_CUDA(cudaStreamSynchronize(st));
    long long unwritten = 0, bad = 0;
    for (auto k : hk) {
      unwritten += k == ~0ULL;
      bad += k != ~0ULL && k2.gmode != GM_HASH && (long long)k >= r->ngroups;
    }
    fprintf(stderr, "[hq multipass] nq %lld unwritten %lld out-of-domain %lld (ngroups %lld)\n", nq, unwritten, bad,
            (long long)r->ngroups);
  }

  if (agg && nq > 0) {
    const size_t m = (size_t)nq;
    long long* vals = r->mp_vals.as<long long>();
    long long* out = vals + (size_t)nvals * m;  // second half: per-aggregate results
    int k = 0;
    if (k2.nkeys == 0) {  // B1: one library reduce per aggregate
      for (int a = 0; a < k2.naggs; ++a) {
        if (k2.agg_fn[a] == HQ_AGG_COUNT) continue;
        const AggOp op{k2.agg_fn[a]};
        const long long init = k2.agg_fn[a] == HQ_AGG_MIN ? LLONG_MAX : (k2.agg_fn[a] == HQ_AGG_MAX ? LLONG_MIN : 0);
        size_t b = 0;
        HQ_CUDA(cub::DeviceReduce::Reduce(nullptr, b, vals + (size_t)k * m, out + k, (int)nq, op, init, st));
        HQ_CUDA(cub::DeviceReduce::Reduce(scratch(ctx, r, b), b, vals + (size_t)k * m, out + k, (int)nq, op, init, st));
        ++k;
      }
      ctx->launches++;
      mp_scalar_entry<<<1, 1, 0, st>>>(k2, out, (unsigned long long)nq);
    } else {  // C1: sort by packed group key, then reduce-by-key per aggregate
      unsigned long long* keys = r->mp_keys.as<unsigned long long>();
      unsigned long long* skeys = keys + m;
      DevBuf idx(ctx, m * 4 * 2), runs(ctx, m * 4 + 16), cnts(ctx, m * 4 + 16), uniq(ctx, m * 8 + 16);
      unsigned* id0 = idx.as<unsigned>();
      unsigned* id1 = id0 + m;
      ctx->launches++;
      mp_iota<<<grid_for(ctx, nq), 256, 0, st>>>(id0, nq);
      int bits = 1;
      if (k2.gmode != GM_HASH) {
        while (bits < 64 && (1ULL << bits) < (unsigned long long)r->ngroups) ++bits;
      } else {
        __int128 prod = 1;
        for (int i = 0; i < k2.nkeys; ++i) prod *= k2.key_card[i];
        while (bits < 64 && ((__int128)1 << bits) < prod) ++bits;
      }
      size_t b = 0;
      HQ_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, b, keys, skeys, id0, id1, (int)nq, 0, bits, st));
      HQ_CUDA(cub::DeviceRadixSort::SortPairs(scratch(ctx, r, b), b, keys, skeys, id0, id1, (int)nq, 0, bits, st));
      int* nruns = runs.as<int>();
      HQ_CUDA(cub::DeviceRunLengthEncode::Encode(nullptr, b, skeys, uniq.as<unsigned long long>(), cnts.as<int>(), nruns,
                                                 (int)nq, st));
      HQ_CUDA(cub::DeviceRunLengthEncode::Encode(scratch(ctx, r, b), b, skeys, uniq.as<unsigned long long>(),
                                                 cnts.as<int>(), nruns, (int)nq, st));
      DevBuf gathered(ctx, m * 8), ukeys2(ctx, m * 8 + 16);
      for (int a = 0; a < k2.naggs; ++a) {
        if (k2.agg_fn[a] == HQ_AGG_COUNT) continue;
        ctx->launches++;
        mp_gather<<<grid_for(ctx, nq), 256, 0, st>>>(vals + (size_t)k * m, id1, nq, gathered.as<long long>());
        const AggOp op{k2.agg_fn[a]};
        HQ_CUDA(cub::DeviceReduce::ReduceByKey(nullptr, b, skeys, ukeys2.as<unsigned long long>(), gathered.as<long long>(),
                                               out + (size_t)k * m, nruns + 1, op, (int)nq, st));
        HQ_CUDA(cub::DeviceReduce::ReduceByKey(scratch(ctx, r, b), b, skeys, ukeys2.as<unsigned long long>(),
                                               gathered.as<long long>(), out + (size_t)k * m, nruns + 1, op, (int)nq, st));
        ++k;
      }
      ctx->launches++;
      mp_scatter_groups<<<grid_for(ctx, nq), 256, 0, st>>>(k2, uniq.as<unsigned long long>(), cnts.as<int>(), out,
                                                          (long long)m, nruns, (long long)nq);
      HQ_CUDA(cudaStreamSynchronize(st));  // scratch buffers above are released on return
    }
  }
  if (ctx->timing) {
    HQ_CUDA(cudaEventRecord(e1, st));
    ctx->events.emplace_back(e0, e1);
  }
  // qualifying rows (result info); materialised outputs hold exactly nq rows
  const unsigned long long cnt = (unsigned long long)nq;
  HQ_CUDA(cudaMemcpyAsync(r->dstate.p, &cnt, 8, cudaMemcpyHostToDevice, st));
  HQ_CUDA(cudaGetLastError());
  HQ_CUDA(cudaStreamSynchronize(st));
}
