// hq_api.cu -- the extern "C" boundary of libhq (include/hq.h): contexts,
// column loading, hash build/import, pipeline runs, result fetch, errors.
#include <cstring>
#include <string>

#include "hq_internal.h"

void hq_build_hashes_impl(hq_ctx* ctx, int n, const hq_build_desc* d, hq_hash* const* h);
void hq_hash_check(hq_ctx* ctx, hq_hash* h);

namespace {
thread_local std::string g_last_error = "";

template <class F>
hq_status guarded(F f) {
  try {
    f();
    return HQ_OK;
  } catch (const HqError& e) {
    g_last_error = e.msg;
    return e.code;
  } catch (const std::bad_alloc&) {
    g_last_error = "host allocation failed";
    return HQ_ERR_OOM;
  } catch (const std::exception& e) {
    g_last_error = e.what();
    return HQ_ERR_ARG;
  }
}

void require_device() {
  int n = 0;
  if (cudaGetDeviceCount(&n) != cudaSuccess || n == 0) {
    cudaGetLastError();
    HQ_THROW(HQ_ERR_NO_DEVICE, "no CUDA device: libhq has no CPU fallback");
  }
}
}  // namespace

void hq_set_error(const std::string& msg) { g_last_error = msg; }

void* hq_ctx::alloc_bytes(size_t bytes) {
  if (bytes == 0) bytes = 16;
  void* p = nullptr;
  if (capturing) {
    // not a captured node: the pool allocation happens now, on a stream of its own,
    // and the memory belongs to the graph's objects (or is freed with the graph)
    if (has_alloc) HQ_THROW(HQ_ERR_UNSUPPORTED, "graph capture needs the stream-ordered pool (no allocator hooks)");
    if (cudaMallocAsync(&p, bytes, alloc_stream) != cudaSuccess || cudaStreamSynchronize(alloc_stream) != cudaSuccess) {
      cudaGetLastError();
      p = nullptr;
    }
  } else if (has_alloc) {
    p = alloc.alloc(bytes, (void*)stream, alloc.user);
  } else {
    cudaError_t e = cudaMallocAsync(&p, bytes, stream);
    if (e != cudaSuccess) {
      cudaGetLastError();
      p = nullptr;
    }
  }
  if (!p) HQ_THROW(HQ_ERR_OOM, "device allocation of " + std::to_string(bytes) + " bytes failed");
  return p;
}
void hq_ctx::free_bytes(void* p, size_t bytes) {
  if (!p) return;
  if (capturing) {  // captured work may still use it at every launch: freed with the graph
    cap_frees.emplace_back(p, bytes);
    return;
  }
  if (has_alloc) alloc.free(p, bytes, (void*)stream, alloc.user);
  else cudaFreeAsync(p, stream);
}

hq_table::~hq_table() {
  owned.clear();
  if (backing) backing->release();
}
hq_result::~hq_result() {
  if (stage_host) cudaFreeHost(stage_host);
  if (fact) fact->release();
  for (auto* h : hashes) h->release();
}

void hq_ctx::release() {
  if (refs.fetch_sub(1) != 1) return;
  hq_ctx* ctx = this;
  {
    cudaStreamSynchronize(ctx->stream);
    for (auto& e : ctx->events) {
      cudaEventDestroy(e.first);
      cudaEventDestroy(e.second);
    }
    for (auto e : ctx->event_pool) cudaEventDestroy(e);
    if (ctx->pinned) cudaFreeHost(ctx->pinned);
    if (ctx->pinned_build) cudaFreeHost(ctx->pinned_build);
    if (ctx->copy_stream) {
      cudaStreamSynchronize(ctx->copy_stream);
      cudaStreamDestroy(ctx->copy_stream);
    }
    for (int i = 0; i < 2; ++i) {
      if (ctx->ev_copied[i]) cudaEventDestroy(ctx->ev_copied[i]);
      if (ctx->ev_consumed[i]) cudaEventDestroy(ctx->ev_consumed[i]);
    }
    for (int i = 0; i < hq_ctx::NSIDE; ++i) {
      if (ctx->side[i]) {
        cudaStreamSynchronize(ctx->side[i]);
        cudaStreamDestroy(ctx->side[i]);
      }
      if (ctx->ev_join[i]) cudaEventDestroy(ctx->ev_join[i]);
    }
    if (ctx->ev_fork) cudaEventDestroy(ctx->ev_fork);
    if (ctx->cap_stream) cudaStreamDestroy(ctx->cap_stream);
    if (ctx->alloc_stream) cudaStreamDestroy(ctx->alloc_stream);
    delete ctx;
  }
}

void hq_sync(hq_ctx* ctx, const char* what) {
  hq_require_eager(ctx, what);
  HQ_CUDA(cudaStreamSynchronize(ctx->stream));
}
void hq_require_eager(hq_ctx* ctx, const char* what) {
  if (ctx->capturing)
    HQ_THROW(HQ_ERR_STATE, std::string("not capturable in a CUDA graph: ") + what +
                               " needs the host (a synchronisation); run the query eagerly");
}

// A captured prepared query: the instantiated graph, the objects its nodes read and
// write (retained), the results whose rows it stages, and buffers freed during capture.
struct hq_graph {
  CtxPtr ctx;
  cudaGraph_t graph = nullptr;
  cudaGraphExec_t exec = nullptr;
  std::vector<RefObj*> objs;
  std::vector<hq_result*> results;
  std::vector<std::pair<void*, size_t>> frees;
  int64_t nkernels = 0;  // kernels one launch runs (hq_ctx_launches accounting)
  ~hq_graph() {
    hq_ctx* c = ctx;
    if (c) cudaStreamSynchronize(c->stream);
    if (exec) cudaGraphExecDestroy(exec);
    if (graph) cudaGraphDestroy(graph);
    for (auto& f : frees) c->free_bytes(f.first, f.second);
    for (RefObj* o : objs) o->release();
  }
};

static void capture_cleanup(hq_ctx* ctx, hq_graph* g) {
  // frees and retained objects go to the graph (or are released if there is none)
  ctx->capturing = false;
  ctx->stream = ctx->user_stream;
  if (g) {
    g->frees.swap(ctx->cap_frees);
    g->objs.swap(ctx->cap_objs);
    g->results.swap(ctx->cap_results);
  } else {
    cudaStreamSynchronize(ctx->stream);
    for (auto& f : ctx->cap_frees) ctx->free_bytes(f.first, f.second);
    for (RefObj* o : ctx->cap_objs) o->release();
  }
  ctx->cap_frees.clear();
  ctx->cap_objs.clear();
  ctx->cap_results.clear();
}


extern "C" {

int32_t hq_abi_version(void) { return HQ_ABI_VERSION; }
const char* hq_last_error(void) { return g_last_error.c_str(); }

size_t hq_sizeof(const char* name) {
  if (!name) return 0;
  const std::string n(name);
  if (n == "hq_column") return sizeof(hq_column);
  if (n == "hq_pred") return sizeof(hq_pred);
  if (n == "hq_build_desc") return sizeof(hq_build_desc);
  if (n == "hq_hash_meta") return sizeof(hq_hash_meta);
  if (n == "hq_insn") return sizeof(hq_insn);
  if (n == "hq_op") return sizeof(hq_op);
  if (n == "hq_plan") return sizeof(hq_plan);
  if (n == "hq_result_info") return sizeof(hq_result_info);
  if (n == "hq_allocator") return sizeof(hq_allocator);
  return 0;
}

hq_status hq_ctx_create(int32_t device, void* stream, const hq_allocator* alloc, hq_ctx** out) {
  return guarded([&] {
    if (!out) HQ_THROW(HQ_ERR_ARG, "out is NULL");
    require_device();
    HQ_CUDA(cudaSetDevice(device));
    hq_ctx* c = new hq_ctx();
    c->device = device;
    c->stream = (cudaStream_t)stream;
    if (alloc && alloc->alloc && alloc->free) {
      c->alloc = *alloc;
      c->has_alloc = true;
    }
    int v = 0;
    HQ_CUDA(cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, device));
    c->num_sms = v;
    HQ_CUDA(cudaDeviceGetAttribute(&v, cudaDevAttrMaxSharedMemoryPerBlockOptin, device));
    c->max_smem = (size_t)v;
    if (!c->has_alloc) {  // keep freed blocks cached in the stream-ordered pool
      cudaMemPool_t pool;
      if (cudaDeviceGetDefaultMemPool(&pool, device) == cudaSuccess) {
        uint64_t thr = UINT64_MAX;
        cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
      }
      cudaGetLastError();
    }
    *out = c;
  });
}

hq_status hq_ctx_destroy(hq_ctx* ctx) {
  return guarded([&] {
    if (ctx) ctx->release();  // objects still alive keep the context until they are freed
  });
}

hq_status hq_ctx_capture_begin(hq_ctx* ctx) {
  return guarded([&] {
    if (!ctx) HQ_THROW(HQ_ERR_ARG, "ctx is NULL");
    if (ctx->capturing) HQ_THROW(HQ_ERR_STATE, "a capture is already running");
    if (ctx->has_alloc) HQ_THROW(HQ_ERR_UNSUPPORTED, "graph capture needs the stream-ordered pool (no allocator hooks)");
    HQ_CUDA(cudaStreamSynchronize(ctx->stream));
    if (!ctx->cap_stream) HQ_CUDA(cudaStreamCreateWithFlags(&ctx->cap_stream, cudaStreamNonBlocking));
    if (!ctx->alloc_stream) HQ_CUDA(cudaStreamCreateWithFlags(&ctx->alloc_stream, cudaStreamNonBlocking));
    ctx->user_stream = ctx->stream;
    ctx->stream = ctx->cap_stream;
    HQ_CUDA(cudaStreamBeginCapture(ctx->cap_stream, cudaStreamCaptureModeRelaxed));
    ctx->capturing = true;
    ctx->cap_launches0 = ctx->launches;
  });
}

hq_status hq_ctx_capture_end(hq_ctx* ctx, hq_graph** out) {
  return guarded([&] {
    if (!ctx || !out) HQ_THROW(HQ_ERR_ARG, "NULL argument");
    if (!ctx->capturing) HQ_THROW(HQ_ERR_STATE, "no capture is running");
    cudaGraph_t graph = nullptr;
    const cudaError_t e = cudaStreamEndCapture(ctx->cap_stream, &graph);
    if (e != cudaSuccess || !graph) {
      cudaGetLastError();
      capture_cleanup(ctx, nullptr);
      HQ_THROW(HQ_ERR_CUDA, std::string("graph capture failed: ") + cudaGetErrorString(e));
    }
    hq_graph* g = new hq_graph();
    g->ctx = ctx;
    g->graph = graph;
    g->nkernels = ctx->launches - ctx->cap_launches0;
    capture_cleanup(ctx, g);
    const cudaError_t ie = cudaGraphInstantiate(&g->exec, graph, 0);
    if (ie != cudaSuccess) {
      cudaGetLastError();
      delete g;
      HQ_THROW(HQ_ERR_CUDA, std::string("graph instantiation failed: ") + cudaGetErrorString(ie));
    }
    *out = g;
  });
}

hq_status hq_ctx_capture_abort(hq_ctx* ctx) {
  return guarded([&] {
    if (!ctx || !ctx->capturing) return;
    cudaGraph_t graph = nullptr;
    cudaStreamEndCapture(ctx->cap_stream, &graph);
    cudaGetLastError();
    if (graph) cudaGraphDestroy(graph);
    capture_cleanup(ctx, nullptr);
  });
}

hq_status hq_graph_launch(hq_ctx* ctx, hq_graph* g) {
  return guarded([&] {
    if (!ctx || !g) HQ_THROW(HQ_ERR_ARG, "NULL argument");
    if (ctx->capturing) HQ_THROW(HQ_ERR_STATE, "launch during a capture");
    for (hq_result* r : g->results) {  // the graph refinalizes them: stale host rows go
      r->host_ready = false;
      r->finalized = false;
      r->checked = false;
      r->checked_counter = -1;
    }
    ctx->launches += g->nkernels;
    HQ_CUDA(cudaGraphLaunch(g->exec, ctx->stream));
    if (g->results.empty()) return;  // nothing to decode: the launch stays asynchronous
    HQ_CUDA(cudaStreamSynchronize(ctx->stream));
    for (hq_result* r : g->results) hq_decode_captured(ctx, r);
  });
}

hq_status hq_graph_destroy(hq_graph* g) {
  return guarded([&] { delete g; });
}

hq_status hq_ctx_set_stream(hq_ctx* ctx, void* stream) {
  return guarded([&] {
    if (!ctx) HQ_THROW(HQ_ERR_ARG, "ctx is NULL");
    ctx->stream = (cudaStream_t)stream;
  });
}

hq_status hq_ctx_sync(hq_ctx* ctx) {
  return guarded([&] {
    if (ctx) hq_require_eager(ctx, "hq_ctx_sync");
    if (!ctx) HQ_THROW(HQ_ERR_ARG, "ctx is NULL");
    HQ_CUDA(cudaStreamSynchronize(ctx->stream));
  });
}

hq_status hq_ctx_enable_timing(hq_ctx* ctx, int32_t on) {
  return guarded([&] {
    if (!ctx) HQ_THROW(HQ_ERR_ARG, "ctx is NULL");
    ctx->timing = on != 0;
  });
}

hq_status hq_ctx_kernel_times(hq_ctx* ctx, float* ms, int32_t max, int32_t* n) {
  return guarded([&] {
    if (ctx) hq_require_eager(ctx, "hq_ctx_kernel_times");
    if (!ctx || !n) HQ_THROW(HQ_ERR_ARG, "NULL argument");
    int32_t k = 0;
    for (auto& e : ctx->events) {
      HQ_CUDA(cudaEventSynchronize(e.second));
      float t = 0;
      HQ_CUDA(cudaEventElapsedTime(&t, e.first, e.second));
      if (ms && k < max) ms[k] = t;
      ++k;
      ctx->event_pool.push_back(e.first);
      ctx->event_pool.push_back(e.second);
    }
    ctx->events.clear();
    *n = k;
  });
}

hq_status hq_ctx_launches(hq_ctx* ctx, int64_t* n) {
  return guarded([&] {
    if (!ctx || !n) HQ_THROW(HQ_ERR_ARG, "NULL argument");
    *n = ctx->launches;
  });
}

// ------------------------------------------------------------------ tables
hq_status hq_load_columns(hq_ctx* ctx, const hq_column* cols, int32_t ncols, int64_t nrows, int32_t flags,
                          hq_table** out) {
  return guarded([&] {
    if (ctx) hq_require_eager(ctx, "hq_load_columns");
    if (!ctx || !out || (!cols && ncols > 0)) HQ_THROW(HQ_ERR_ARG, "NULL argument");
    if (ncols < 0 || ncols > HQ_MAX_COLS) HQ_THROW(HQ_ERR_UNSUPPORTED, "tables have 0..16 columns");
    if (nrows < 0) HQ_THROW(HQ_ERR_ARG, "nrows < 0");
    if (flags != HQ_HOST_COPY && flags != HQ_DEVICE_BORROW && flags != HQ_HOST_STREAM)
      HQ_THROW(HQ_ERR_ARG, "flags must be HQ_HOST_COPY, HQ_DEVICE_BORROW or HQ_HOST_STREAM");
    hq_table* t = new hq_table();
    t->ctx = ctx;
    t->nrows = nrows;
    t->ncols = ncols;
    try {
      for (int c = 0; c < ncols; ++c) {
        const int w = hq_type_width(cols[c].type);
        if (w == 0 || cols[c].type == HQ_F64) HQ_THROW(HQ_ERR_ARG, "column type must be HQ_I8/I32/I64");
        if (!cols[c].data && nrows > 0) HQ_THROW(HQ_ERR_ARG, "column data is NULL");
        t->cols[c].type = cols[c].type;
        t->cols[c].width = w;
        if (flags == HQ_HOST_COPY) {
          const size_t bytes = (size_t)nrows * w;
          // padded to a 16-B multiple so every TMA tile of the column is in bounds
          t->owned.emplace_back(ctx, (bytes + 255) / 256 * 256 + 256);
          if (bytes) HQ_CUDA(cudaMemcpyAsync(t->owned.back().p, cols[c].data, bytes, cudaMemcpyHostToDevice, ctx->stream));
          t->cols[c].ptr = t->owned.back().p;
        } else if (flags == HQ_HOST_STREAM) {  // stays on the host; pipelines stream it in blocks
          t->host_stream = true;
          t->cols[c].ptr = cols[c].data;
        } else {
          if (((uintptr_t)cols[c].data & 15) != 0) HQ_THROW(HQ_ERR_ARG, "device column pointer must be 16-byte aligned");
          t->cols[c].ptr = cols[c].data;
        }
      }
    } catch (...) {
      t->release();
      throw;
    }
    *out = t;
  });
}

hq_status hq_column_range(hq_ctx* ctx, const hq_table* t, int32_t col, int64_t* min, int64_t* max) {
  return guarded([&] {
    if (ctx) hq_require_eager(ctx, "hq_column_range");
    if (!ctx || !t || !min || !max) HQ_THROW(HQ_ERR_ARG, "NULL argument");
    if (col < 0 || col >= t->ncols) HQ_THROW(HQ_ERR_ARG, "column out of range");
    hq_column_range_impl(ctx, t, col, min, max);
  });
}

hq_status hq_table_info(const hq_table* t, int64_t* nrows, int32_t* ncols) {
  return guarded([&] {
    if (!t) HQ_THROW(HQ_ERR_ARG, "table is NULL");
    if (nrows) *nrows = t->nrows;
    if (ncols) *ncols = t->ncols;
  });
}

hq_status hq_table_column(const hq_table* t, int32_t col, const void** dev_ptr, int32_t* type) {
  return guarded([&] {
    if (!t || col < 0 || col >= t->ncols) HQ_THROW(HQ_ERR_ARG, "bad table/column");
    if (t->host_stream) HQ_THROW(HQ_ERR_UNSUPPORTED, "HQ_HOST_STREAM table: its columns are not in device memory");
    if (dev_ptr) *dev_ptr = t->cols[col].ptr;
    if (type) *type = t->cols[col].type;
  });
}

hq_status hq_free_table(hq_table* t) {
  return guarded([&] {
    if (t) t->release();
  });
}

// -------------------------------------------------------------- hash tables
hq_status hq_build_hash(hq_ctx* ctx, const hq_build_desc* desc, hq_hash** out) {
  return hq_build_hashes(ctx, 1, desc, out);
}

hq_status hq_build_hashes(hq_ctx* ctx, int32_t n, const hq_build_desc* descs, hq_hash** out) {
  return guarded([&] {
    if (!ctx || !descs || !out || n < 1) HQ_THROW(HQ_ERR_ARG, "NULL argument or n < 1");
    std::vector<hq_hash*> hs((size_t)n, nullptr);
    for (auto& h : hs) {
      h = new hq_hash();
      h->ctx = ctx;
    }
    try {
      hq_build_hashes_impl(ctx, n, descs, hs.data());
    } catch (...) {
      for (auto* h : hs) h->release();
      throw;
    }
    for (int i = 0; i < n; ++i) {  // a captured build re-reads its source at every launch
      hs[i]->capture_retain(ctx);
      const_cast<hq_table*>(descs[i].src)->capture_retain(ctx);
      out[i] = hs[i];
    }
  });
}

hq_status hq_hash_info(hq_ctx* ctx, const hq_hash* h, hq_hash_meta* meta) {
  return guarded([&] {
    if (!ctx || !h) HQ_THROW(HQ_ERR_ARG, "NULL argument");
    hq_hash_check(ctx, const_cast<hq_hash*>(h));
    if (meta) *meta = h->meta;
  });
}

hq_status hq_hash_device_view(const hq_hash* h, void** dev_ptr, hq_hash_meta* meta) {
  return guarded([&] {
    if (!h) HQ_THROW(HQ_ERR_ARG, "hash is NULL");
    if (dev_ptr) *dev_ptr = h->compact_only ? const_cast<void*>(h->compact_ptr()) : (void*)h->slots;
    if (meta) {
      *meta = h->meta;
      if (h->compact_only) {  // the buffer is the compact form
        meta->compact_kind = h->ckind;
        meta->bytes = h->cbytes;
      } else {
        meta->compact_kind = 0;
      }
    }
  });
}

hq_status hq_hash_import(hq_ctx* ctx, const hq_hash_meta* meta, void* dev_ptr, hq_hash** out) {
  return guarded([&] {
    if (ctx) hq_require_eager(ctx, "hq_hash_import");
    if (!ctx || !meta || !dev_ptr || !out) HQ_THROW(HQ_ERR_ARG, "NULL argument");
    const int64_t cap = meta->capacity;
    if (meta->layout == HQ_HT_DIRECT) {
      if (cap < 1 || cap > (1LL << 30)) HQ_THROW(HQ_ERR_ARG, "import: direct capacity out of range");
    } else if (meta->layout == HQ_HT_LINEAR) {
      if (cap < 16 || (cap & (cap - 1)) != 0) HQ_THROW(HQ_ERR_ARG, "import: capacity must be a power of two >= 16");
    } else {
      HQ_THROW(HQ_ERR_ARG, "import: unknown layout");
    }
    if (meta->slot_words != 1 && meta->slot_words != 2 && meta->slot_words != 4) HQ_THROW(HQ_ERR_ARG, "import: slot_words");
    if (meta->npayload < 0 || meta->npayload > meta->slot_words - 1 + (meta->slot_words == 1 ? 0 : 0) ||
        (meta->slot_words == 1 && meta->npayload != 0))
      HQ_THROW(HQ_ERR_ARG, "import: npayload");
    if (((uintptr_t)dev_ptr & 15) != 0) HQ_THROW(HQ_ERR_ARG, "import: pointer must be 16-byte aligned");
    if (meta->compact_kind == 4) {  // the ranked form of a sparse-key table (hq_build.cu)
      const int64_t range = (int64_t)meta->key_max - meta->key_min + 1;
      if (meta->layout != HQ_HT_LINEAR || meta->composite || meta->nkeys < 1 || range < 1 || range > (1LL << 31))
        HQ_THROW(HQ_ERR_ARG, "import: a ranked form needs a linear, non-composite table with its key range and count");
      int64_t od = 0, op = 0, tot = 0;
      int stride = 0;
      hq_ranked_layout(range, meta->nkeys, meta->npayload, &od, &op, &tot, &stride);
      if (meta->bytes < tot) HQ_THROW(HQ_ERR_ARG, "import: ranked form too small");
      hq_hash* h = new hq_hash();
      h->ctx = ctx;
      h->meta = *meta;
      h->meta.compact_kind = 0;
      h->meta.bytes = cap * meta->slot_words * 4;
      h->compact_borrow = dev_ptr;
      h->ckind = 4;
      h->cbytes = tot;
      h->roff_dir = od;
      h->roff_pay = op;
      h->rstride = stride;
      h->compact_only = true;
      int l = 0;
      while ((1LL << l) < cap) ++l;
      h->log2cap = l;
      h->checked = true;
      *out = h;
      return;
    }
    if (meta->compact_kind != 0) {  // a compact-only direct table: the buffer is its compact form
      if (meta->layout != HQ_HT_DIRECT ||
          meta->compact_kind != hq_compact_kind(meta->npayload, meta->pay_min, meta->pay_max))
        HQ_THROW(HQ_ERR_ARG, "import: compact_kind does not match the table");
      if (meta->bytes < hq_compact_words(meta->compact_kind, cap) * 4) HQ_THROW(HQ_ERR_ARG, "import: compact form too small");
      hq_hash* h = new hq_hash();
      h->ctx = ctx;
      h->meta = *meta;
      h->meta.compact_kind = 0;
      h->meta.bytes = cap * meta->slot_words * 4;
      h->compact_borrow = dev_ptr;
      h->ckind = meta->compact_kind;
      unsigned char lut[256];
      h->crank = h->ckind == 2 ? hq_rank_lut(*meta, lut) : 0;
      h->cbytes = hq_compact_words(h->ckind, cap) * 4;
      h->compact_only = true;
      int l = 0;
      while ((1LL << l) < cap) ++l;
      h->log2cap = l;
      h->checked = true;
      *out = h;
      return;
    }
    hq_hash* h = new hq_hash();
    h->ctx = ctx;
    h->meta = *meta;
    h->meta.bytes = cap * meta->slot_words * 4;
    h->slots = (uint32_t*)dev_ptr;
    int l = 0;
    while ((1LL << l) < cap) ++l;
    h->log2cap = l;
    h->checked = true;
    try {
      hq_build_compact(ctx, h);
    } catch (...) {
      h->release();
      throw;
    }
    *out = h;
  });
}

hq_status hq_free_hash(hq_hash* h) {
  return guarded([&] {
    if (h) h->release();
  });
}

// ---------------------------------------------------------------- pipelines
static void run_pipeline(hq_ctx* ctx, const hq_plan* plan, int64_t block_rows, hq_result** out) {
    if (!ctx || !plan || !out) HQ_THROW(HQ_ERR_ARG, "NULL argument");
    if (!plan->fact) HQ_THROW(HQ_ERR_ARG, "plan: fact table is NULL");
    if (plan->fact->dev_rows) {  // a view sized by a cached row count: check it once (host read)
      hq_require_eager(ctx, "a pipeline over a result view sized by its cached row count");
      unsigned long long* hc = (unsigned long long*)pinned_staging(ctx, 8);
      HQ_CUDA(cudaMemcpyAsync(hc, plan->fact->dev_rows, 8, cudaMemcpyDeviceToHost, ctx->stream));
      HQ_CUDA(cudaStreamSynchronize(ctx->stream));
      if ((int64_t)*hc != plan->fact->nrows) {
        ctx->derived_rows.erase(plan->fact->uid);
        HQ_THROW(HQ_ERR_STATE, "result view: the result's row count differs from the cached one (re-run the query)");
      }
      const_cast<hq_table*>(plan->fact)->dev_rows = nullptr;
    }
    hq_result* r = new hq_result();
    if (plan->fact->host_stream) r->stream_block = block_rows > 0 ? block_rows : HQ_STREAM_BLOCK_ROWS;
    r->fact = const_cast<hq_table*>(plan->fact);
    r->fact->retain();
    for (int o = 0; o < plan->nops && o < HQ_MAX_OPS; ++o)
      if (plan->ops[o].kind == HQ_OP_PROBE && plan->ops[o].ht) {
        hq_hash* h = const_cast<hq_hash*>(plan->ops[o].ht);
        h->retain();
        r->hashes.push_back(h);
      }
    try {
      if (ctx->capturing && (r->stream_block > 0 || (plan->exec != HQ_EXEC_FUSED && plan->exec != HQ_EXEC_FUSED_INTERP)))
        HQ_THROW(HQ_ERR_STATE, "not capturable in a CUDA graph: batch processing, multi-pass or operator-at-a-time");
      hq_prepare_result(ctx, plan, r);
    } catch (...) {
      r->release();
      throw;
    }
    r->capture_retain(ctx);
    *out = r;
}

hq_status hq_run_pipeline(hq_ctx* ctx, const hq_plan* plan, hq_result** out) {
  return guarded([&] { run_pipeline(ctx, plan, 0, out); });
}

hq_status hq_run_pipeline_streamed(hq_ctx* ctx, const hq_plan* plan, int64_t block_rows, hq_result** out) {
  return guarded([&] {
    if (plan && plan->fact && !plan->fact->host_stream)
      HQ_THROW(HQ_ERR_ARG, "hq_run_pipeline_streamed: the fact table is not HQ_HOST_STREAM");
    if (block_rows < 0) HQ_THROW(HQ_ERR_ARG, "block_rows < 0");
    run_pipeline(ctx, plan, block_rows, out);
  });
}

hq_status hq_finalize(hq_ctx* ctx, hq_result* r) {
  return guarded([&] {
    if (!ctx || !r) HQ_THROW(HQ_ERR_ARG, "NULL argument");
    hq_finalize_impl(ctx, r);
  });
}

hq_status hq_result_info_get(hq_ctx* ctx, hq_result* r, hq_result_info* out) {
  return guarded([&] {
    if (ctx) hq_require_eager(ctx, "hq_result_info_get");
    if (!ctx || !r || !out) HQ_THROW(HQ_ERR_ARG, "NULL argument");
    hq_finalize_impl(ctx, r);
    std::memset(out, 0, sizeof(*out));
    out->nrows = r->nrows;
    out->qualifying_rows = r->qualifying;
    out->ncols = r->ncols;
    for (int c = 0; c < r->ncols; ++c) out->types[c] = r->types[c];
    out->segment_rows = r->sink == HQ_SINK_MATERIALISE ? r->segment_rows : 0;
  });
}

hq_status hq_fetch_result(hq_ctx* ctx, hq_result* r, void* const* host_cols, int64_t capacity_rows,
                          int64_t* nrows_out) {
  return guarded([&] {
    if (ctx) hq_require_eager(ctx, "hq_fetch_result");
    if (!ctx || !r) HQ_THROW(HQ_ERR_ARG, "NULL argument");
    hq_finalize_impl(ctx, r);
    const int64_t n = std::min<int64_t>(r->nrows, capacity_rows);
    if (n > 0 && !host_cols) HQ_THROW(HQ_ERR_ARG, "host_cols is NULL");
    if (r->host_ready) {  // small result: rows came back with the finalize (no device access)
      for (int c = 0; c < r->ncols && n > 0; ++c)
        if (host_cols[c]) std::memcpy(host_cols[c], r->host_rows.data() + (size_t)c * r->nrows, (size_t)n * 8);
      if (nrows_out) *nrows_out = r->nrows;
      return;
    }
    for (int c = 0; c < r->ncols && n > 0; ++c) {
      if (!host_cols[c]) continue;
      const void* src = r->sink == HQ_SINK_MATERIALISE ? r->outcols[c].p : r->rescol[c];
      const size_t w = (size_t)hq_type_width(r->types[c]);
      HQ_CUDA(cudaMemcpyAsync(host_cols[c], src, (size_t)n * w, cudaMemcpyDeviceToHost, ctx->stream));
    }
    HQ_CUDA(cudaStreamSynchronize(ctx->stream));
    if (nrows_out) *nrows_out = r->nrows;
  });
}

// Identity of a result viewed as a table: its plan with every input replaced by the
// input's own identity (the fact table's uid, each probed table's build-statistics key),
// so that the same pipeline over the same tables yields the same uid step after step and
// a build over it (TPC-H Q3's orders side) finds its cached statistics -- verified on the
// device like any other (hq_build.cu).  0 (a fresh uid) when an input has no identity
// (an imported or expected_rows-sized table).
static uint64_t derived_uid(const hq_result* r) {
  if (!r->fact) return 0;
  hq_plan P = r->plan;
  std::string k;
  k.append((const char*)&r->fact->uid, sizeof(r->fact->uid));
  P.fact = nullptr;
  for (int i = 0; i < P.nops; ++i) {
    if (P.ops[i].kind != HQ_OP_PROBE) continue;
    if (!P.ops[i].ht || P.ops[i].ht->stats_key.empty()) return 0;
    const std::string& sk = P.ops[i].ht->stats_key;
    const uint64_t n = sk.size();
    k.append((const char*)&n, sizeof n);
    k.append(sk);
    P.ops[i].ht = nullptr;
  }
  k.append((const char*)&P, sizeof P);
  return std::hash<std::string>{}(k) | (1ull << 63);  // (counter uids stay below 2^63)
}

hq_status hq_result_as_table(hq_ctx* ctx, hq_result* r, hq_table** out) {
  return guarded([&] {
    if (!ctx || !r || !out) HQ_THROW(HQ_ERR_ARG, "NULL argument");
    const bool mat = r->sink == HQ_SINK_MATERIALISE;
    const uint64_t duid = derived_uid(r);
    // a materialised result seen before under the same identity: its row count is known,
    // the view needs no finalize (no host sync; also inside a graph capture) -- the row
    // counter on the device is checked by the table's consumers instead (dev_rows)
    // (only where the count is the result's one possible fault: no division / modulo in
    // its expressions, whose faults only the finalize would read)
    bool faultless = true;
    for (int i = 0; i < r->plan.nops; ++i)
      if (r->plan.ops[i].kind == HQ_OP_COMPUTE)
        for (int k = 0; k < r->plan.ops[i].ninsn && k < HQ_MAX_INSN; ++k)
          faultless = faultless && r->plan.ops[i].code[k].opc != HQ_I_DIV && r->plan.ops[i].code[k].opc != HQ_I_MOD;
    auto known = duid && mat && faultless && !r->finalized ? ctx->derived_rows.find(duid) : ctx->derived_rows.end();
    const bool lazy = known != ctx->derived_rows.end() && !getenv("HQ_NO_DERIVED_ROWS");
    if (lazy) {
      r->nrows = known->second;
      r->ncols = r->plan.nout;
      for (int j = 0; j < r->plan.nout; ++j) r->types[j] = r->plan.out_type[j];
      if (r->capacity < r->nrows) HQ_THROW(HQ_ERR_STATE, "result view: cached row count exceeds the capacity");
    } else {
      hq_require_eager(ctx, "hq_result_as_table");
      hq_finalize_impl(ctx, r, /*unordered=*/true);
      if (duid && mat) ctx->derived_rows[duid] = r->nrows;
    }
    for (int c = 0; c < r->ncols; ++c)
      if (r->types[c] == HQ_F64) HQ_THROW(HQ_ERR_UNSUPPORTED, "result has fp64 (AVG) columns: not a table");
    hq_table* t = new hq_table();
    t->ctx = ctx;
    if (duid) t->uid = duid;
    if (lazy) t->dev_rows = (const unsigned long long*)r->dstate.p;  // the materialise counter
    t->nrows = r->nrows;
    t->ncols = r->ncols;
    for (int c = 0; c < r->ncols; ++c) {
      t->cols[c].ptr = mat ? r->outcols[c].p : r->rescol[c];
      t->cols[c].type = r->types[c];
      t->cols[c].width = hq_type_width(r->types[c]);
    }
    r->retain();
    t->backing = r;
    *out = t;
  });
}

hq_status hq_result_partials_view(hq_result* r, void** dev_ptr, size_t* bytes) {
  return guarded([&] {
    if (!r) HQ_THROW(HQ_ERR_ARG, "result is NULL");
    if (r->sink != HQ_SINK_AGG || r->gmode == hqk::GM_HASH)
      HQ_THROW(HQ_ERR_UNSUPPORTED, "partials view needs a dense (or scalar) aggregation result");
    for (int a = 0; a < r->plan.naggs; ++a)
      if (r->plan.agg_fn[a] == HQ_AGG_MIN || r->plan.agg_fn[a] == HQ_AGG_MAX)
        HQ_THROW(HQ_ERR_UNSUPPORTED, "partials view: MIN/MAX do not combine with a SUM reduce");
    if (r->finalized) HQ_THROW(HQ_ERR_STATE, "result already finalized");
    if (dev_ptr) *dev_ptr = r->gtab.p;
    if (bytes) *bytes = (size_t)r->ngroups * r->vwords * 8;
  });
}

hq_status hq_result_from_partials(hq_ctx* ctx, hq_result* r, const void* dev_ptr, size_t bytes) {
  return guarded([&] {
    if (!ctx || !r || !dev_ptr) HQ_THROW(HQ_ERR_ARG, "NULL argument");
    void* p = nullptr;
    size_t n = 0;
    const hq_status st = hq_result_partials_view(r, &p, &n);
    if (st != HQ_OK) HQ_THROW(st, g_last_error);
    if (bytes != n) HQ_THROW(HQ_ERR_ARG, "hq_result_from_partials: size differs from the partials view");
    if (p != dev_ptr && n > 0) HQ_CUDA(cudaMemcpyAsync(p, dev_ptr, n, cudaMemcpyDeviceToDevice, ctx->stream));
  });
}

hq_status hq_result_to_partials(hq_ctx* ctx, const hq_result* r, void* dev_dst, size_t bytes) {
  return guarded([&] {
    if (!ctx || !r || !dev_dst) HQ_THROW(HQ_ERR_ARG, "NULL argument");
    void* p = nullptr;
    size_t n = 0;
    const hq_status st = hq_result_partials_view(const_cast<hq_result*>(r), &p, &n);
    if (st != HQ_OK) HQ_THROW(st, g_last_error);
    if (bytes != n) HQ_THROW(HQ_ERR_ARG, "hq_result_to_partials: size differs from the partials view");
    if (p != dev_dst && n > 0) HQ_CUDA(cudaMemcpyAsync(dev_dst, p, n, cudaMemcpyDeviceToDevice, ctx->stream));
  });
}

hq_status hq_hash_pack(hq_ctx* ctx, const hq_hash* const* hashes, int32_t n, const int64_t* offs, void* dev_dst) {
  return guarded([&] {
    if (!ctx || n < 0 || (n > 0 && (!hashes || !offs || !dev_dst))) HQ_THROW(HQ_ERR_ARG, "NULL argument");
    for (int i = 0; i < n; ++i) {
      const hq_hash* h = hashes[i];
      if (!h) HQ_THROW(HQ_ERR_ARG, "hq_hash_pack: NULL hash");
      if (offs[i] < 0 || (offs[i] & 15)) HQ_THROW(HQ_ERR_ARG, "hq_hash_pack: offsets must be 16-B aligned");
      const void* src = h->compact_only ? h->compact_ptr() : (const void*)h->slots;
      const size_t bytes = (size_t)(h->compact_only ? h->cbytes : h->meta.bytes);
      if (bytes) HQ_CUDA(cudaMemcpyAsync((char*)dev_dst + offs[i], src, bytes, cudaMemcpyDeviceToDevice, ctx->stream));
    }
  });
}

hq_status hq_gather_faults(hq_ctx* ctx, const hq_hash* const* hashes, int32_t nh, const hq_result* const* results,
                           int32_t nr, int64_t* dev_out) {
  return guarded([&] {
    if (!ctx || !dev_out || nh < 0 || nr < 0) HQ_THROW(HQ_ERR_ARG, "NULL argument or negative count");
    if ((nh > 0 && !hashes) || (nr > 0 && !results)) HQ_THROW(HQ_ERR_ARG, "NULL handle array");
    std::vector<const int*> hw, rw;
    for (int i = 0; i < nh; ++i) {
      if (!hashes[i]) HQ_THROW(HQ_ERR_ARG, "NULL hash");
      if (hashes[i]->dstate.p) hw.push_back(hashes[i]->dstate.as<int>());  // imported tables: no build here
    }
    for (int i = 0; i < nr; ++i) {
      if (!results[i]) HQ_THROW(HQ_ERR_ARG, "NULL result");
      if (results[i]->dstate.p) rw.push_back((const int*)(results[i]->dstate.as<char>() + 8));
    }
    hq_launch_gather_faults(ctx, hw, rw, (long long*)dev_out);
  });
}

hq_status hq_raise_faults(const int64_t* w) {
  return guarded([&] {
    if (!w) HQ_THROW(HQ_ERR_ARG, "NULL argument");
    auto b = [&](int bit) { return w[bit] != 0; };
    auto pb = [&](int flag) { int k = 0; while ((1 << k) != flag) ++k; return w[16 + k] != 0; };
    auto hb = [&](int flag) { int k = 0; while ((1 << k) != flag) ++k; return b(k); };
    // (stale statistics first: a table sized from them can also report keys out of range)
    if (hb(HQF_STALE)) HQ_THROW(HQ_ERR_STATE, "hash build: source rows differ from the cached build statistics");
    if (hb(HQF_DUP_KEY)) HQ_THROW(HQ_ERR_DUP_KEY, "hash build: duplicate key (join keys must be unique)");
    if (hb(HQF_BAD_KEY)) HQ_THROW(HQ_ERR_ARG, "hash build: key INT32_MIN or outside int32");
    if (hb(HQF_BAD_PAYLOAD)) HQ_THROW(HQ_ERR_ARG, "hash build: payload outside int32");
    if (hb(HQF_HT_FULL)) HQ_THROW(HQ_ERR_OVERFLOW, "hash build: table full (expected_rows too small)");
    if (pb(HQF_DIV_ZERO)) HQ_THROW(HQ_ERR_ARG, "pipeline: division by zero");
    if (pb(HQF_KEY_DOMAIN)) HQ_THROW(HQ_ERR_ARG, "pipeline: group key outside its declared [min, min+card)");
    if (pb(HQF_OVERFLOW)) HQ_THROW(HQ_ERR_OVERFLOW, "aggregate exceeds the int64 guard (|v| >= 2^62)");
  });
}

hq_status hq_free_result(hq_result* r) {
  return guarded([&] {
    if (r) r->release();
  });
}

}  // extern "C"
