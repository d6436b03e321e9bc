// jit_codegen_check.cu -- CPU-side check of libhq's query compiler (hq_jit.cu):
// builds device plans for a matrix of pipeline shapes from fake (never
// dereferenced) device pointers, generates each kernel's CUDA source and
// compiles it with NVRTC for sm_100a.  No GPU needed: NVRTC is a compiler.
//
// Shapes mirror what the engine emits (§5.2 compound kernels):
// star joins with staged / global compact / direct / linear probes, scalar,
// dense, lane-private and hash group-by sinks, materialisation, and the C2
// (atomic) ablation.  Usage: jit_codegen_check [dump_dir]; prints "OK <n>".
#include <nvrtc.h>

#include <cstdio>
#include <cstdlib>
#include <string>
#include <vector>

#include "hq_internal.h"

using namespace hqk;

namespace {
void* fake_alloc(size_t bytes, void*, void*) { return calloc(1, bytes + 64); }
void fake_free(void* p, size_t, void*, void*) { free(p); }

hq_ctx* make_ctx() {
  hq_ctx* c = new hq_ctx();
  c->has_alloc = true;
  c->alloc = {fake_alloc, fake_free, nullptr};
  return c;
}

// fact table: k1..k4 i32 keys, v1 v2 i32, v64 i64, f8 i8 (pointers are fake)
hq_table* make_fact(hq_ctx* c) {
  hq_table* t = new hq_table();
  t->ctx = c;
  t->nrows = 6000000;
  const int types[8] = {HQ_I32, HQ_I32, HQ_I32, HQ_I32, HQ_I32, HQ_I32, HQ_I64, HQ_I8};
  t->ncols = 8;
  for (int i = 0; i < 8; ++i) {
    t->cols[i].ptr = (const void*)(uintptr_t)(0x7f0000000000ull + (uint64_t)i * 0x10000000ull);
    t->cols[i].type = types[i];
    t->cols[i].width = hq_type_width(types[i]);
  }
  return t;
}

// ckind: 0 none, 1 bitmap, 2 byte, 3 nibble; linear: HQ_HT_LINEAR (+ prefilter)
hq_hash* make_hash(hq_ctx* c, int layout, int npay, int ckind, int64_t range, bool prefilter = false) {
  hq_hash* h = new hq_hash();
  h->ctx = c;
  h->meta.layout = layout;
  h->meta.npayload = npay;
  h->meta.slot_words = npay == 0 ? 1 : (npay == 1 ? 2 : 4);
  h->meta.key_min = 7;
  h->meta.key_max = (int32_t)(7 + range - 1);
  h->meta.pay_min = ckind == 3 ? 1992 : 0;
  h->meta.pay_max = ckind == 3 ? 1998 : 24;
  if (layout == HQ_HT_DIRECT) {
    h->meta.capacity = range;
  } else {
    int l = 10;
    while ((1ll << l) < range * 2) ++l;
    h->meta.capacity = 1ll << l;
    h->log2cap = l;
  }
  h->meta.bytes = h->meta.capacity * h->meta.slot_words * 4;
  h->slots = (uint32_t*)(uintptr_t)0x7e0000000000ull;
  if (ckind) {
    h->ckind = ckind;
    h->cbytes = ckind == 1 ? (range + 31) / 32 * 4 : (ckind == 2 ? (range + 3) / 4 * 4 : (range + 7) / 8 * 4);
    h->compact = DevBuf(c, 64);
  }
  if (prefilter) {
    h->pf_words = (range + 31) / 32;
    h->prefilter = DevBuf(c, 64);
  }
  return h;
}

// ranked form of a sparse-key linear table (hq_hash::ranked): bitmap | directory | rows
hq_hash* make_ranked(hq_ctx* c, int npay, int64_t range, int64_t nkeys) {
  hq_hash* h = make_hash(c, HQ_HT_LINEAR, npay, 0, range);
  h->slots = nullptr;
  h->meta.nkeys = nkeys;
  int64_t od, op, tot;
  int st;
  hq_ranked_layout(range, nkeys, npay, &od, &op, &tot, &st);
  h->ckind = 4;
  h->cbytes = tot;
  h->roff_dir = od;
  h->roff_pay = op;
  h->rstride = st;
  h->compact = DevBuf(c, 64);
  h->compact_only = true;
  return h;
}

hq_op probe(const hq_hash* h, int key, int mode, int dst = -1, int dst2 = -1) {
  hq_op o{};
  o.kind = HQ_OP_PROBE;
  o.ht = h;
  o.key_reg = key;
  o.mode = mode;
  if (dst >= 0) {
    o.npayload = 1;
    o.payload_dst[0] = dst;
  }
  if (dst2 >= 0) {
    o.npayload = 2;
    o.payload_dst[1] = dst2;
  }
  return o;
}
hq_op filter(int reg, int cmp, int64_t lo, int64_t hi = 0) {
  hq_op o{};
  o.kind = HQ_OP_FILTER;
  o.filter.reg = reg;
  o.filter.cmp = cmp;
  o.filter.lo = lo;
  o.filter.hi = hi;
  return o;
}
hq_op compute(int dst, std::vector<hq_insn> code) {
  hq_op o{};
  o.kind = HQ_OP_COMPUTE;
  o.dst = dst;
  o.ninsn = (int)code.size();
  for (size_t i = 0; i < code.size(); ++i) o.code[i] = code[i];
  return o;
}

struct Shape {
  std::string name;
  hq_plan plan;
  const char* env_r;  // HQ_JIT_R override (nullptr = default)
  int mp = 0;         // multi-pass kernel: 1 = count, 2 = write
};

bool compile(const std::string& name, const std::string& src, const char* dump) {
  if (dump) {
    const std::string path = std::string(dump) + "/" + name + ".cu";
    if (FILE* f = fopen(path.c_str(), "w")) {
      fwrite(src.data(), 1, src.size(), f);
      fclose(f);
    }
  }
  nvrtcProgram prog;
  if (nvrtcCreateProgram(&prog, src.c_str(), (name + ".cu").c_str(), 0, nullptr, nullptr) != NVRTC_SUCCESS) return false;
  const char* opts[] = {"--gpu-architecture=sm_100a", "-std=c++17", "-lineinfo", "--device-int128"};
  const nvrtcResult rc = nvrtcCompileProgram(prog, 4, opts);
  bool ok = rc == NVRTC_SUCCESS;
  if (ok) {
    size_t n = 0;
    ok = nvrtcGetCUBINSize(prog, &n) == NVRTC_SUCCESS && n > 0;
  } else {
    size_t n = 0;
    nvrtcGetProgramLogSize(prog, &n);
    std::string log(n, '\0');
    nvrtcGetProgramLog(prog, &log[0]);
    fprintf(stderr, "FAIL %s:\n%s\n", name.c_str(), log.substr(0, 3000).c_str());
  }
  nvrtcDestroyProgram(&prog);
  return ok;
}
}  // namespace

int main(int argc, char** argv) {
  const char* dump = argc > 1 ? argv[1] : nullptr;
  hq_ctx* c = make_ctx();
  hq_table* F = make_fact(c);
  hq_hash* semi_small = make_hash(c, HQ_HT_DIRECT, 0, 1, 20000);      // staged bitmap
  hq_hash* byte_big = make_hash(c, HQ_HT_DIRECT, 1, 2, 3000000);      // global byte map
  hq_hash* semi_big = make_hash(c, HQ_HT_DIRECT, 0, 1, 1400000);      // global bitmap (> stage budget)
  hq_hash* nib = make_hash(c, HQ_HT_DIRECT, 1, 3, 61131);             // staged nibbles
  hq_hash* byte_small = make_hash(c, HQ_HT_DIRECT, 1, 2, 20000);      // staged byte map
  hq_hash* direct2 = make_hash(c, HQ_HT_DIRECT, 2, 0, 500000);        // slot array, 4 words
  hq_hash* direct1 = make_hash(c, HQ_HT_DIRECT, 1, 0, 500000);        // slot array, 2 words
  hq_hash* lin_pf = make_hash(c, HQ_HT_LINEAR, 2, 0, 800000, true);   // linear + prefilter
  hq_hash* lin_semi = make_hash(c, HQ_HT_LINEAR, 0, 0, 300000, false);
  hq_hash* lin_1 = make_hash(c, HQ_HT_LINEAR, 1, 0, 300000, false);

  std::vector<Shape> shapes;
  auto star = [&](int res) {
    hq_plan P{};
    P.fact = F;
    P.row_end = -1;
    P.ops[P.nops++] = probe(semi_small, 1, HQ_PROBE_SEMI);
    P.ops[P.nops++] = probe(byte_big, 0, HQ_PROBE_INNER, HQ_TMP(0));
    P.ops[P.nops++] = probe(semi_big, 2, HQ_PROBE_SEMI);
    P.ops[P.nops++] = probe(nib, 3, HQ_PROBE_INNER, HQ_TMP(1));
    P.ops[P.nops++] = compute(HQ_TMP(2), {{HQ_I_LOAD, 4, 0}, {HQ_I_SUB, 5, 0}});
    P.sink = HQ_SINK_AGG;
    P.resolution = res;
    P.nkeys = 2;
    P.key_reg[0] = HQ_TMP(1); P.key_min[0] = 1992; P.key_card[0] = 7;
    P.key_reg[1] = HQ_TMP(0); P.key_min[1] = 0; P.key_card[1] = 25;
    P.naggs = 2;
    P.agg_fn[0] = HQ_AGG_SUM; P.agg_reg[0] = HQ_TMP(2);
    P.agg_fn[1] = HQ_AGG_COUNT;
    return P;
  };
  shapes.push_back({"star_dense_lrgp", star(HQ_RES_LRGP), nullptr});
  shapes.push_back({"star_dense_atomic", star(HQ_RES_ATOMIC), nullptr});
  shapes.push_back({"star_dense_r4", star(HQ_RES_LRGP), "4"});
  {  // Q3.1-like: three inner probes, dense keys too big for a shared dense table
    hq_plan P{};
    P.fact = F;
    P.row_end = -1;
    P.ops[P.nops++] = probe(byte_small, 1, HQ_PROBE_INNER, HQ_TMP(0));
    P.ops[P.nops++] = probe(byte_big, 0, HQ_PROBE_INNER, HQ_TMP(1));
    P.ops[P.nops++] = probe(nib, 2, HQ_PROBE_INNER, HQ_TMP(2));
    P.sink = HQ_SINK_AGG;
    P.nkeys = 3;
    P.key_reg[0] = HQ_TMP(1); P.key_card[0] = 25;
    P.key_reg[1] = HQ_TMP(0); P.key_card[1] = 25;
    P.key_reg[2] = HQ_TMP(2); P.key_min[2] = 1992; P.key_card[2] = 7;
    P.naggs = 2;
    P.agg_fn[0] = HQ_AGG_SUM; P.agg_reg[0] = 3;
    P.agg_fn[1] = HQ_AGG_COUNT;
    shapes.push_back({"star_smem_hash", P, nullptr});
    // the same with build-side payload ranges 8..20 (one region's nations):
    // the shared table becomes dense over the narrowed 13 x 13 x 7 domain
    hq_hash* na = make_hash(c, HQ_HT_DIRECT, 1, 2, 20000);
    hq_hash* nb = make_hash(c, HQ_HT_DIRECT, 1, 2, 3000000);
    na->meta.pay_min = nb->meta.pay_min = 8;
    na->meta.pay_max = nb->meta.pay_max = 20;
    P.ops[0] = probe(na, 1, HQ_PROBE_INNER, HQ_TMP(0));
    P.ops[1] = probe(nb, 0, HQ_PROBE_INNER, HQ_TMP(1));
    shapes.push_back({"star_narrowed_dense", P, nullptr});
    // payloads of five distinct values spread over 4..24 (SSB Q3.1's ASIA
    // nations): keys indexed by rank, a 5 x 5 x 7 dense shared table
    hq_hash* ra = make_hash(c, HQ_HT_DIRECT, 1, 2, 20000);
    hq_hash* rb = make_hash(c, HQ_HT_DIRECT, 1, 2, 3000000);
    for (hq_hash* h : {ra, rb}) {
      h->meta.pay_min = 4;
      h->meta.pay_max = 24;
      for (int v : {4, 9, 10, 13, 24}) h->meta.pay_set[v >> 6] |= 1ull << (v & 63);
      h->crank = 1;  // rank-coded byte maps (hq_build_compact)
    }
    P.ops[0] = probe(ra, 1, HQ_PROBE_INNER, HQ_TMP(0));
    P.ops[1] = probe(rb, 0, HQ_PROBE_INNER, HQ_TMP(1));
    shapes.push_back({"star_ranked_dense", P, nullptr});
  }
  {  // Q6-like scalar aggregate with an int8 bitmap filter and an i64 expression
    hq_plan P{};
    P.fact = F;
    P.row_end = -1;
    P.ops[P.nops++] = filter(4, HQ_BETWEEN, 19940101, 19941231);
    hq_op f = filter(7, HQ_IN_BITMAP, 0);
    f.filter.bitmap[0] = 0x1Cull;
    P.ops[P.nops++] = f;
    P.ops[P.nops++] = filter(5, HQ_LT, 24);
    P.ops[P.nops++] = compute(HQ_TMP(0), {{HQ_I_LOAD, 6, 0}, {HQ_I_MUL, 7, 0}});
    P.sink = HQ_SINK_AGG;
    P.naggs = 2;
    P.agg_fn[0] = HQ_AGG_SUM; P.agg_reg[0] = HQ_TMP(0);
    P.agg_fn[1] = HQ_AGG_MAX; P.agg_reg[1] = 6;
    shapes.push_back({"scalar_filters", P, nullptr});
  }
  {  // Q1-like: probe-free, tiny dense domain -> lane-private tables
    hq_plan P{};
    P.fact = F;
    P.row_end = -1;
    P.ops[P.nops++] = filter(4, HQ_LE, 19980902);
    P.ops[P.nops++] = compute(HQ_TMP(0), {{HQ_I_LOAD, 5, 0}, {HQ_I_RSUB, -1, 100}, {HQ_I_MUL, 6, 0}});
    P.sink = HQ_SINK_AGG;
    P.nkeys = 2;
    P.key_reg[0] = 7; P.key_card[0] = 3;
    P.key_reg[1] = 0; P.key_card[1] = 2;
    P.naggs = 5;
    P.agg_fn[0] = HQ_AGG_SUM; P.agg_reg[0] = 6;
    P.agg_fn[1] = HQ_AGG_SUM; P.agg_reg[1] = HQ_TMP(0);
    P.agg_fn[2] = HQ_AGG_AVG; P.agg_reg[2] = 6;
    P.agg_fn[3] = HQ_AGG_COUNT;
    P.agg_fn[4] = HQ_AGG_MIN; P.agg_reg[4] = 5;
    shapes.push_back({"lane_private", P, nullptr});
  }
  auto mat = [&](int res) {
    hq_plan P{};
    P.fact = F;
    P.row_end = -1;
    P.ops[P.nops++] = filter(4, HQ_GT, 10);
    P.ops[P.nops++] = probe(direct2, 0, HQ_PROBE_INNER, HQ_TMP(0));
    P.ops[P.nops++] = probe(lin_pf, 1, HQ_PROBE_INNER, HQ_TMP(1));
    P.ops[P.nops++] = probe(direct1, 2, HQ_PROBE_SEMI);
    P.sink = HQ_SINK_MATERIALISE;
    P.resolution = res;
    P.nout = 3;
    P.out_reg[0] = 0; P.out_type[0] = HQ_I32;
    P.out_reg[1] = HQ_TMP(1); P.out_type[1] = HQ_I32;
    P.out_reg[2] = 6; P.out_type[2] = HQ_I64;
    return P;
  };
  shapes.push_back({"materialise_lrgp", mat(HQ_RES_LRGP), nullptr});
  shapes.push_back({"materialise_atomic", mat(HQ_RES_ATOMIC), nullptr});
  {  // anti + linear semi + linear inner, hash group-by over a huge key domain (TPC-H Q3-like)
    hq_plan P{};
    P.fact = F;
    P.row_end = -1;
    P.ops[P.nops++] = probe(lin_semi, 0, HQ_PROBE_ANTI);
    P.ops[P.nops++] = probe(lin_1, 1, HQ_PROBE_INNER, HQ_TMP(0));
    P.ops[P.nops++] = probe(semi_big, 2, HQ_PROBE_ANTI);
    P.sink = HQ_SINK_AGG;
    P.nkeys = 2;
    P.key_reg[0] = 1; P.key_card[0] = 1ll << 31;
    P.key_reg[1] = HQ_TMP(0); P.key_card[1] = 8;
    P.naggs = 2;
    P.agg_fn[0] = HQ_AGG_SUM; P.agg_reg[0] = 6;
    P.agg_fn[1] = HQ_AGG_COUNT;
    P.group_capacity = 100000;
    shapes.push_back({"global_hash_groups", P, nullptr});
    shapes.push_back({"global_hash_groups_r4", P, "4"});
  }

  {  // ranked sparse-key tables: an inner probe with two payloads (TPC-H Q3's orders:
     // orderdate, shippriority), a semi-join (bitmap only) and an outer probe with one payload
    hq_hash* rk2 = make_ranked(c, 2, 180000000, 4400000);
    hq_hash* rk0 = make_ranked(c, 0, 6000000, 1000000);
    hq_hash* rk1 = make_ranked(c, 1, 3000000, 200000);
    hq_plan P{};
    P.fact = F;
    P.row_end = -1;
    P.ops[P.nops++] = filter(3, HQ_GT, 19950315);
    P.ops[P.nops++] = probe(rk2, 1, HQ_PROBE_INNER, HQ_TMP(0), HQ_TMP(1));
    P.ops[P.nops++] = probe(rk0, 2, HQ_PROBE_SEMI);
    P.ops[P.nops++] = probe(rk1, 0, HQ_PROBE_OUTER, HQ_TMP(2));
    P.sink = HQ_SINK_AGG;
    P.nkeys = 3;
    P.key_reg[0] = 1; P.key_card[0] = 1ll << 31;
    P.key_reg[1] = HQ_TMP(0); P.key_min[1] = 19920101; P.key_card[1] = 70000;
    P.key_reg[2] = HQ_TMP(1); P.key_card[2] = 8;
    P.naggs = 2;
    P.agg_fn[0] = HQ_AGG_SUM; P.agg_reg[0] = HQ_TMP(2);
    P.agg_fn[1] = HQ_AGG_COUNT;
    P.group_capacity = 600000;
    shapes.push_back({"ranked_probes", P, nullptr});
  }

  {  // LEFT OUTER probes (byte map, linear, direct) and predicate expressions (TPC-H Q13 / Q19 shapes)
    // the byte map rank-coded over a sparse payload set (Q13's orders-per-customer counts)
    byte_big = make_hash(c, HQ_HT_DIRECT, 1, 2, 3000000);
    for (int v : {1, 2, 5, 7, 24}) byte_big->meta.pay_set[v >> 6] |= 1ull << (v & 63);
    byte_big->crank = 1;
    hq_plan P{};
    P.fact = F;
    P.row_end = -1;
    P.ops[P.nops++] = probe(byte_big, 0, HQ_PROBE_OUTER, HQ_TMP(0));
    P.ops[P.nops++] = probe(lin_1, 1, HQ_PROBE_OUTER, HQ_TMP(1));
    P.ops[P.nops++] = probe(direct2, 2, HQ_PROBE_OUTER, HQ_TMP(2));
    P.ops[P.nops++] = compute(HQ_TMP(3), {{HQ_I_LOAD, -1, 1}, {HQ_I_AND_EQ, HQ_TMP(0), 3}, {HQ_I_AND_IN, 7, 0x0F0F},
                                          {HQ_I_AND_LE, 5, 7}});
    P.ops[P.nops++] = compute(HQ_TMP(4), {{HQ_I_LOAD, -1, 1}, {HQ_I_AND_GE, HQ_TMP(1), 2}, {HQ_I_AND_NE, 4, 9},
                                          {HQ_I_AND_LT, 5, 3}, {HQ_I_AND_GT, 6, 0}, {HQ_I_OR, HQ_TMP(3), 0}});
    P.ops[P.nops++] = filter(HQ_TMP(4), HQ_NE, 0);
    P.sink = HQ_SINK_AGG;
    P.nkeys = 1;
    P.key_reg[0] = HQ_TMP(0); P.key_card[0] = 25;
    P.naggs = 2;
    P.agg_fn[0] = HQ_AGG_SUM; P.agg_reg[0] = 6;
    P.agg_fn[1] = HQ_AGG_COUNT;
    shapes.push_back({"outer_predicates", P, nullptr});
  }

  {  // composite (two-column) join key in a linear table: slot {k1, k2, payload, -} (TPC-H Q9)
    hq_hash* comp = make_hash(c, HQ_HT_LINEAR, 2, 0, 800000, true);
    comp->meta.composite = 1;
    hq_plan P{};
    P.fact = F;
    P.row_end = -1;
    hq_op pc = probe(comp, 1, HQ_PROBE_INNER, HQ_TMP(0));
    pc.key2_reg = 2;
    P.ops[P.nops++] = pc;
    hq_op ps = probe(comp, 3, HQ_PROBE_SEMI);
    ps.key2_reg = 0;
    P.ops[P.nops++] = ps;
    P.sink = HQ_SINK_AGG;
    P.nkeys = 1;
    P.key_reg[0] = 7; P.key_card[0] = 16;
    P.naggs = 2;
    P.agg_fn[0] = HQ_AGG_SUM; P.agg_reg[0] = HQ_TMP(0);
    P.agg_fn[1] = HQ_AGG_COUNT;
    shapes.push_back({"composite_probe", P, nullptr});
  }

  // Resolution:WE (App C, Fig 24) variants: B3-WE tree, A3-WE scan, C3-WE sort +
  // segmented scan into a dense and into a hash global table
  {
    std::vector<Shape> wes;
    for (const Shape& s : shapes) {
      if (s.name != "star_ranked_dense" && s.name != "materialise_lrgp" && s.name != "scalar_filters" &&
          s.name != "global_hash_groups" && s.name != "ranked_probes")
        continue;
      Shape w = s;
      w.name = s.name + "_we";
      w.plan.resolution = HQ_RES_WE;
      wes.push_back(w);
    }
    for (const Shape& w : wes) shapes.push_back(w);
  }

  // multi-pass count / write kernels (HQ_EXEC_MULTIPASS) of a grouped star
  // join, a materialising pipeline and a scalar aggregate
  {
    std::vector<Shape> mps;
    for (const Shape& s : shapes) {
      if (s.name != "star_ranked_dense" && s.name != "materialise_lrgp" && s.name != "scalar_filters" &&
          s.name != "outer_predicates" && s.name != "composite_probe" && s.name != "ranked_probes")
        continue;
      for (int pass : {1, 2}) {
        Shape m = s;
        m.name = s.name + "_mp" + std::to_string(pass);
        m.plan.exec = HQ_EXEC_MULTIPASS;
        m.mp = pass;
        mps.push_back(m);
      }
    }
    for (const Shape& m : mps) shapes.push_back(m);
  }

  int ok = 0;
  for (const Shape& s : shapes) {
    if (s.env_r) {  // R = 4 rows per lane needs fewer consumer warps
      setenv("HQ_JIT_R", s.env_r, 1);
      setenv("HQ_JIT_NW", "15", 1);
    } else {
      unsetenv("HQ_JIT_R");
      unsetenv("HQ_JIT_NW");
    }
    hq_result* r = new hq_result();
    r->ctx = c;
    r->plan = s.plan;
    r->fact = F;
    r->dstate = DevBuf(c, 32);
    r->mp_flags_col = (const char*)(uintptr_t)0x7d0000000000ull;
    r->mp_pos_col = (const char*)(uintptr_t)0x7d8000000000ull;
    std::string src;
    try {
      KPlan kp;
      hq_build_kplan(c, r, kp, 0, s.mp ? 1000 : 0, true, s.mp);
      if (s.mp == 1) {
        kp.nout = 1;
        kp.out_ptr[0] = (void*)r->mp_flags_col;
      }
      src = hq_jit_source(kp);
    } catch (const HqError& e) {
      fprintf(stderr, "FAIL %s: plan: %s\n", s.name.c_str(), e.msg.c_str());
      continue;
    }
    if (compile(s.name, src, dump)) ++ok;
  }
  printf("OK %d of %d\n", ok, (int)shapes.size());
  return ok == (int)shapes.size() ? 0 : 1;
}
