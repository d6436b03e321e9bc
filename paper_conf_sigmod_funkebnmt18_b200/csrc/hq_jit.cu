// hq_jit.cu -- query compilation of a fusion operator into a specialised
// sm_100a kernel with NVRTC (§4.3 code templates + code frame,
// P:652-704; §5.2 compound-kernel code generation).
//
// The validated device plan (KPlan, hq_plan.cu) is turned into CUDA source:
// the code frame is the same persistent TMA-ring kernel as the interpreter
// (hq_pipeline.cu) -- producer warp, mbarrier full/empty ring, ragged tiles,
// LRGP sinks -- but every operator becomes straight-line code with its
// constants folded, columns loaded from the stage on first use and
// temporaries (probe payloads, expression results) kept in registers.  The
// source is compiled once per distinct plan shape (cached by source text),
// loaded with the driver API (entry points from cudaGetDriverEntryPoint, so
// libhq does not link libcuda) and launched on the context stream.
#include <cuda.h>
#include <nvrtc.h>

#include <climits>
#include <map>
#include <mutex>
#include <set>
#include <sstream>

#include "hq_internal.h"

using namespace hqk;

// kernel parameters of every generated kernel (mirrored in the generated source)
#define HQ_JPARAMS_DEF                                                                                         \
  struct JParams {                                                                                             \
    long long row_begin, row_end;                                                                              \
    const char* col[16];                                                                                       \
    const unsigned* ht[8];                                                                                     \
    const void* ctab[8];                                                                                       \
    const unsigned* pf[8];                                                                                     \
    const int* rpay[8];                                                                                        \
    long long* gtab;                                                                                           \
    unsigned long long gmask;                                                                                  \
    int glog2, pad;                                                                                            \
    void* out[8];                                                                                              \
    long long capacity;                                                                                        \
    unsigned long long* counter;                                                                               \
    int* err;                                                                                                  \
    long long* prof;                                                                                           \
  };
HQ_JPARAMS_DEF
#define HQ_XSTR(...) #__VA_ARGS__
#define HQ_STR(...) HQ_XSTR(__VA_ARGS__)

namespace {

const char* kPrelude =
#include "hq_jit_prelude.inc"
    ;

// ---- driver API through the runtime's entry-point query
typedef CUresult (*PFN_modload)(CUmodule*, const void*);
typedef CUresult (*PFN_getfn)(CUfunction*, CUmodule, const char*);
typedef CUresult (*PFN_setattr)(CUfunction, CUfunction_attribute, int);
typedef CUresult (*PFN_launch)(CUfunction, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned,
                               CUstream, void**, void**);
struct Driver {
  PFN_modload modload = nullptr;
  PFN_getfn getfn = nullptr;
  PFN_setattr setattr = nullptr;
  PFN_launch launch = nullptr;
};
template <class F>
F entry(const char* name) {
  void* fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  if (cudaGetDriverEntryPoint(name, &fn, cudaEnableDefault, &q) != cudaSuccess || !fn) {
    cudaGetLastError();
    HQ_THROW(HQ_ERR_CUDA, std::string("driver entry point missing: ") + name);
  }
  return (F)fn;
}
Driver& driver() {
  static Driver d;
  static std::once_flag once;
  std::call_once(once, [] {
    d.modload = entry<PFN_modload>("cuModuleLoadData");
    d.getfn = entry<PFN_getfn>("cuModuleGetFunction");
    d.setattr = entry<PFN_setattr>("cuFuncSetAttribute");
    d.launch = entry<PFN_launch>("cuLaunchKernel");
  });
  return d;
}

std::mutex g_mu;
std::map<std::pair<int, std::string>, CUfunction> g_cache;  // (device, source) -> kernel

// ------------------------------------------------------------------ codegen
std::string lit(long long v) {
  if (v == LLONG_MIN) return "HQ_LL_MIN";
  return std::to_string(v) + "LL";
}
const char* ctype(int w) { return w == 1 ? "signed char" : (w == 4 ? "int" : "long long"); }

struct Gen {
  const KPlan& kp;
  std::ostringstream o;
  std::set<int> loaded;        // registers materialised as variables
  std::map<int, std::string> vtype;  // C type of each materialised register
  std::set<int> dead;          // materialised before the compaction point, not carried over
  std::map<int, std::pair<long long, long long>> known;  // value range of probe payloads (count pass)
  std::map<int, int> stage_k;  // table column -> stage column index
  std::set<int> vec_loaded;    // stage columns read with ONE vector load per lane (all R rows)
  std::map<int, int> lazy_k;   // lazy fact column register -> kernel column index
  explicit Gen(const KPlan& k) : kp(k) {
    // kernel columns follow the fact columns in order (hq_build_kplan)
    int k2 = 0;
    for (int c = 0; c < HQ_MAX_COLS && k2 < kp.ncols; ++c) {
      if (!kp.regs[c].width || !kp.regs[c].in_stage) continue;
      if (kp.regs[c].in_stage == 2) lazy_k[c] = k2;
      else stage_k[c] = k2;
      ++k2;
    }
  }
  std::string var(int reg) const { return reg < HQ_MAX_COLS ? "c" + std::to_string(reg) : "t" + std::to_string(reg - HQ_MAX_COLS); }
  int width(int reg) const { return kp.regs[reg].width; }
  // value of register `reg` for row slot r, as a C++ expression
  std::string val(int reg) {
    use(reg);
    auto rk = rank_of.find(reg);
    // rank -> value (a dead row's register may hold anything: the index is masked to the table)
    if (rk != rank_of.end()) return "RV_" + std::to_string(rk->second) + "[(u32)" + var(reg) + "[r] & 255u]";
    return var(reg) + "[r]";
  }
  // payload registers holding the payload's rank in its build's value set (rank-coded
  // byte maps, hq_build_compact): register -> probe index (RV_<i> maps rank -> value)
  std::map<int, int> rank_of;
  std::set<int> rank_probe;  // rank-coded probes whose payload is decoded to its value at the probe
  void use(int reg) {
    if (dead.count(reg)) HQ_THROW(HQ_ERR_STATE, "jit: register used after compaction but not carried over");
    if (loaded.count(reg)) return;
    if (reg >= HQ_MAX_COLS) HQ_THROW(HQ_ERR_ARG, "jit: temporary read before definition");
    auto lz = lazy_k.find(reg);
    if (lz != lazy_k.end()) {  // lazy column: only the rows still live read it, from global memory
      const KCol& c = kp.cols[lz->second];
      sync_mask();
      dvar(ctype(c.width), var(reg));
      o << "#pragma unroll\n      for (int r = 0; r < R; ++r) " << var(reg) << "[r] = ((mask >> r) & 1u) ? __ldg((const "
        << ctype(c.width) << "*)p.col[" << lz->second << "] + (tb_ + row0 + r)) : (" << ctype(c.width) << ")0;\n";
      loaded.insert(reg);
      vtype[reg] = ctype(c.width);
      return;
    }
    const KCol& c = kp.cols[stage_k.at(reg)];
    // a lane's R rows are consecutive (row0 .. row0 + R - 1): one vector load
    // when they span 8 or 16 bytes (stage columns are 16-B aligned)
    const int vb = compacted_R ? 0 : (int)c.width * kp.R;
    const char* vt = vb == 16 ? (c.width == 4 ? "int4" : "longlong2") : (vb == 8 ? (c.width == 4 ? "int2" : "long long") : nullptr);
    dvar(ctype(c.width), var(reg));
    if (vt && c.width >= 4) {
      vec_loaded.insert(reg);
      o << "      { const " << vt << " q_ = *(const " << vt << "*)((const " << ctype(c.width) << "*)(st + " << c.soff << "u) + row0);";
      if (vb == 8 && c.width == 8) o << " " << var(reg) << "[0] = q_; }\n";
      else if (vb == 8) o << " " << var(reg) << "[0] = q_.x; " << var(reg) << "[1] = q_.y; }\n";
      else if (c.width == 8) o << " " << var(reg) << "[0] = q_.x; " << var(reg) << "[1] = q_.y; }\n";
      else o << " " << var(reg) << "[0] = q_.x; " << var(reg) << "[1] = q_.y; " << var(reg) << "[2] = q_.z; " << var(reg) << "[3] = q_.w; }\n";
    } else {
      o << "      { const " << ctype(c.width) << "* b_ = (const " << ctype(c.width) << "*)(st + " << c.soff
        << "u) + row0;\n#pragma unroll\n        for (int r = 0; r < R; ++r) " << var(reg) << "[r] = b_[r]; }\n";
    }
    loaded.insert(reg);
    vtype[reg] = ctype(c.width);
  }
  // skip the rest of the operator block when no row of the warp is live; the
  // block stays structured (nested ifs, closed in generate()) so that the
  // compiler reconverges the warp at its end -- with break-style exits a warp
  // could stay split for the rest of the kernel and run at half speed
  // software pipelining (generate(): two tiles per warp in flight): the arrays the
  // first phase of a tile defines are declared once at function scope (`decl`) and
  // renamed per tile parity; otherwise declarations stay inline
  std::ostringstream* decl = nullptr;
  std::vector<std::string> hoisted;
  void dvar(const std::string& ty, const std::string& name, bool zero = false) {
    if (decl) {
      *decl << "  " << ty << " " << name << "[R];\n";
      hoisted.push_back(name);
      if (zero) o << "#pragma unroll\n      for (int r = 0; r < R; ++r) " << name << "[r] = 0;\n";
    } else {
      o << "      " << ty << " " << name << (zero ? "[R] = {};\n" : "[R];\n");
    }
  }
  int open = 0;
  void early_exit() {
    sync_mask();  // mask must be right on the path that skips the block
    o << "      if (__any_sync(HQ_FULL, mask)) {\n";
    ++open;
  }
  // Row liveness inside the operator section: one bool per row slot (al_[r], kept in
  // predicate registers) for filters and direct probes, and the R-bit `mask` the sinks,
  // votes and linear probes use; whichever was written last is synced on demand.
  enum { LIVE_BOTH = 0, LIVE_AL = 1, LIVE_MASK = 2 };
  int live = LIVE_MASK;
  bool al_declared = false;
  void begin_al() {
    if (!al_declared) {
      dvar("bool", "al_");
      al_declared = true;
      live = LIVE_MASK;
    }
    sync_al();
  }
  void sync_al() {
    if (live != LIVE_MASK) return;
    o << "#pragma unroll\n      for (int r = 0; r < R; ++r) al_[r] = (mask >> r) & 1u;\n";
    live = LIVE_BOTH;
  }
  void sync_mask() {
    if (live != LIVE_AL) return;
    o << "      mask = 0u;\n#pragma unroll\n      for (int r = 0; r < R; ++r) mask |= (u32)al_[r] << r;\n";
    live = LIVE_BOTH;
  }
  void mask_written() { live = LIVE_MASK; }

  void filter(const KPred& f, int idx) {
    std::string cond;
    if (f.kind == 0) {
      const bool narrow = width(f.reg) <= 4;
      std::string v = narrow ? "(int)" + val(f.reg) : "(long long)" + val(f.reg);
      if (narrow) {
        if (f.lo32 > f.hi32) cond = "false";
        else if (f.lo32 == f.hi32) cond = v + " == " + std::to_string(f.lo32);
        else {
          std::string a = f.lo32 == INT_MIN ? "" : v + " >= " + std::to_string(f.lo32);
          std::string b = f.hi32 == INT_MAX ? "" : v + " <= " + std::to_string(f.hi32);
          cond = a.empty() ? (b.empty() ? "true" : b) : (b.empty() ? a : a + " && " + b);
        }
      } else {
        if (f.lo > f.hi) cond = "false";
        else {
          std::string a = f.lo == LLONG_MIN ? "" : v + " >= " + lit(f.lo);
          std::string b = f.hi == LLONG_MAX ? "" : v + " <= " + lit(f.hi);
          cond = a.empty() ? (b.empty() ? "true" : b) : (b.empty() ? a : a + " && " + b);
        }
      }
      if (f.neg) cond = "!(" + cond + ")";
    } else {
      std::string v = "(unsigned long long)(long long)" + val(f.reg);
      const std::string bm = "BM_" + std::to_string(idx);
      cond = "(" + v + " < 256ull && ((" + bm + "[" + v + " >> 6] >> (" + v + " & 63ull)) & 1ull))";
      bitmaps << "static constexpr __device__ u64 " << bm << "[4] = {" << f.bm[0] << "ull, " << f.bm[1] << "ull, "
              << f.bm[2] << "ull, " << f.bm[3] << "ull};\n";
    }
    sync_al();
    o << "#pragma unroll\n      for (int r = 0; r < R; ++r) al_[r] = al_[r] && (" << cond << ");\n";
    live = LIVE_AL;
  }

  // ---- probes.  A direct-mapped probe is three steps: address (key - min,
  // range check), load (staged compact table in shared memory, compact table in
  // global memory, or the slot array), resolve (hit test, payload, mask).
  // Global loads of adjacent probes are issued together (one L2 round trip for
  // the batch instead of one per probe), see generate().
  enum { AK_SMEM = 1, AK_GCOMPACT = 2, AK_DIRECT = 3, AK_LINEAR = 4 };
  static int access(const KProbe& pr) {
    if (!pr.direct) return AK_LINEAR;
    if (pr.ckind && pr.smem_off) return AK_SMEM;
    if (pr.ckind && pr.compact) return AK_GCOMPACT;
    return AK_DIRECT;
  }
  static std::string pv(int i, const char* what) { return "p" + std::to_string(i) + what; }
  void probe_defs(const KProbe& pr, int idx = -1) {
    const int npay = hq_probe_has_payload(pr.mode) ? pr.npay : 0;
    const bool outer = pr.mode == HQ_PROBE_OUTER;  // a miss leaves 0
    if (npay > 0 && idx >= 0 && access(pr) != AK_DIRECT && access(pr) != AK_LINEAR && pr.ckind == 2 && pr.crank) {
      // a rank-coded byte map: the register keeps the rank (an OUTER probe's 0 default
      // is a value, so there the byte is mapped back at the probe instead)
      if (!outer) rank_of[pr.dst[0]] = idx;
      else rank_probe.insert(idx);
      bitmaps << "static constexpr __device__ int RV_" << idx << "[256] = {";
      int n = 0;
      for (int d = 0; d <= pr.pay_max - pr.pay_min; ++d) {
        const uint32_t v = (uint32_t)(pr.pay_min + d) & 255u;
        if ((pr.pay_set[v >> 6] >> (v & 63)) & 1ull) bitmaps << (n++ ? ", " : "") << (pr.pay_min + d);
      }
      bitmaps << "};\n";
    }
    for (int k = 0; k < npay; ++k) {
      dvar("int", var(pr.dst[k]), outer);
      if (k == 0 && pr.pay_min <= pr.pay_max)
        known[pr.dst[0]] = {outer ? std::min(pr.pay_min, 0) : pr.pay_min, outer ? std::max(pr.pay_max, 0) : pr.pay_max};
      loaded.insert(pr.dst[k]);
      vtype[pr.dst[k]] = "int";
    }
  }
  static const char* mask_after(const KProbe& pr) {
    if (pr.mode == HQ_PROBE_ANTI) return "mask & ~found_";
    if (pr.mode == HQ_PROBE_OUTER) return "mask; (void)found_";
    return "mask & found_";
  }
  void probe_addr(const KProbe& pr, int i) {
    const std::string key = val(pr.key_reg);
    const std::string D = pv(i, "d_"), M = pv(i, "m_");
    sync_al();
    dvar("u32", D);
    dvar("bool", M);
    o << "#pragma unroll\n      for (int r = 0; r < R; ++r) {";
    if (width(pr.key_reg) <= 4)  // int32 keys: (k - min) mod 2^32 < range  <=>  min <= k < min + range
      o << " const u32 d_ = (u32)(int)" << key << " - " << (uint32_t)pr.dmin << "u; const bool in_ = d_ < " << pr.mask << "u;";
    else
      o << " const long long k_ = (long long)" << key << "; const u32 d_ = (u32)(k_ - " << pr.dmin
        << "LL); const bool in_ = k_ >= " << pr.dmin << "LL && k_ < " << pr.dmin << "LL + " << pr.mask << "LL;";
    o << " " << D << "[r] = d_; " << M << "[r] = al_[r] && in_; }\n";
  }
  void probe_load(const KProbe& pr, int i) {
    const std::string D = pv(i, "d_"), M = pv(i, "m_"), V = pv(i, "v_");
    const int ak = access(pr);
    if (ak == AK_DIRECT) {
      const int W = pr.words;
      dvar("int4", V);
      o << "#pragma unroll\n      for (int r = 0; r < R; ++r) if (" << M << "[r]) ";
      if (W == 1) o << V << "[r].x = __ldg((const int*)p.ht[" << i << "] + " << D << "[r]);\n";
      else if (W == 2)
        o << "{ const int2 q_ = __ldg((const int2*)p.ht[" << i << "] + " << D << "[r]); " << V << "[r].x = q_.x; " << V
          << "[r].y = q_.y; }\n";
      else o << V << "[r] = __ldg((const int4*)p.ht[" << i << "] + " << D << "[r]);\n";
      return;
    }
    std::string idx = D + "[r]";
    if (pr.ckind == 1) idx = "(" + D + "[r] >> 5)";
    else if (pr.ckind == 3) idx = "(" + D + "[r] >> 1)";
    std::string ld;
    if (ak == AK_SMEM)
      // 32-bit shared-window addresses from a base taken once (a generic
      // pointer made ptxas re-derive the window from SR_CgaCtaId per probe)
      ld = pr.ckind == 1 ? "lds_u32(sm0_ + " + std::to_string(pr.smem_off) + "u + (" + idx + ") * 4u)"
                         : "lds_u8(sm0_ + " + std::to_string(pr.smem_off) + "u + (" + idx + "))";
    else
      ld = pr.ckind == 1 ? "__ldg((const u32*)p.ctab[" + std::to_string(i) + "] + " + idx + ")"
                         : "(u32)__ldg((const unsigned char*)p.ctab[" + std::to_string(i) + "] + " + idx + ")";
    dvar("u32", V);
    o << "#pragma unroll\n      for (int r = 0; r < R; ++r) if (" << M << "[r]) " << V << "[r] = " << ld << ";\n";
  }
  void probe_resolve(const KProbe& pr, int i) {
    const std::string D = pv(i, "d_"), M = pv(i, "m_"), V = pv(i, "v_");
    const int npay = hq_probe_has_payload(pr.mode) ? pr.npay : 0;
    o << "#pragma unroll\n      for (int r = 0; r < R; ++r) { bool f_ = false; if (" << M << "[r]) {";
    if (access(pr) == AK_DIRECT) {
      static const char* comp[3] = {"y", "z", "w"};
      o << " if (" << V << "[r].x != HQ_INT_MIN) { f_ = true;";
      for (int k = 0; k < npay; ++k) o << " " << var(pr.dst[k]) << "[r] = " << V << "[r]." << comp[k] << ";";
      o << " }";
    } else if (pr.ckind == 1) {
      o << " f_ = (" << V << "[r] >> (" << D << "[r] & 31u)) & 1u;";
    } else {
      if (pr.ckind == 3) o << " const u32 b_ = (" << V << "[r] >> ((" << D << "[r] & 1u) * 4u)) & 15u; if (b_ != 15u) {";
      else o << " const u32 b_ = " << V << "[r]; if (b_ != 0xFFu) {";
      o << " f_ = true;";
      if (npay > 0 && rank_of.count(pr.dst[0])) o << " " << var(pr.dst[0]) << "[r] = (int)b_;";  // the rank
      else if (npay > 0 && rank_probe.count(i)) o << " " << var(pr.dst[0]) << "[r] = RV_" << i << "[b_ & 255u];";
      else if (npay > 0) o << " " << var(pr.dst[0]) << "[r] = (int)b_ + (" << pr.pay_min << ");";
      o << " }";
    }
    o << " }";
    if (pr.mode == HQ_PROBE_ANTI) o << " al_[r] = al_[r] && !f_;";
    else if (pr.mode == HQ_PROBE_OUTER) o << " (void)f_;";
    else o << " al_[r] = al_[r] && f_;";  // (a batched probe's address step saw the liveness before the batch)
    o << " }\n";
    live = LIVE_AL;
  }

  // ranked sparse-key table (hq_hash::ranked): the key's bit in the range bitmap
  // (misses stop here, L2-resident); with payloads the bitmap word comes with the rank
  // directory word in one 8-B load, and a hit's payload row is at dir + popcount(bits
  // below it) -- two dependent loads; each step's loads for the lane's R rows together
  void probe_ranked(const KProbe& pr, int idx) {
    const int npay = hq_probe_has_payload(pr.mode) ? pr.npay : 0;
    probe_defs(pr);
    const std::string key = val(pr.key_reg), I = std::to_string(idx);
    const bool pairs = pr.rstride > 0;  // the table's layout (a semi-join may probe a table with payloads)
    o << "      { u32 found_ = 0u; u32 w_[R]; u32 e_[R]; bool h_[R];" << (npay > 0 ? " u32 k_[R];" : "") << "\n"
      << "#pragma unroll\n        for (int r = 0; r < R; ++r) {\n"
      << "          const long long d_ = (long long)" << key << " - (" << pr.pf_min << "LL); e_[r] = (u32)d_;\n"
      << "          h_[r] = ((mask >> r) & 1u) && d_ >= 0 && d_ < " << pr.pf_range << "LL;\n";
    if (pairs && npay > 0)
      o << "          uint2 q_ = make_uint2(0u, 0u); if (h_[r]) q_ = __ldg((const uint2*)p.pf[" << I
        << "] + (e_[r] >> 5)); w_[r] = q_.x; k_[r] = q_.y; }\n";
    else
      o << "          w_[r] = h_[r] ? __ldg(p.pf[" << I << "] + (e_[r] >> 5)" << (pairs ? " * 2u" : "") << ") : 0u; }\n";
    o << "#pragma unroll\n        for (int r = 0; r < R; ++r) { h_[r] = (w_[r] >> (e_[r] & 31u)) & 1u;"
      << " if (h_[r]) found_ |= 1u << r; }\n";
    if (npay > 0) {
      static const char* comp[4] = {"x", "y", "z", "w"};
      o << "#pragma unroll\n        for (int r = 0; r < R; ++r) if (h_[r]) {"
        << " const u32 rk_ = k_[r] + __popc(w_[r] & ((1u << (e_[r] & 31u)) - 1u));";
      if (pr.rstride == 1) {
        o << " " << var(pr.dst[0]) << "[r] = __ldg(p.rpay[" << I << "] + rk_);";
      } else {
        o << " const " << (pr.rstride == 2 ? "int2" : "int4") << " v_ = __ldg((const " << (pr.rstride == 2 ? "int2" : "int4")
          << "*)p.rpay[" << I << "] + rk_);";
        for (int k = 0; k < npay; ++k) o << " " << var(pr.dst[k]) << "[r] = v_." << comp[k] << ";";
      }
      o << " }\n";
    }
    o << "        mask = " << mask_after(pr) << "; }\n";
    mask_written();
  }

  // linear-probing table (sparse keys): optional exact key-range bitmap, then
  // 16-B group scans until the key or an empty slot
  void probe_linear(const KProbe& pr, int idx) {
    sync_mask();
    if (pr.ranked) {
      probe_ranked(pr, idx);
      return;
    }
    const int W = pr.words;
    const int npay = hq_probe_has_payload(pr.mode) ? pr.npay : 0;
    probe_defs(pr);
    const std::string key = val(pr.key_reg);
    // composite keys: the slot's word 1 must also equal the second key (TPC-H Q9)
    const bool cmp2 = pr.composite;
    const std::string key2 = cmp2 ? val(pr.key2_reg) : std::string();
    o << "      { const u32* ht_ = p.ht[" << idx << "]; u32 found_ = 0u; int kk_[R]; u32 pend_ = 0u; u32 pos_[R];"
      << (cmp2 ? " int kk2_[R];" : "") << "\n"
      << "#pragma unroll\n        for (int r = 0; r < R; ++r) {\n"
      << "          const long long k_ = (long long)" << key << "; kk_[r] = (int)k_;\n";
    if (cmp2) o << "          kk2_[r] = (int)(long long)" << key2 << ";\n";
    const int G = W == 1 ? 4 : (W == 2 ? 2 : 1);
    o << "          bool ok_ = ((mask >> r) & 1u) && k_ > (long long)HQ_INT_MIN && k_ <= (long long)HQ_INT_MAX;\n";
    if (pr.pf) {  // exact key-range bitmap first: misses mostly stop here (L2-resident)
      o << "          if (ok_) { const long long d_ = k_ - (" << pr.pf_min << "LL);\n"
        << "            ok_ = d_ >= 0 && d_ < " << pr.pf_range << "LL && ((__ldg(p.pf[" << idx
        << "] + (d_ >> 5)) >> (d_ & 31)) & 1u); }\n";
    }
    o << "          pos_[r] = ((u32)(int)k_ * 0x9E3779B1u) >> " << (32 - pr.log2cap) << "; if (ok_) pend_ |= 1u << r; }\n"
      << "        while (pend_) {\n          int4 sl_[R];\n"
      << "#pragma unroll\n          for (int r = 0; r < R; ++r) if (pend_ & (1u << r)) sl_[r] = __ldg((const int4*)ht_ + pos_[r] / "
      << G << ");\n"
      << "#pragma unroll\n          for (int r = 0; r < R; ++r) if (pend_ & (1u << r)) {\n"
      << "            int hit_ = -1; bool stop_ = false; const int first_ = (int)(pos_[r] % " << G << ");\n";
    const char* keys4[4] = {"x", "y", "z", "w"};
    for (int j = 0; j < G; ++j) {
      const char* kc = G == 4 ? keys4[j] : (G == 2 ? (j == 0 ? "x" : "z") : "x");
      const char* k2c = G == 2 ? (j == 0 ? "y" : "w") : "y";  // composite: the slot's word 1
      const std::string m2 = cmp2 ? std::string(" && sl_[r].") + k2c + " == kk2_[r]" : std::string();
      o << "            if (!stop_ && " << j << " >= first_) { if (sl_[r]." << kc << " == kk_[r]" << m2 << ") { hit_ = " << j
        << "; stop_ = true; } else if (sl_[r]." << kc << " == HQ_INT_MIN) stop_ = true; }\n";
    }
    o << "            if (hit_ >= 0) { found_ |= 1u << r; pend_ &= ~(1u << r);\n";
    if (npay > 0) {
      if (G == 2) o << "              " << var(pr.dst[0]) << "[r] = hit_ == 0 ? sl_[r].y : sl_[r].w;\n";
      else {
        static const char* comp[3] = {"y", "z", "w"};
        for (int k = 0; k < npay; ++k)
          o << "              " << var(pr.dst[k]) << "[r] = sl_[r]." << comp[k + (cmp2 ? 1 : 0)] << ";\n";
      }
    }
    o << "            } else if (stop_) pend_ &= ~(1u << r);\n"
      << "            else pos_[r] = ((pos_[r] / " << G << " + 1) * " << G << ") & " << pr.mask << "u;\n"
      << "          }\n        }\n";
    o << "        mask = " << mask_after(pr) << "; }\n";
    mask_written();
  }

  // ops [i, end): one probe batch starting at op i (see probe_addr)
  // part 0: the whole batch; 1: definitions, addresses and loads (the batch is kept);
  // 2: the kept batch's resolution (software pipelining splits a tile there)
  std::vector<int> kept_batch;
  int probe_batch(int i, int part = 0) {
    if (part == 2) {
      for (int j : kept_batch) probe_resolve(kp.probes[kp.ops[j].idx], kp.ops[j].idx);
      return kept_batch.back() + 1;
    }
    const KProbe& first = kp.probes[kp.ops[i].idx];
    const int ak = access(first);
    if (ak == AK_LINEAR) {
      early_exit();
      probe_linear(first, kp.ops[i].idx);
      return i + 1;
    }
    std::vector<int> b = {i};
    if (ak != AK_SMEM) {  // a global probe: the following independent global probes join its batch
      // (no early exit in front: the warp rarely has no live row here, and the
      // extra branch measured slower); so do following shared-memory probes, whose
      // loads then issue under the global round trip instead of after it (they cost a
      // few shared loads for rows the batch drops; HQ_JIT_NOSMEMJOIN=1: not joined)
      const bool smem_join = !getenv("HQ_JIT_NOSMEMJOIN");
      std::set<int> defs(first.dst, first.dst + (hq_probe_has_payload(first.mode) ? first.npay : 0));
      for (int j = i + 1; j < kp.nops && kp.ops[j].kind == OP_PROBE && !kp.op_skip[j]; ++j) {
        const KProbe& pr = kp.probes[kp.ops[j].idx];
        if (access(pr) == AK_LINEAR || (access(pr) == AK_SMEM && !smem_join) || defs.count(pr.key_reg)) break;
        b.push_back(j);
        for (int k = 0; k < (hq_probe_has_payload(pr.mode) ? pr.npay : 0); ++k) defs.insert(pr.dst[k]);
      }
    }
    for (int j : b) probe_defs(kp.probes[kp.ops[j].idx], kp.ops[j].idx);
    for (int j : b) probe_addr(kp.probes[kp.ops[j].idx], kp.ops[j].idx);
    for (int j : b) probe_load(kp.probes[kp.ops[j].idx], kp.ops[j].idx);
    if (part == 1) {
      kept_batch = b;
      return b.back() + 1;
    }
    for (int j : b) probe_resolve(kp.probes[kp.ops[j].idx], kp.ops[j].idx);
    return b.back() + 1;
  }

  std::string operand(const KInsn& in) {
    if (in.reg < 0) return lit(in.imm);
    return "(long long)" + val(in.reg);
  }
  void compute(const KCompute& c) {
    sync_mask();  // DIV / MOD flag faults of live rows only
    // operands first (column loads must not land inside the row loop)
    std::vector<std::string> ops;
    for (int k = 0; k < c.n; ++k) ops.push_back(operand(kp.insns[c.first + k]));
    const std::string dst = var(c.dst);
    dvar("long long", dst);
    o << "#pragma unroll\n      for (int r = 0; r < R; ++r) { long long a_ = 0;\n";
    for (int k = 0; k < c.n; ++k) {
      const KInsn& in = kp.insns[c.first + k];
      const std::string& x = ops[k];
      switch (in.opc) {
        case HQ_I_LOAD: o << "        a_ = " << x << ";\n"; break;
        case HQ_I_ADD: o << "        a_ += " << x << ";\n"; break;
        case HQ_I_SUB: o << "        a_ -= " << x << ";\n"; break;
        case HQ_I_RSUB: o << "        a_ = " << x << " - a_;\n"; break;
        case HQ_I_MUL: o << "        a_ *= " << x << ";\n"; break;
        case HQ_I_AND_EQ: case HQ_I_AND_NE: case HQ_I_AND_LT: case HQ_I_AND_LE: case HQ_I_AND_GT: case HQ_I_AND_GE: {
          static const char* cmp[6] = {"==", "!=", "<", "<=", ">", ">="};
          o << "        a_ = (a_ != 0 && " << x << " " << cmp[in.opc - HQ_I_AND_EQ] << " " << lit(in.imm) << ") ? 1 : 0;\n";
          break;
        }
        case HQ_I_AND_IN:
          o << "        { const long long v_ = " << x << "; a_ = (a_ != 0 && v_ >= 0 && v_ < 64 && ((" << (unsigned long long)in.imm
            << "ULL >> v_) & 1ull)) ? 1 : 0; }\n";
          break;
        case HQ_I_OR: o << "        a_ = (a_ != 0 || " << x << " != 0) ? 1 : 0;\n"; break;
        default:
          o << "        { const long long d_ = " << x << "; if (d_ == 0) { if ((mask >> r) & 1u) atomicOr(p.err, F_DIV_ZERO); a_ = 0; }"
            << " else a_ = a_ " << (in.opc == HQ_I_DIV ? "/" : "%") << " d_; }\n";
      }
    }
    o << "        " << dst << "[r] = a_; }\n";
    loaded.insert(c.dst);
    vtype[c.dst] = "long long";
  }
  // registers read by ops [from, nops) and by the sink
  std::set<int> uses_from(int from) const {
    std::set<int> u;
    for (int j = from; j < kp.nops; ++j) {
      const KOp& op = kp.ops[j];
      if (op.kind == OP_FILTER) u.insert(kp.preds[op.idx].reg);
      else if (op.kind == OP_PROBE) {
        u.insert(kp.probes[op.idx].key_reg);
        if (kp.probes[op.idx].composite) u.insert(kp.probes[op.idx].key2_reg);
      }
      else {
        const KCompute& c = kp.comps[op.idx];
        for (int k = 0; k < c.n; ++k)
          if (kp.insns[c.first + k].reg >= 0) u.insert(kp.insns[c.first + k].reg);
      }
    }
    for (int a = 0; a < kp.naggs; ++a)
      if (kp.agg_fn[a] != HQ_AGG_COUNT) u.insert(kp.agg_reg[a]);
    for (int i = 0; i < kp.nkeys; ++i) u.insert(kp.key_reg[i]);
    return u;
  }
  // Warp compaction of the live rows (selection vector in registers): after a
  // selective probe most of the R row slots are dead, but predicated code pays
  // for them.  The live rows of the warp's R slots move into consecutive lanes
  // (ballot prefix, k-th set bit by popc bisection), registers still needed are
  // shuffled over, and the rest of the pipeline runs in rounds of 32 rows with
  // ONE row slot (R redefined to 1 in that scope).  Columns not loaded yet are
  // read from the stage at the compacted row (row0 redefined).
  void compact(int from) {
    sync_mask();
    const int R0 = kp.R;
    std::vector<int> live;
    for (int r : uses_from(from))
      if (loaded.count(r)) live.push_back(r);
    o << "      {\n      u32 cb_[R]; int cp_[R + 1]; cp_[0] = 0;\n"
      << "#pragma unroll\n      for (int r = 0; r < R; ++r) { cb_[r] = __ballot_sync(HQ_FULL, (mask >> r) & 1u); cp_[r + 1] = cp_[r] + __popc(cb_[r]); }\n"
      << "      for (int i0_ = 0; i0_ < cp_[R]; i0_ += 32) {\n"
      << "        const int ct_ = i0_ + lane; const bool lv_ = ct_ < cp_[R];\n"
      << "        int rr_ = 0; u32 cm_ = cb_[0]; int ck_ = ct_;\n"
      << "#pragma unroll\n        for (int r = 1; r < R; ++r) if (ct_ >= cp_[r]) { rr_ = r; cm_ = cb_[r]; ck_ = ct_ - cp_[r]; }\n"
      << "        int src_ = 0;\n#pragma unroll\n        for (int s_ = 16; s_ > 0; s_ >>= 1) { const int c_ = __popc((cm_ >> src_) & ((1u << s_) - 1u)); if (ck_ >= c_) { ck_ -= c_; src_ += s_; } }\n"
      << "        if (!lv_) { src_ = lane; rr_ = 0; }\n";
    for (int r : live) {
      const std::string& t = vtype.at(r);
      o << "        " << t << " x_" << var(r) << " = 0;\n#pragma unroll\n        for (int r = 0; r < R; ++r) { const " << t
        << " y_ = __shfl_sync(HQ_FULL, " << var(r) << "[r], src_); if (r == rr_) x_" << var(r) << " = y_; }\n";
    }
    o << "        {\n#undef R\n#define R 1\n"
      << "        u32 mask = lv_ ? 1u : 0u;\n"
      << "        const int row0 = warp * 32 * " << R0 << " + src_ * " << R0 << " + rr_;\n";
    for (int r : live) o << "        " << vtype.at(r) << " " << var(r) << "[R] = {x_" << var(r) << "};\n";
    std::set<int> keep(live.begin(), live.end());
    for (int r : loaded)
      if (!keep.count(r)) dead.insert(r);
    open += 3;
    compacted_R = R0;
    mask_written();
  }
  int compacted_R = 0;  // original R when compact() ran (restored after the scope)
  std::ostringstream bitmaps;
};

// LCOL[a]: the shared-table word of aggregate a (0 = the count word, for COUNT);
// LFN[c]: the aggregate function of word c (for its identity)
std::string lcol_tables(const KPlan& kp) {
  std::ostringstream s;
  s << "static constexpr __device__ int LCOL[" << (kp.naggs > 0 ? kp.naggs : 1) << "] = {";
  for (int a = 0; a < (kp.naggs > 0 ? kp.naggs : 1); ++a) s << (a ? ", " : "") << (a < kp.naggs ? (int)kp.lcol[a] : 0);
  s << "};\nstatic constexpr __device__ int LFN[" << (kp.lvwords > 0 ? kp.lvwords : 1) << "] = {";
  std::vector<int> fn(kp.lvwords > 0 ? kp.lvwords : 1, HQ_AGG_COUNT);
  for (int a = 0; a < kp.naggs; ++a)
    if (kp.lcol[a]) fn[kp.lcol[a]] = kp.agg_fn[a];
  for (size_t c = 0; c < fn.size(); ++c) s << (c ? ", " : "") << fn[c];
  s << "};\n";
  return s.str();
}

// staged A3: copy a tile's rows [0, n) from its staging buffer to base + i (all
// consumer threads, coalesced per column); positions past the capacity set F_CAPACITY
std::string a3_flush_fn(const KPlan& kp) {
  if (!kp.a3stage) return "";
  std::ostringstream s;
  if (kp.a3stage == 2) {
    // warp-workgroup A3: the warp's n buffered rows get n global positions with one
    // atomicAdd and are copied out, coalesced per column (positions past the capacity
    // set F_CAPACITY; the counter still counts them, for the re-run)
    s << "#define A3WBYTES " << kp.a3_buf << "u\n#define A3WROWS " << kp.a3_rows << "\n"
      << "__device__ __forceinline__ void a3w_flush(const JParams& p, const char* wb, int n) {\n"
      << "  unsigned long long g = 0;\n"
      << "  if ((threadIdx.x & 31) == 0) g = atomicAdd(p.counter, (unsigned long long)n);\n"
      << "  g = __shfl_sync(0xffffffffu, g, 0);\n"
      << "  for (int i = threadIdx.x & 31; i < n; i += 32) {\n"
      << "    const long long pos = (long long)(g + i);\n"
      << "    if (pos >= p.capacity) { atomicOr(p.err, 1); continue; }\n";
    for (int j = 0; j < kp.nout; ++j) {
      const char* ty = kp.out_width[j] == 1 ? "signed char" : (kp.out_width[j] == 4 ? "int" : "long long");
      s << "    ((" << ty << "*)p.out[" << j << "])[pos] = ((const " << ty << "*)(wb + " << kp.a3_col[j] << "u))[i];\n";
    }
    s << "  }\n  __syncwarp();\n}\n";
    return s.str();
  }
  s << "#define A3BUF " << kp.a3_buf << "u\n"
    << "__device__ __forceinline__ void a3_flush(const JParams& p, long long base, int n, const char* sb) {\n"
    << "  for (int i = threadIdx.x; i < n; i += NW * 32) {\n"
    << "    const long long pos = base + i;\n"
    << "    if (pos >= p.capacity) { atomicOr(p.err, 1); continue; }\n";
  for (int j = 0; j < kp.nout; ++j) {
    const char* ty = kp.out_width[j] == 1 ? "signed char" : (kp.out_width[j] == 4 ? "int" : "long long");
    s << "    ((" << ty << "*)p.out[" << j << "])[pos] = ((const " << ty << "*)(sb + " << kp.a3_col[j] << "u))[i];\n";
  }
  s << "  }\n}\n";
  return s.str();
}

std::string fn_list(const uint8_t* fns, int n) {
  std::ostringstream s;
  s << "{";
  for (int i = 0; i < (n > 0 ? n : 1); ++i) s << (i ? ", " : "") << (i < n ? (int)fns[i] : 0);
  s << "}";
  return s.str();
}

// Resolution:WE tile code (App C, "Work-Efficient Reduction", Fig 24,
// P:1989-2029; Table 4 A3/B3/C3): every consumer thread takes part (NT = NW * 32 is a
// power of two for WE plans, hq_plan.cu), one consumer barrier per tree level.
//  B3-WE: up-sweep of the threads' tile partials -> one global atomic per tile;
//  A3-WE: Blelloch exclusive scan of the threads' row counts -> one atomicAdd per tile,
//         rows written at base + scan + their rank among the thread's rows;
//  C3-WE: bitonic sort of the tile's (key, count, values) by key, a work-efficient
//         segmented scan with (f1,v1)+(f2,v2) = (f1|f2, f2 ? v2 : v1+v2), and every
//         segment's last entry updates the global group table (atomic hash reduce).
void gen_we_tile(std::ostringstream& o, const KPlan& kp, int sk) {
  const int NT = kp.nw * 32;
  if (NT & (NT - 1)) HQ_THROW(HQ_ERR_STATE, "jit: Resolution:WE needs a power-of-two thread count");
  const std::string nt = std::to_string(NT);
  o << "    { const int tid_ = threadIdx.x;\n";
  if (sk == 0) {
    o << "      i64* wr_ = (i64*)(smem + OFF_AGG);  // [1 + NAGGS][NT]: count, aggregates\n"
      << "      wr_[tid_] = (i64)wc_;\n";
    for (int a = 0; a < kp.naggs; ++a) o << "      wr_[" << (1 + a) * NT << " + tid_] = wa_[" << a << "];\n";
    o << "      for (int d_ = 1; d_ < " << nt << "; d_ <<= 1) {\n        consumer_bar();\n"
      << "        const int i_ = (tid_ + 1) * 2 * d_ - 1;\n        if (i_ < " << nt << ") { wr_[i_] += wr_[i_ - d_];";
    for (int a = 0; a < kp.naggs; ++a)
      o << " wr_[" << (1 + a) * NT << " + i_] = agg_combine(AGG_FN[" << a << "], wr_[" << (1 + a) * NT << " + i_ - d_], wr_["
        << (1 + a) * NT << " + i_]);";
    o << " }\n      }\n      consumer_bar();\n"
      << "      if (tid_ == 0 && wr_[" << NT - 1 << "] != 0) { const u64 cnt_ = (u64)wr_[" << NT - 1 << "]; g_add64(p.gtab, (i64)cnt_);";
    for (int a = 0; a < kp.naggs; ++a)
      o << " g_agg(AGG_FN[" << a << "], p.gtab + " << 1 + a << ", wr_[" << (1 + a) * NT + NT - 1 << "], cnt_);";
    o << " }\n      consumer_bar();  // the next tile rewrites the tree\n    }\n";
    return;
  }
  if (sk == 2) {
    o << "      int* ws_ = (int*)(smem + OFF_AGG);\n      const u32 msk_ = mask;\n      ws_[tid_] = __popc(msk_);\n"
      << "      for (int d_ = 1; d_ < " << nt << "; d_ <<= 1) { consumer_bar(); const int i_ = (tid_ + 1) * 2 * d_ - 1;"
      << " if (i_ < " << nt << ") ws_[i_] += ws_[i_ - d_]; }\n      consumer_bar();\n"
      << "      if (tid_ == 0) { const int tot_ = ws_[" << NT - 1 << "]; s_base[0] = tot_ > 0 ? atomicAdd(p.counter, (u64)tot_) : 0ull;"
      << " ws_[" << NT - 1 << "] = 0; }\n"
      << "      for (int d_ = " << NT / 2 << "; d_ >= 1; d_ >>= 1) { consumer_bar(); const int i_ = (tid_ + 1) * 2 * d_ - 1;"
      << " if (i_ < " << nt << ") { const int t_ = ws_[i_ - d_]; ws_[i_ - d_] = ws_[i_]; ws_[i_] += t_; } }\n"
      << "      consumer_bar();\n      const u64 base_ = s_base[0] + (u64)ws_[tid_];\n"
      << "#pragma unroll\n      for (int r = 0; r < R; ++r) if ((msk_ >> r) & 1u) { const u64 pos_ = base_ + __popc(msk_ & ((1u << r) - 1u));\n"
      << "        if ((long long)pos_ < p.capacity) {\n";
    for (int j = 0; j < kp.nout; ++j)
      o << "          ((" << ctype(kp.out_width[j]) << "*)p.out[" << j << "])[pos_] = (" << ctype(kp.out_width[j]) << ")ov" << j << "[r];\n";
    o << "        } else atomicOr(p.err, F_CAPACITY); }\n      consumer_bar();  // s_base / the scan are rewritten by the next tile\n    }\n";
    return;
  }
  // C3-WE over N = NT * R entries
  const int N = NT * kp.R;
  const std::string n = std::to_string(N);
  const int na = kp.naggs;
  o << "      u64* wk_s = (u64*)(smem + OFF_AGG); i64* wn_ = (i64*)(wk_s + " << N << "); i64* wv_s = wn_ + " << N
    << "; int* wf_ = (int*)(wv_s + " << (size_t)N * (na > 0 ? na : 1) << ");\n"
    << "#pragma unroll\n      for (int r = 0; r < R; ++r) { const int e_ = tid_ * R + r; const bool l_ = (wm_ >> r) & 1u;"
    << " wk_s[e_] = l_ ? wk_[r] : HQ_EMPTY_KEY; wn_[e_] = l_ ? 1 : 0;";
  for (int a = 0; a < na; ++a) o << " wv_s[" << a * N << " + e_] = l_ ? wv_[" << a << "][r] : agg_identity(AGG_FN[" << a << "]);";
  o << " }\n";
  // bitonic sort by key (empty keys = ~0 sort last)
  o << "      for (int k_ = 2; k_ <= " << n << "; k_ <<= 1)\n        for (int j_ = k_ >> 1; j_ > 0; j_ >>= 1) {\n          consumer_bar();\n"
    << "          for (int e_ = tid_; e_ < " << n << "; e_ += " << nt << ") { const int q_ = e_ ^ j_; if (q_ > e_) {\n"
    << "            const u64 a_ = wk_s[e_], b_ = wk_s[q_];\n"
    << "            if ((a_ > b_) == ((e_ & k_) == 0)) { wk_s[e_] = b_; wk_s[q_] = a_; { const i64 x_ = wn_[e_]; wn_[e_] = wn_[q_]; wn_[q_] = x_; }";
  for (int a = 0; a < na; ++a)
    o << " { const i64 x_ = wv_s[" << a * N << " + e_]; wv_s[" << a * N << " + e_] = wv_s[" << a * N << " + q_]; wv_s[" << a * N
      << " + q_] = x_; }";
  o << " } } }\n        }\n      consumer_bar();\n";
  // head flags, then the segmented up-sweep: node i = op(left, node)
  o << "      for (int e_ = tid_; e_ < " << n << "; e_ += " << nt << ") wf_[e_] = (e_ == 0 || wk_s[e_] != wk_s[e_ - 1]) ? 1 : 0;\n"
    << "      for (int d_ = 1; d_ < " << n << "; d_ <<= 1) {\n        consumer_bar();\n"
    << "        for (int t_ = tid_; t_ < " << n << " / (2 * d_); t_ += " << nt << ") { const int i_ = (t_ + 1) * 2 * d_ - 1, l_ = i_ - d_;\n"
    << "          if (!wf_[i_]) { wn_[i_] += wn_[l_];";
  for (int a = 0; a < na; ++a)
    o << " wv_s[" << a * N << " + i_] = agg_combine(AGG_FN[" << a << "], wv_s[" << a * N << " + l_], wv_s[" << a * N << " + i_]);";
  o << " }\n          wf_[i_] |= wf_[l_]; }\n      }\n      consumer_bar();\n"
    // the root is the last segment's total; then it becomes the identity for the down-sweep
    << "      if (tid_ == 0) { s_red[0] = wn_[" << N - 1 << "];";
  for (int a = 0; a < na; ++a) o << " s_red[" << 1 + a << "] = wv_s[" << a * N + N - 1 << "];";
  o << " wf_[" << N - 1 << "] = 0; wn_[" << N - 1 << "] = 0;";
  for (int a = 0; a < na; ++a) o << " wv_s[" << a * N + N - 1 << "] = agg_identity(AGG_FN[" << a << "]);";
  o << " }\n"
    // down-sweep: left <- parent prefix; right <- op(parent prefix, left total)
    << "      for (int d_ = " << N / 2 << "; d_ >= 1; d_ >>= 1) {\n        consumer_bar();\n"
    << "        for (int t_ = tid_; t_ < " << n << " / (2 * d_); t_ += " << nt << ") { const int i_ = (t_ + 1) * 2 * d_ - 1, l_ = i_ - d_;\n"
    << "          const int tf_ = wf_[l_]; const i64 tn_ = wn_[l_]; wf_[l_] = wf_[i_]; wn_[l_] = wn_[i_];";
  for (int a = 0; a < na; ++a)
    o << " const i64 tv" << a << "_ = wv_s[" << a * N << " + l_]; wv_s[" << a * N << " + l_] = wv_s[" << a * N << " + i_];";
  o << "\n          wf_[i_] |= tf_;\n          if (tf_) { wn_[i_] = tn_;";
  for (int a = 0; a < na; ++a) o << " wv_s[" << a * N << " + i_] = tv" << a << "_;";
  o << " } else { wn_[i_] += tn_;";
  for (int a = 0; a < na; ++a)
    o << " wv_s[" << a * N << " + i_] = agg_combine(AGG_FN[" << a << "], wv_s[" << a * N << " + i_], tv" << a << "_);";
  o << " } }\n      }\n      consumer_bar();\n"
    // every segment's last entry: its total is the exclusive prefix of the next entry
    << "      for (int e_ = tid_; e_ < " << n << "; e_ += " << nt << ") { const u64 key_ = wk_s[e_];\n"
    << "        if (key_ == HQ_EMPTY_KEY || (e_ + 1 < " << n << " && wk_s[e_ + 1] == key_)) continue;\n"
    << "        const bool last_ = e_ + 1 == " << n << "; i64 v_[NAGGS > 0 ? NAGGS : 1];\n"
    << "        const u64 cnt_ = (u64)(last_ ? s_red[0] : wn_[e_ + 1]);\n";
  for (int a = 0; a < na; ++a) o << "        v_[" << a << "] = last_ ? s_red[" << 1 + a << "] : wv_s[" << a * N << " + e_ + 1];\n";
  o << "        group_update(p, sagg, sl0_, key_, false, cnt_, v_); }\n      consumer_bar();  // the next tile rewrites the sort buffers\n    }\n";
}

std::string generate(const KPlan& kp) {
  Gen g(kp);
  // HQ_JIT_PROF=1 (debug): per-CTA globaltimer start/end and barrier-wait cycles
  const bool prof = getenv("HQ_JIT_PROF") != nullptr;
  int wait_ns = 128;  // consumer back-off between barrier polls (HQ_JIT_WAIT_NS: tuning)
  if (const char* e = getenv("HQ_JIT_WAIT_NS")) wait_ns = atoi(e);
  std::ostringstream& o = g.o;
  const bool c2 = kp.resolution == HQ_RES_ATOMIC;
  // Resolution:WE (App C, Fig 24): per tile, a work-efficient
  // (Blelloch) tree in shared memory with one consumer barrier per level produces one
  // pre-aggregate / write offset per workgroup (the CTA) for global propagation
  const bool we = kp.resolution == HQ_RES_WE;
  // warp update queues (kp.gq_cap) in front of a global hash group table
  const bool gq = kp.gq_cap > 0 && !c2 && !we && !kp.mp_pass && kp.sink == HQ_SINK_AGG && kp.nkeys > 0 &&
                  kp.smode == SM_NONE && kp.gmode == GM_HASH && kp.R <= 2 && !getenv("HQ_JIT_COMPACT");
  const int sk = kp.sink == HQ_SINK_MATERIALISE ? 2 : (kp.nkeys == 0 ? 0 : 1);
  const int mp = kp.mp_pass;  // multi-pass: 1 = count kernel, 2 = write kernel (hq_multipass.cu)
  // the sink's per-tile code (aggregation into registers / shared tables, or the
  // materialised values handed to the block scan), emitted where the ops end
  auto sink_tile = [&]() {
  if (sk != 2) g.early_exit();  // the sinks below only touch live rows
  // ------------------------------------------------------------ sink (tile)
  auto aggval = [&](int a) -> std::string {
    if (kp.agg_fn[a] == HQ_AGG_COUNT) return "1LL";
    return "(i64)" + g.val(kp.agg_reg[a]);
  };
  if (sk == 0) {
    std::vector<std::string> vv;
    for (int a = 0; a < kp.naggs; ++a) vv.push_back(aggval(a));
    if (we) {  // B3-WE: the thread's partial over its R rows of this tile
      o << "      wc_ = __popc(mask);\n#pragma unroll\n      for (int r = 0; r < R; ++r) if ((mask >> r) & 1u) {\n";
      for (int a = 0; a < kp.naggs; ++a)
        if (kp.agg_fn[a] != HQ_AGG_COUNT) o << "        wa_[" << a << "] = agg_combine(AGG_FN[" << a << "], wa_[" << a << "], " << vv[a] << ");\n";
      o << "      }\n";
    } else if (c2) {  // B2: per-row global atomic reduce
      o << "#pragma unroll\n      for (int r = 0; r < R; ++r) if ((mask >> r) & 1u) { g_add64(p.gtab, 1);\n";
      for (int a = 0; a < kp.naggs; ++a) o << "        g_agg(AGG_FN[" << a << "], p.gtab + " << 1 + a << ", " << vv[a] << ", 1);\n";
      o << "      }\n";
    } else {
      o << "      scount_ += __popc(mask);\n#pragma unroll\n      for (int r = 0; r < R; ++r) if ((mask >> r) & 1u) {\n";
      for (int a = 0; a < kp.naggs; ++a)
        if (kp.agg_fn[a] != HQ_AGG_COUNT) o << "        sacc" << a << " = agg_combine(AGG_FN[" << a << "], sacc" << a << ", " << vv[a] << ");\n";
      o << "      }\n";
    }
  } else if (sk == 1) {
    // local dense / lane-private tables index < 2^32 groups: when no key needs a
    // domain check the index is computed in 32-bit arithmetic
    bool all_in = true;
    std::vector<bool> indom(kp.nkeys);
    for (int i = 0; i < kp.nkeys; ++i) {
      auto kr = g.known.find(kp.key_reg[i]);
      indom[i] = kr != g.known.end() && kr->second.first >= kp.key_min[i] &&
                 kr->second.second < kp.key_min[i] + kp.key_card[i];
      all_in = all_in && indom[i];
    }
    const bool k32 = all_in && (kp.smode == SM_DENSE || kp.smode == SM_LANE);
    o << "      u64 gk_[R]; bool bad_ = false;\n";
    if (k32) o << "      u32 gk32_[R];\n#pragma unroll\n      for (int r = 0; r < R; ++r) gk32_[r] = 0u;\n";
    else o << "#pragma unroll\n      for (int r = 0; r < R; ++r) gk_[r] = 0;\n";
    for (int i = 0; i < kp.nkeys; ++i) {
      const std::string v = g.val(kp.key_reg[i]);
      // the shared table may index a narrowed domain (kp.local_keys): only keys
      // whose payload range is known are narrowed, and those need no check
      const int64_t kmin = kp.local_keys ? kp.lkey_min[i] : kp.key_min[i];
      const int64_t kstr = kp.local_keys ? kp.lkey_stride[i] : kp.key_stride[i];
      const uint64_t* ls = kp.lkey_set[i];
      const bool ranked = kp.local_keys && (ls[0] | ls[1] | ls[2] | ls[3]);
      std::string dexpr;  // the key's offset (or rank) in the (narrowed) domain
      const std::string off32 = "((u32)(long long)" + v + " - " + std::to_string((uint32_t)kmin) + "u)";
      auto rkr = g.rank_of.find(kp.key_reg[i]);
      if (ranked && rkr != g.rank_of.end() && kp.probes[rkr->second].pay_min == kmin) {
        dexpr = "(u32)" + g.var(kp.key_reg[i]) + "[r]";  // the byte map holds the rank already
      } else if (ranked) {  // index by the rank of the value among the build side's distinct payloads
        int top = 0;
        for (int d = 0; d < 256; ++d)
          if ((ls[d >> 6] >> (d & 63)) & 1ull) top = d + 1;
        char buf[64];
        if (top <= 32) {  // rank = popcount of the set below the value
          snprintf(buf, sizeof buf, "0x%08xu", (unsigned)ls[0]);
          dexpr = "(u32)__popc(" + std::string(buf) + " & ((1u << (" + off32 + " & 31u)) - 1u))";
        } else if (top <= 64) {
          snprintf(buf, sizeof buf, "0x%016llxull", (unsigned long long)ls[0]);
          dexpr = "(u32)__popcll(" + std::string(buf) + " & ((1ull << (" + off32 + " & 63u)) - 1ull))";
        } else {
          const std::string rk = "RK_" + std::to_string(i);
          g.bitmaps << "static constexpr __device__ unsigned char " << rk << "[] = {";
          int64_t n = 0;
          for (int64_t d = 0; d < 256; ++d) {
            const bool on = (ls[d >> 6] >> (d & 63)) & 1ull;
            g.bitmaps << (d ? ", " : "") << (on ? n : 255);
            n += on;
          }
          g.bitmaps << "};\n";
          dexpr = "(((mask >> r) & 1u) ? (u32)" + rk + "[" + off32 + " & 255u] : 0u)";
        }
      }
      if (k32) {
        o << "#pragma unroll\n      for (int r = 0; r < R; ++r) gk32_[r] += " << (ranked ? dexpr : off32) << " * "
          << (uint32_t)kstr << "u;\n";
        continue;
      }
      if (ranked)
        o << "#pragma unroll\n      for (int r = 0; r < R; ++r) { const long long d_ = (long long)" << dexpr << ";";
      else
        o << "#pragma unroll\n      for (int r = 0; r < R; ++r) { const long long d_ = (long long)" << v << " - " << lit(kmin) << ";";
      if (!indom[i])  // payload ranges known from the build's count pass need no domain check
        o << " if (d_ < 0 || d_ >= " << lit(kp.key_card[i]) << ") { if ((mask >> r) & 1u) bad_ = true; mask &= ~(1u << r); }";
      o << " gk_[r] += (u64)d_ * " << kstr << "ull; }\n";
    }
    if (k32) o << "#pragma unroll\n      for (int r = 0; r < R; ++r) gk_[r] = gk32_[r];\n";
    o << "      if (bad_) atomicOr(p.err, F_KEY_DOMAIN);\n";
    if (we) {  // C3-WE: hand the live rows' keys and values to the tile's sort below
      std::vector<std::string> vv;
      for (int a = 0; a < kp.naggs; ++a) vv.push_back(aggval(a));
      o << "      wm_ = mask;\n#pragma unroll\n      for (int r = 0; r < R; ++r) { wk_[r] = gk_[r];";
      for (int a = 0; a < kp.naggs; ++a) o << " wv_[" << a << "][r] = " << vv[a] << ";";
      o << " }\n";
    } else if (kp.smode == SM_LANE) {
      std::vector<std::string> av(kp.nacc);
      for (int a = 1; a < kp.nacc; ++a) av[a] = "(i64)" + g.val(kp.acc_reg[a]);
      o << "      i64* lt_ = (i64*)sagg + threadIdx.x;\n#pragma unroll\n      for (int r = 0; r < R; ++r) if ((mask >> r) & 1u) {\n"
        << "        i64* e_ = lt_ + gk_[r] * (u64)(NACC * NW * 32);\n        e_[0] += 1;\n";
      for (int a = 1; a < kp.nacc; ++a)
        o << "        e_[" << a << " * NW * 32] = agg_combine(ACC_FN[" << a << "], e_[" << a << " * NW * 32], " << av[a] << ");\n";
      o << "      }\n";
    } else {
      std::vector<std::string> vv;
      for (int a = 0; a < kp.naggs; ++a) vv.push_back(aggval(a));
      o << "      i64 va_[NAGGS > 0 ? NAGGS : 1][R];\n#pragma unroll\n      for (int r = 0; r < R; ++r) {";
      for (int a = 0; a < kp.naggs; ++a) o << " va_[" << a << "][r] = " << vv[a] << ";";
      o << " }\n";
      if (gq) {
        // warp update queue (kp.gq_cap): a lane's consecutive rows of one group are folded
        // (the lines of an order), the live rows are appended at the warp's ballot prefix;
        // a queue that cannot take them is applied first, one update per lane (gq_flush),
        // and a tile with more live rows than the queue holds updates directly
        o << "      u64 cn_[R];\n#pragma unroll\n      for (int r = 0; r < R; ++r) cn_[r] = 1ull;\n"
          << "#pragma unroll\n      for (int r = 1; r < R; ++r) if (((mask >> r) & 1u) && ((mask >> (r - 1)) & 1u) && gk_[r] == gk_[r - 1]) {\n"
          << "#pragma unroll\n        for (int a = 0; a < NAGGS; ++a) va_[a][r] = agg_combine(AGG_FN[a], va_[a][r], va_[a][r - 1]);\n"
          << "        cn_[r] += cn_[r - 1]; mask &= ~(1u << (r - 1)); }\n"
          << "      { const int mine_ = __popc(mask); int lin_ = mine_;\n"
          << "#pragma unroll\n        for (int o_ = 1; o_ < 32; o_ <<= 1) { const int t_ = __shfl_up_sync(HQ_FULL, lin_, o_); if (lane >= o_) lin_ += t_; }\n"
          << "        const int wtot_ = __shfl_sync(HQ_FULL, lin_, 31);\n"
          << "        if (gqn_ + wtot_ > GQ_CAP) { gq_flush(p, sagg, sl0_, gq_, gqn_); gqn_ = 0; }\n"
          << "        if (wtot_ > GQ_CAP) {\n"
          << "#pragma unroll\n          for (int r = 0; r < R; ++r) if ((mask >> r) & 1u) { i64 v_[NAGGS > 0 ? NAGGS : 1];\n"
          << "#pragma unroll\n            for (int a = 0; a < NAGGS; ++a) v_[a] = va_[a][r];\n"
          << "            group_update(p, sagg, sl0_, gk_[r], false, cn_[r], v_); }\n"
          << "        } else {\n"
          << "          int pos_ = gqn_ + lin_ - mine_;\n"
          << "#pragma unroll\n          for (int r = 0; r < R; ++r) if ((mask >> r) & 1u) { gq_[pos_] = gk_[r]; gq_[GQ_CAP + pos_] = cn_[r];\n"
          << "#pragma unroll\n            for (int a = 0; a < NAGGS; ++a) gq_[(2 + a) * GQ_CAP + pos_] = (u64)va_[a][r];\n"
          << "            ++pos_; }\n"
          << "          gqn_ += wtot_;\n        }\n      }\n";
      } else {
      const char* ce = getenv("HQ_JIT_COMPACT");  // A/B: compaction of R >= 4 row slots
      const bool wcompact = ce ? ce[0] == '1' : kp.R >= 4;
      if (wcompact) {
        // warp compaction: the warp's live rows (over all R row slots) move into
        // consecutive lanes (ballot prefix, k-th set bit by popc bisection,
        // shuffles), so table updates run as rounds of 32 rows instead of R slots
        o << "      u32 bm_[R]; int pre_[R + 1]; pre_[0] = 0;\n"
          << "#pragma unroll\n      for (int r = 0; r < R; ++r) { bm_[r] = __ballot_sync(HQ_FULL, (mask >> r) & 1u); pre_[r + 1] = pre_[r] + __popc(bm_[r]); }\n"
          << "      for (int i0_ = 0; i0_ < pre_[R]; i0_ += 32) {\n"
          << "        const int t_ = i0_ + lane; const bool live_ = t_ < pre_[R];\n"
          << "        int rr_ = 0; u32 m_ = bm_[0]; int k_ = t_;\n"
          << "#pragma unroll\n        for (int r = 1; r < R; ++r) if (t_ >= pre_[r]) { rr_ = r; m_ = bm_[r]; k_ = t_ - pre_[r]; }\n"
          << "        int src_ = 0;\n#pragma unroll\n        for (int s_ = 16; s_ > 0; s_ >>= 1) { const int c_ = __popc((m_ >> src_) & ((1u << s_) - 1u)); if (k_ >= c_) { k_ -= c_; src_ += s_; } }\n"
          << "        if (!live_) src_ = lane;\n"
          << "        u64 key_ = 0; i64 v_[NAGGS > 0 ? NAGGS : 1];\n"
          << "#pragma unroll\n        for (int r = 0; r < R; ++r) { const u64 kx_ = __shfl_sync(HQ_FULL, gk_[r], src_); if (r == rr_) key_ = kx_;\n"
          << "#pragma unroll\n          for (int a = 0; a < NAGGS; ++a) { const i64 x_ = __shfl_sync(HQ_FULL, va_[a][r], src_); if (r == rr_) v_[a] = x_; } }\n";
      } else if (!c2) {
        // few live rows (selective joins): each live lane updates its own group
        // (the shared atomics resolve collisions), then one vote reconverges
        // the warp -- without it a warp could leave the divergent hash probing
        // split and run the rest of the kernel at half speed.  Otherwise rows
        // of equal keys are combined in registers first (match_any + reduce).
        o << "      u32 act_[R]; int nact_ = 0;\n#pragma unroll\n      for (int r = 0; r < R; ++r) { act_[r] = __ballot_sync(HQ_FULL, (mask >> r) & 1u); nact_ += __popc(act_[r]); }\n"
          // replicated tables, few live rows, or a dense shared domain of >= 1,024 groups
          // (keys rarely repeat inside a warp: match_any would find 32 singletons)
          << "      if (SCOPIES > 1 || nact_ <= 4 * R" << (kp.smode == SM_DENSE && kp.smem_cap >= 1024 ? " || true" : "")
          << ") {  // every live lane updates directly\n"
          // a lane's consecutive rows of one group (clustered keys: the lines of
          // an order) are folded first: one table update instead of a chain of
          // dependent global round trips (TPC-H Q3)
          << "        u64 cn_[R];\n#pragma unroll\n        for (int r = 0; r < R; ++r) cn_[r] = 1ull;\n";
        if (kp.smode == SM_NONE)  // only where an update is a dependent global round trip
          o << "#pragma unroll\n        for (int r = 1; r < R; ++r) if (((mask >> r) & 1u) && ((mask >> (r - 1)) & 1u) && gk_[r] == gk_[r - 1]) {\n"
            << "#pragma unroll\n          for (int a = 0; a < NAGGS; ++a) va_[a][r] = agg_combine(AGG_FN[a], va_[a][r], va_[a][r - 1]);\n"
            << "          cn_[r] += cn_[r - 1]; mask &= ~(1u << (r - 1)); }\n";
        o
          << "#pragma unroll\n        for (int r = 0; r < R; ++r) if ((mask >> r) & 1u) {\n"
          << "          i64 v_[NAGGS > 0 ? NAGGS : 1];\n#pragma unroll\n          for (int a = 0; a < NAGGS; ++a) v_[a] = va_[a][r];\n"
          << "          group_update(p, sagg, sl0_, gk_[r], true, cn_[r], v_); }\n"
          << "        nact_ = __popc(__ballot_sync(HQ_FULL, nact_ > 0));\n";
        o << "      } else {\n"
          << "#pragma unroll\n      for (int r = 0; r < R; ++r) {\n"
          << "        const bool live_ = (mask >> r) & 1u; const u64 key_ = gk_[r];\n"
          << "        i64 v_[NAGGS > 0 ? NAGGS : 1];\n#pragma unroll\n        for (int a = 0; a < NAGGS; ++a) v_[a] = va_[a][r];\n"
          << "        const u32 am_ = act_[r];\n";
      } else {
        o << "#pragma unroll\n      for (int r = 0; r < R; ++r) {\n"
          << "        const bool live_ = (mask >> r) & 1u; const u64 key_ = gk_[r];\n"
          << "        i64 v_[NAGGS > 0 ? NAGGS : 1];\n#pragma unroll\n        for (int a = 0; a < NAGGS; ++a) v_[a] = va_[a][r];\n";
      }
      if (wcompact || c2) o << "        const u32 am_ = __ballot_sync(HQ_FULL, live_);\n";
      if (c2) {
        o << "        if (live_) group_update(p, sagg, sl0_, key_, false, 1ull, v_);\n      }\n";
      } else {
        o << "        const bool sparse_ = __popc(am_) <= 4;\n"
          << "        const u64 mk_ = live_ ? key_ : HQ_EMPTY_KEY;\n"
          << "        const u32 peers_ = sparse_ ? ((1u << lane) & am_) : (__match_any_sync(HQ_FULL, mk_) & am_);\n"
          << "        const bool single_ = live_ && __popc(peers_) == 1;\n"
          // groups of several lanes are reduced in registers first (the loop has
          // no memory access); then every single lane and every group leader
          // updates the table in ONE pass, so the global round trips of a warp's
          // groups overlap instead of queueing one per group (TPC-H Q18/Q21:
          // GROUP BY l_orderkey, ~16 groups per warp)
          << "        u32 multi_ = am_ & ~__ballot_sync(HQ_FULL, single_);\n";
        // one pass only where an update is a global round trip (C2 straight to global):
        // with a shared-memory table the per-group updates are cheap and the extra
        // live registers cost ~1.5 % (SSB Q3.1 / Q4.1); HQ_JIT_ONEPASS=0/1 forces (A/B)
        const char* op1 = getenv("HQ_JIT_ONEPASS");
        const bool onepass = op1 ? op1[0] == '1' : kp.smode == SM_NONE;
        if (!onepass) {
          o << "        if (single_) group_update(p, sagg, sl0_, key_, true, 1ull, v_);\n"
            << "        while (multi_) {\n          const int leader_ = __ffs(multi_) - 1;\n"
            << "          const u32 grp_ = __shfl_sync(HQ_FULL, peers_, leader_); const bool mine_ = (grp_ >> lane) & 1u;\n"
            << "          i64 w_[NAGGS > 0 ? NAGGS : 1];\n#pragma unroll\n          for (int a = 0; a < NAGGS; ++a) w_[a] = warp_reduce(AGG_FN[a], mine_ ? v_[a] : agg_identity(AGG_FN[a]));\n"
            << "          if (lane == leader_) group_update(p, sagg, sl0_, key_, true, (u64)__popc(grp_), w_);\n"
            << "          multi_ &= ~grp_;\n        }\n      }\n";
        } else {
          o << "        bool upd_ = single_; u64 uc_ = 1ull;\n"
            << "        while (multi_) {\n          const int leader_ = __ffs(multi_) - 1;\n"
            << "          const u32 grp_ = __shfl_sync(HQ_FULL, peers_, leader_); const bool mine_ = (grp_ >> lane) & 1u;\n"
            << "          i64 w_[NAGGS > 0 ? NAGGS : 1];\n#pragma unroll\n          for (int a = 0; a < NAGGS; ++a) w_[a] = warp_reduce(AGG_FN[a], mine_ ? v_[a] : agg_identity(AGG_FN[a]));\n"
            << "          if (lane == leader_) {\n#pragma unroll\n            for (int a = 0; a < NAGGS; ++a) v_[a] = w_[a];\n"
            << "            uc_ = (u64)__popc(grp_); upd_ = true; }\n"
            << "          multi_ &= ~grp_;\n        }\n"
            << "        if (upd_) group_update(p, sagg, sl0_, key_, true, uc_, v_);\n      }\n";
        }
        if (!wcompact) o << "      }\n";  // else of the sparse path
      }
      }  // !gq
    }
  } else {  // materialise: hand the output values to the block scan below
    std::vector<std::string> ov;
    for (int j = 0; j < kp.nout; ++j) ov.push_back(g.val(kp.out_reg[j]));
    o << "#pragma unroll\n      for (int r = 0; r < R; ++r) {";
    for (int j = 0; j < kp.nout; ++j) o << " ov" << j << "[r] = (long long)" << ov[j] << ";";
    o << " }\n";
  }
  };
  // ---------------------------------------------------------------- kernel
  o << "extern \"C\" __global__ void __launch_bounds__((NW + 1) * 32, 1) hq_jit_kernel(const __grid_constant__ JParams p) {\n"
    << "  extern __shared__ __align__(128) char smem[];\n"
    << "  u64* full = (u64*)smem; u64* empty = full + 10;\n"
    << "  u64* s_base = (u64*)(empty + 10); int* s_wtot = (int*)(s_base + 32); i64* s_red = (i64*)(s_wtot + 32);\n"
    << "  char* sagg = smem + OFF_AGG; char* stages = smem + OFF_STAGE;\n"
    << "  const u32 sl0_ = smem_u32(sagg) + (u32)(((threadIdx.x >> 5) % SCOPIES) * SMEM_CAP * LVWORDS * 8u); (void)sl0_;\n"
    << "  const u32 sm0_ = smem_u32(smem); (void)sm0_;\n"
    << "  (void)s_base; (void)s_wtot; (void)s_red; (void)sagg;\n"
    << "  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;\n"
    << "  const long long first_tile = p.row_begin / T;\n"
    << "  const long long ntiles = p.row_end > p.row_begin ? (p.row_end + T - 1) / T - first_tile : 0;\n"
    << "  const long long nj = ntiles > blockIdx.x ? (ntiles - blockIdx.x + gridDim.x - 1) / gridDim.x : 0;\n"
    << "  const long long tstep = (long long)gridDim.x * T;\n"
    << "  if (threadIdx.x == 0) { for (int s = 0; s < S; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], NW); } fence_mbar_init(); }\n";
  if (prof) o << "  long long pt0_ = 0; if (threadIdx.x == 0) asm volatile(\"mov.u64 %0, %%globaltimer;\" : \"=l\"(pt0_));\n"
              << "  long long pw_ = 0, pl0_ = clock64(); int pdv_ = 0;\n";
  // smem table init
  if (sk == 1 && kp.smode == SM_LANE) {
    o << "  if (warp < NW) { i64* t_ = (i64*)sagg; for (u32 i = threadIdx.x; i < SMEM_CAP * NACC * NW * 32; i += NW * 32) {"
      << " const int a_ = (int)((i / (NW * 32)) % NACC); t_[i] = a_ == 0 ? 0 : agg_identity(ACC_FN[a_]); } }\n";
  } else if (sk == 1 && kp.smode == SM_DENSE) {
    o << "  if (warp < NW) { i64* t_ = (i64*)sagg; for (u32 i = threadIdx.x; i < SMEM_CAP * LVWORDS * SCOPIES; i += NW * 32) {"
      << " const int c_ = (int)(i % LVWORDS); t_[i] = c_ == 0 ? 0 : agg_identity(LFN[c_]); } }\n";
  } else if (sk == 1 && kp.smode == SM_HASH) {
    o << "  if (warp < NW) { u64* k_ = (u64*)sagg; i64* e_ = (i64*)sagg + SMEM_CAP;\n"
      << "    for (u32 i = threadIdx.x; i < SMEM_CAP; i += NW * 32) k_[i] = HQ_EMPTY_KEY;\n"
      << "    for (u32 i = threadIdx.x; i < SMEM_CAP * LVWORDS; i += NW * 32) { const int c_ = (int)(i % LVWORDS); e_[i] = c_ == 0 ? 0 : agg_identity(LFN[c_]); } }\n";
  }
  // staged compact probe tables: one cooperative 16-B copy per CTA
  for (int i = 0; i < MAX_PROBES; ++i) {
    const KProbe& pr = kp.probes[i];
    if (!pr.smem_off) continue;
    o << "  { const uint4* src_ = (const uint4*)p.ctab[" << i << "]; uint4* dst_ = (uint4*)(smem + " << pr.smem_off << "u);\n"
      << "    for (u32 x = threadIdx.x; x < " << (pr.cbytes + 15) / 16 << "u; x += blockDim.x) dst_[x] = __ldg(src_ + x); }\n";
  }
  o << "  __syncthreads();\n";
  // producer
  o << "  if (warp == NW) {\n    if (lane == 0) {\n      const u64 pol = policy_evict_first();\n"
    << "      int s = 0; u32 ph = 0; long long t0 = (first_tile + blockIdx.x) * (long long)T;\n"
    << "      for (long long j = 0; j < nj; ++j, t0 += tstep) {\n"
    << "        " << (prof ? "{ const long long c_ = clock64(); if (j >= S) mbar_wait(&empty[s], ph ^ 1u); pw_ += clock64() - c_; }" : "if (j >= S) mbar_wait(&empty[s], ph ^ 1u);") << "\n"
    << "        char* st = stages + (size_t)s * STAGE_STRIDE;\n"
    << "        if (t0 >= p.row_begin && t0 + T <= p.row_end) {\n          mbar_expect_tx(&full[s], STAGE_BYTES);\n";
  for (int k = 0; k < kp.ncols; ++k)
    if (!kp.cols[k].lazy)
    o << "          tma_load_1d(st + " << kp.cols[k].soff << "u, p.col[" << k << "] + t0 * " << kp.cols[k].width << ", "
      << kp.tile_rows * kp.cols[k].width << "u, &full[s], pol);\n";
  o << "        } else mbar_arrive(&full[s]);\n        if (++s == S) { s = 0; ph ^= 1u; }\n      }\n";
  if (prof) o << "      p.prof[blockIdx.x * 128 + 3] = pw_; p.prof[blockIdx.x * 128 + 4] = clock64() - pl0_;\n";
  o << "    }\n    return;\n  }\n";
  // consumer state
  o << "  const int row0 = warp * 32 * R + lane * R;  // the lane's rows: row0 .. row0 + R - 1\n";
  if (kp.a3stage == 1) o << "  u64 a3pend_ = 0;  // thread 0: the pending atomicAdd of the last tile (staged A3)\n";
  if (kp.a3stage == 2)
    o << "  char* wb_ = smem + OFF_AGG + (u32)warp * A3WBYTES; int wcnt_ = 0;  // the warp's row buffer (A3, warp workgroups)\n";
  if (gq)
    o << "  u64* gq_ = (u64*)(smem + OFF_AGG + (u32)warp * (GQ_CAP * (2u + NAGGS) * 8u)); int gqn_ = 0;  // the warp's update queue\n";
  if (sk == 0 && !c2 && !we) {
    o << "  u64 scount_ = 0;\n";
    for (int a = 0; a < kp.naggs; ++a) o << "  i64 sacc" << a << " = agg_identity(AGG_FN[" << a << "]);\n";
  }
  // HQ_JIT_WAIT=sleep: the older poll + nanosleep loop (A/B)
  const char* wm = getenv("HQ_JIT_WAIT");
  const std::string cwait = (wm && std::string(wm) == "sleep") ? "mbar_wait_sleep(&full[s], ph);" : "mbar_wait_suspend_a(sm0_ + 8u * (u32)s, ph);";
  // ---- software pipelining (two tiles per warp in flight).  A star join whose first
  // global-memory probe batch (byte maps / bitmaps in L2) every row waits on is split
  // there: phase A of a tile = stage wait, ragged copy, columns, filters and shared-memory
  // probes, and the batch's address + LOAD; phase B = the batch's resolution, the rest
  // of the operators and the sink.  The loop runs A(j+1) before B(j), so each warp has
  // two tiles' probe loads in flight instead of stalling on every tile's round trip.
  // The stage of tile j is held until B(j) ends (no early release), A's arrays are
  // declared once per tile parity (a / b, renamed with #define).
  int swp_split = -1;
  if (!mp && !c2 && !we && (sk == 0 || sk == 1) && kp.R == 2 && kp.smode != SM_LANE && !prof &&
      !(wm && std::string(wm) == "sleep") && g.lazy_k.empty() && getenv("HQ_JIT_SWP") && getenv("HQ_JIT_SWP")[0] == '1') {
    // opt-in: measured on B200 it LOSES (SSB Q3.1 SF30 0.56 -> 0.73 ms, Q4.1 SF100
    // 2.50 -> 3.29 ms): holding two stages per warp starves the 3-stage TMA ring and
    // the second tile's arrays spill at 64 registers; kept for experiments
    for (int i = 0; i < kp.nops && swp_split < 0; ++i) {
      if (kp.op_skip[i] || kp.ops[i].kind != OP_PROBE) continue;
      const int ak = Gen::access(kp.probes[kp.ops[i].idx]);
      if (ak == Gen::AK_LINEAR) break;
      if (ak == Gen::AK_GCOMPACT || ak == Gen::AK_DIRECT) swp_split = i;
    }
  }
  if (swp_split >= 0) {
    const std::string pre = o.str();
    o.str(std::string());
    o.clear();
    std::ostringstream decls;
    // ---- phase A (as text with base names)
    g.decl = &decls;
    decls << "  int si_; const char* st; long long tt_; u32 mask;\n";
    g.hoisted = {"si_", "st", "tt_", "mask"};
    o << "      mbar_wait_suspend_a(sm0_ + 8u * (u32)s, ph);\n"
      << "      si_ = s; st = stages + (size_t)s * STAGE_STRIDE; tt_ = t00_ + (long long)jt_ * tstep;\n"
      << "      mask = (1u << R) - 1u;\n"
      << "      if (jt_ == rj0_ || jt_ == rj1_) {  // ragged head / tail tile: lanes copy their rows\n"
      << "        const int lo = (int)(p.row_begin > tt_ ? p.row_begin - tt_ : 0);\n"
      << "        const int hi = (int)(p.row_end - tt_ < T ? p.row_end - tt_ : T);\n"
      << "        mask = 0;\n#pragma unroll\n        for (int r = 0; r < R; ++r) { const int row = row0 + r; if (row >= lo && row < hi) mask |= 1u << r; }\n";
    for (int k = 0; k < kp.ncols; ++k) {
      if (kp.cols[k].lazy) continue;
      const char* ty = ctype(kp.cols[k].width);
      o << "#pragma unroll\n        for (int r = 0; r < R; ++r) if (mask & (1u << r)) { const int row = row0 + r; ((" << ty
        << "*)(st + " << kp.cols[k].soff << "u))[row] = ((const " << ty << "*)p.col[" << k << "])[tt_ + row]; }\n";
    }
    o << "        fence_proxy_async(); __syncwarp();\n      }\n";
    g.begin_al();
    int i = 0;
    while (i < swp_split) {
      if (kp.op_skip[i]) { ++i; continue; }
      const KOp op = kp.ops[i];
      if (op.kind == OP_PROBE) { i = g.probe_batch(i); continue; }
      if (op.kind == OP_FILTER) g.filter(kp.preds[op.idx], op.idx);
      else g.compute(kp.comps[op.idx]);
      ++i;
    }
    i = g.probe_batch(swp_split, 1);
    o << "      if (++s == S) { s = 0; ph ^= 1u; }\n";
    const std::string acode = o.str();
    o.str(std::string());
    o.clear();
    // ---- phase B
    g.decl = nullptr;
    g.probe_batch(swp_split, 2);
    while (i < kp.nops) {
      if (kp.op_skip[i]) { ++i; continue; }
      const KOp op = kp.ops[i];
      if (op.kind == OP_PROBE) { i = g.probe_batch(i); continue; }
      if (op.kind == OP_FILTER) g.filter(kp.preds[op.idx], op.idx);
      else g.compute(kp.comps[op.idx]);
      ++i;
    }
    g.sync_mask();
    sink_tile();
    for (int k = 0; k < g.open; ++k) o << "      }\n";
    g.open = 0;
    o << "      __syncwarp();\n      if (lane == 0) mbar_arrive_a(sm0_ + 80u + 8u * (u32)si_);\n";
    const std::string bcode = o.str();
    // ---- assembly
    auto def = [&](const char* x) {
      std::string d;
      for (const auto& n : g.hoisted) d += "#define " + n + " " + n + "_" + x + "\n";
      return d;
    };
    auto undef = [&]() {
      std::string d;
      for (const auto& n : g.hoisted) d += "#undef " + n + "\n";
      return d;
    };
    o.str(pre);
    o.seekp(0, std::ios_base::end);
    o << "  // software-pipelined tile loop: A(j+1) before B(j)\n" << def("a") << decls.str() << undef() << def("b")
      << decls.str() << undef()
      << "  int s = 0; u32 ph = 0; const long long t00_ = (first_tile + blockIdx.x) * (long long)T;\n"
      << "  const int njc = (int)nj;\n"
      << "  const long long tl_ = t00_ + (nj - 1) * tstep;\n"
      << "  const int rj0_ = (nj > 0 && (t00_ < p.row_begin || t00_ + T > p.row_end)) ? 0 : -1;\n"
      << "  const int rj1_ = (nj > 0 && (tl_ < p.row_begin || tl_ + T > p.row_end)) ? njc - 1 : -1;\n"
      << "  if (njc > 0) {\n    const int jt_ = 0;\n" << def("a") << acode << undef() << "  }\n"
      << "  for (int j = 0; j < njc; j += 2) {\n"
      << "    if (j + 1 < njc) {\n      const int jt_ = j + 1;\n" << def("b") << acode << undef() << "    }\n"
      << "    {\n" << def("a") << bcode << undef() << "    }\n"
      << "    if (j + 1 >= njc) break;\n"
      << "    if (j + 2 < njc) {\n      const int jt_ = j + 2;\n" << def("a") << acode << undef() << "    }\n"
      << "    {\n" << def("b") << bcode << undef() << "    }\n"
      << "  }\n";
  } else {
  o << "  int s = 0; u32 ph = 0; long long t0 = (first_tile + blockIdx.x) * (long long)T;\n"
    << "  const int njc = (int)nj;\n"
    // only a CTA's first and last tile can be ragged (partition boundaries): decided once
    << "  const long long tl_ = t0 + (nj - 1) * tstep;\n"
    << "  const int rj0_ = (nj > 0 && (t0 < p.row_begin || t0 + T > p.row_end)) ? 0 : -1;\n"
    << "  const int rj1_ = (nj > 0 && (tl_ < p.row_begin || tl_ + T > p.row_end)) ? njc - 1 : -1;\n"
    << "  for (int j = 0; j < njc; ++j, t0 += tstep) {\n"
    << (prof ? "    { const long long c_ = clock64(); " + cwait + " pw_ += clock64() - c_; if (__activemask() != 0xffffffffu) ++pdv_; }\n" : "    " + cwait + "\n")
    << "    const char* st = stages + (size_t)s * STAGE_STRIDE;\n"
    << "    const long long tb_ = t0;  // tile start (temporaries t0, t1, ... shadow it below)\n"
    << "    u32 mask = (1u << R) - 1u;\n"
    << "    if (j == rj0_ || j == rj1_) {  // ragged head / tail tile: lanes copy their rows\n"
    << "      const int lo = (int)(p.row_begin > t0 ? p.row_begin - t0 : 0);\n"
    << "      const int hi = (int)(p.row_end - t0 < T ? p.row_end - t0 : T);\n"
    << "      mask = 0;\n#pragma unroll\n      for (int r = 0; r < R; ++r) { const int row = row0 + r; if (row >= lo && row < hi) mask |= 1u << r; }\n";
  for (int k = 0; k < kp.ncols; ++k) {
    if (kp.cols[k].lazy) continue;
    const char* ty = ctype(kp.cols[k].width);
    o << "#pragma unroll\n      for (int r = 0; r < R; ++r) if (mask & (1u << r)) { const int row = row0 + r; ((" << ty
      << "*)(st + " << kp.cols[k].soff << "u))[row] = ((const " << ty << "*)p.col[" << k << "])[t0 + row]; }\n";
  }
  o << "      fence_proxy_async(); __syncwarp();\n    }\n";
  if (sk == 2)  // output values leave the operator block in registers; the block scan runs after it
    for (int j = 0; j < kp.nout; ++j) o << "    long long ov" << j << "[R];\n";
  if (we && sk == 0 && !mp) {  // the tile's per-thread partials leave the operator block for the WE tree
    o << "    u32 wc_ = 0u; i64 wa_[NAGGS > 0 ? NAGGS : 1];\n#pragma unroll\n    for (int a = 0; a < NAGGS; ++a) wa_[a] = agg_identity(AGG_FN[a]);\n";
  } else if (we && sk == 1 && !mp) {  // the tile's live (key, values) leave it for the WE sort + segmented scan
    o << "    u32 wm_ = 0u; u64 wk_[R]; i64 wv_[NAGGS > 0 ? NAGGS : 1][R];\n";
  }
  o << "    {\n";
  if (kp.early_release) {
    // every referenced column of the lane's rows into registers, then the stage
    // goes back to the producer (mbarrier.arrive releases the warp's prior
    // shared loads); the operators below run on registers only
    for (const auto& sk2 : g.stage_k) g.use(sk2.first);
    // The arrive must not overtake the lanes' shared loads of the stage (the
    // producer's next TMA overwrites it): measured on B200, a bare __syncwarp +
    // arrive let ~1 % of SSB Q4.1 runs read a refilled value.  Every lane folds
    // its loaded registers, a ballot over the fold completes only after all
    // loads did, and lane 0 stores the ballot before its (release) arrive.
    const char* rf = getenv("HQ_JIT_RELFIX");  // A/B: dep (default), fence, none
    const std::string fix = rf ? rf : "dep";
    if (fix == "dep") {
      // one destination register per shared load instruction: a vector load
      // completes all its registers together, so element 0 stands for it
      o << "    { u32 f_ = 0u";
      for (const auto& sk2 : g.stage_k)
        if (g.vec_loaded.count(sk2.first)) o << " ^ (u32)" << g.var(sk2.first) << "[0]";
      o << ";\n";
      bool scalar = false;
      for (const auto& sk2 : g.stage_k) scalar = scalar || !g.vec_loaded.count(sk2.first);
      if (scalar) {
        o << "#pragma unroll\n      for (int r = 0; r < R; ++r) f_ ^= 0u";
        for (const auto& sk2 : g.stage_k)
          if (!g.vec_loaded.count(sk2.first)) o << " ^ (u32)" << g.var(sk2.first) << "[r]";
        o << ";\n";
      }
      o << "      const u32 b_ = __ballot_sync(HQ_FULL, f_ == 0x9E3779B9u);\n"
        << "      if (lane == 0) { *(volatile u32*)(smem + " << (MISC_DEP) << "u + 4u * warp) = b_; mbar_arrive_a(sm0_ + 80u + 8u * (u32)s); } }\n";
    } else if (fix == "fence") {
      o << "    fence_proxy_async(); __syncwarp();\n    if (lane == 0) mbar_arrive(&empty[s]);\n";
    } else {
      o << "    __syncwarp();\n    if (lane == 0) mbar_arrive(&empty[s]);\n";
    }
  }
  if (mp == 2) {  // the count kernel's flags select the rows
    const std::string f = g.val(kp.mp_flag_reg);
    o << "#pragma unroll\n      for (int r = 0; r < R; ++r) if (!" << f << ") mask &= ~(1u << r);\n";
  }
  // compaction point (Gen::compact): after the first probe that passes at most
  // half of the rows (build-side key density), aggregation sinks only, R >= 2
  int cpt = -1;
  if (sk != 2 && !c2 && kp.R >= 4 && kp.smode != SM_LANE)  // at R = 2 the shuffles cost more than they save (B200)
    for (int i = 0; i < kp.nops && cpt < 0; ++i)
      if (kp.ops[i].kind == OP_PROBE && kp.probes[kp.ops[i].idx].pass_est <= 0.5f) cpt = i;
  if (const char* e = getenv("HQ_JIT_CPT")) cpt = (e[0] == 'o') ? -1 : (sk != 2 ? atoi(e) : -1);
  if (mp) cpt = -1;
  g.begin_al();
  for (int i = 0; i < kp.nops;) {
    if (cpt >= 0 && !g.compacted_R && i > cpt) g.compact(i);
    if (kp.op_skip[i]) { ++i; continue; }  // not executed in this pass
    const KOp op = kp.ops[i];
    if (op.kind == OP_PROBE) { i = g.probe_batch(i); continue; }
    if (op.kind == OP_FILTER) g.filter(kp.preds[op.idx], op.idx);
    else g.compute(kp.comps[op.idx]);
    ++i;
  }
  if (cpt >= 0 && !g.compacted_R) g.compact(kp.nops);
  g.sync_mask();  // the sinks, the block scan and the count kernel's flags read mask
  if (mp == 1) {
    // count kernel: the flags are written below, after the early-exit blocks
    // close -- every row of the range gets its flag, also in a warp whose rows
    // all died before a linear probe (the buffer is not cleared)
  } else if (mp == 2) {
    // write kernel (Fig 8): flagged rows write at their prefix-sum position --
    // the projections (A1) or the aggregation inputs: packed group key, values (B1/C1)
    const std::string pv = g.val(kp.mp_pos_reg);
    if (sk == 2) {
      std::vector<std::string> ov;
      for (int j = 0; j < kp.nout; ++j) ov.push_back(g.val(kp.out_reg[j]));
      o << "#pragma unroll\n      for (int r = 0; r < R; ++r) if ((mask >> r) & 1u) { const u64 pos_ = (u64)(u32)" << pv << ";";
      for (int j = 0; j < kp.nout; ++j)
        o << " ((" << ctype(kp.out_width[j]) << "*)p.out[" << j << "])[pos_] = (" << ctype(kp.out_width[j]) << ")" << ov[j] << ";";
      o << " }\n";
    } else {
      o << "      u64 gk_[R]; bool bad_ = false;\n#pragma unroll\n      for (int r = 0; r < R; ++r) gk_[r] = 0;\n";
      for (int i = 0; i < kp.nkeys; ++i) {
        const std::string v = g.val(kp.key_reg[i]);
        o << "#pragma unroll\n      for (int r = 0; r < R; ++r) { const long long d_ = (long long)" << v << " - " << lit(kp.key_min[i])
          << "; if (d_ < 0 || d_ >= " << lit(kp.key_card[i]) << ") { if ((mask >> r) & 1u) bad_ = true; mask &= ~(1u << r); }"
          << " gk_[r] += (u64)d_ * " << kp.key_stride[i] << "ull; }\n";
      }
      o << "      if (bad_) atomicOr(p.err, F_KEY_DOMAIN);\n";
      std::vector<std::string> vv;
      for (int a = 0; a < kp.naggs; ++a) vv.push_back(kp.agg_fn[a] == HQ_AGG_COUNT ? std::string() : g.val(kp.agg_reg[a]));
      o << "#pragma unroll\n      for (int r = 0; r < R; ++r) if ((mask >> r) & 1u) { const u64 pos_ = (u64)(u32)" << pv << ";";
      int oc = 0;
      if (kp.nkeys > 0) o << " ((u64*)p.out[" << oc++ << "])[pos_] = gk_[r];";
      for (int a = 0; a < kp.naggs; ++a)
        if (kp.agg_fn[a] != HQ_AGG_COUNT) o << " ((i64*)p.out[" << oc++ << "])[pos_] = (i64)" << vv[a] << ";";
      o << " }\n";
    }
  } else {
  sink_tile();
  }  // !mp
  for (int k = 0; k < g.open; ++k) o << "    }\n";
  if (mp == 1)  // count kernel (Fig 8): one int32 flag per row, indexed by absolute row (base offset by the host)
    o << "      { int* fl_ = (int*)p.out[0];\n#pragma unroll\n      for (int r = 0; r < R; ++r) { const long long row_ = tb_ + row0 + r;"
      << " if (row_ >= p.row_begin && row_ < p.row_end) fl_[row_] = (int)((mask >> r) & 1u); } }\n";
  if (g.compacted_R) o << "#undef R\n#define R " << g.compacted_R << "\n";
  o << "    }\n";
  if (we && !mp) gen_we_tile(o, kp, sk);
  if (sk == 2 && !mp && !we && !c2 && kp.a3stage == 2) {
    // A3 with warp workgroups (LRGP: local resolution = the warp's ballot
    // prefix over its buffer, global propagation = one atomicAdd per full buffer): the
    // warp appends its live rows to its shared buffer and flushes it when the next tile's
    // rows might not fit -- no block barrier, no atomic round trip per tile.  Output:
    // each flush's rows contiguous, in row order; flushes permuted.
    o << "    {\n      const int mine_ = __popc(mask); int lin_ = mine_;\n"
      << "#pragma unroll\n      for (int o_ = 1; o_ < 32; o_ <<= 1) { const int t_ = __shfl_up_sync(HQ_FULL, lin_, o_); if (lane >= o_) lin_ += t_; }\n"
      << "      const int wtot_ = __shfl_sync(HQ_FULL, lin_, 31);\n"
      << "      if (wcnt_ + wtot_ > A3WROWS) { a3w_flush(p, wb_, wcnt_); wcnt_ = 0; }\n"
      << "      const int wo_ = wcnt_ + lin_ - mine_;\n"
      << "#pragma unroll\n      for (int r = 0; r < R; ++r) if ((mask >> r) & 1u) { const int pos_ = wo_ + __popc(mask & ((1u << r) - 1u));\n";
    for (int j = 0; j < kp.nout; ++j)
      o << "        ((" << ctype(kp.out_width[j]) << "*)(wb_ + " << kp.a3_col[j] << "u))[pos_] = (" << ctype(kp.out_width[j]) << ")ov" << j << "[r];\n";
    o << "      }\n      wcnt_ += wtot_;\n      __syncwarp();\n    }\n";
  } else if (sk == 2 && !mp && !we && !c2 && kp.a3stage == 1) {
    // A3 (Fig 25 / P:1069-1072) with a deferred write-out: warp ballots -> block scan
    // over the warps -> ONE atomicAdd per block and tile, issued by thread 0 and not
    // waited for: the tile's rows go to a shared staging buffer at their tile-local
    // positions, and during the NEXT tile (after its first barrier) the whole CTA
    // copies them, coalesced, to base + position -- the atomic's round trip is off the
    // tile's critical path.  Output order: each tile's rows contiguous, in row order.
    o << "    {\n      const int buf_ = j & 1;\n"
      << "      if (threadIdx.x == 0 && j > 0) s_red[buf_ ^ 1] = (i64)a3pend_;  // the previous tile's base\n"
      << "      const int mine_ = __popc(mask); int lin_ = mine_;\n"
      << "#pragma unroll\n      for (int o_ = 1; o_ < 32; o_ <<= 1) { const int t_ = __shfl_up_sync(HQ_FULL, lin_, o_); if (lane >= o_) lin_ += t_; }\n"
      << "      const int wtot_ = __shfl_sync(HQ_FULL, lin_, 31);\n"
      << "      if (lane == 0) s_wtot[warp] = wtot_;\n      consumer_bar();\n"
      << "      if (j > 0) a3_flush(p, s_red[buf_ ^ 1], (int)s_red[2 + (buf_ ^ 1)], smem + OFF_AGG + (buf_ ^ 1) * A3BUF);\n"
      << "      if (warp == 0) { const int v_ = lane < NW ? s_wtot[lane] : 0; int incl_ = v_;\n"
      << "#pragma unroll\n        for (int o_ = 1; o_ < 32; o_ <<= 1) { const int t_ = __shfl_up_sync(HQ_FULL, incl_, o_); if (lane >= o_) incl_ += t_; }\n"
      << "        const int total_ = __shfl_sync(HQ_FULL, incl_, 31);\n"
      << "        if (lane < NW) s_base[lane] = (u64)(incl_ - v_);\n"
      << "        if (lane == 0) { s_red[2 + buf_] = total_; a3pend_ = total_ > 0 ? atomicAdd(p.counter, (u64)total_) : 0ull; } }\n"
      << "      consumer_bar();\n"
      << "      char* sb_ = smem + OFF_AGG + buf_ * A3BUF;\n"
      << "      const int wo_ = (int)s_base[warp] + (lin_ - mine_);\n"
      << "#pragma unroll\n      for (int r = 0; r < R; ++r) if ((mask >> r) & 1u) { const int pos_ = wo_ + __popc(mask & ((1u << r) - 1u));\n";
    for (int j = 0; j < kp.nout; ++j)
      o << "        ((" << ctype(kp.out_width[j]) << "*)(sb_ + " << kp.a3_col[j] << "u))[pos_] = (" << ctype(kp.out_width[j]) << ")ov" << j << "[r];\n";
    o << "      }\n    }\n";
  } else if (sk == 2 && !mp && !we) {
    // A3 (Fig 25 / P:1069-1072): warp ballots -> block scan over the warps ->
    // one atomicAdd per block and tile -> writes at local + global offset.
    // Every consumer warp takes part in every tile (its mask may be empty).
    // a lane's rows are consecutive: positions in row order are the lane's
    // exclusive prefix over the warp plus its live rows below r
    if (c2) {
      o << "    {\n#pragma unroll\n      for (int r = 0; r < R; ++r) if ((mask >> r) & 1u) { const u64 pos_ = atomicAdd(p.counter, 1ull);\n";
    } else {
      o << "    {\n      const int mine_ = __popc(mask); int lin_ = mine_;\n"
        << "#pragma unroll\n      for (int o_ = 1; o_ < 32; o_ <<= 1) { const int t_ = __shfl_up_sync(HQ_FULL, lin_, o_); if (lane >= o_) lin_ += t_; }\n"
        << "      const int wtot_ = __shfl_sync(HQ_FULL, lin_, 31);\n"
        << "      if (lane == 0) s_wtot[warp] = wtot_;\n      consumer_bar();\n"
        << "      if (warp == 0) { const int v_ = lane < NW ? s_wtot[lane] : 0; int incl_ = v_;\n"
        << "#pragma unroll\n        for (int o_ = 1; o_ < 32; o_ <<= 1) { const int t_ = __shfl_up_sync(HQ_FULL, incl_, o_); if (lane >= o_) incl_ += t_; }\n"
        << "        const int total_ = __shfl_sync(HQ_FULL, incl_, 31); u64 g_ = 0;\n"
        << "        if (lane == 0 && total_ > 0) g_ = atomicAdd(p.counter, (u64)total_);\n"
        << "        g_ = __shfl_sync(HQ_FULL, g_, 0); if (lane < NW) s_base[lane] = g_ + (u64)(incl_ - v_); }\n"
        << "      consumer_bar();\n"
        << "      const u64 base_ = s_base[warp] + (u64)(lin_ - mine_);\n"
        << "#pragma unroll\n      for (int r = 0; r < R; ++r) { if ((mask >> r) & 1u) { const u64 pos_ = base_ + __popc(mask & ((1u << r) - 1u));\n";
    }
    o << "        if ((long long)pos_ < p.capacity) {\n";
    for (int j = 0; j < kp.nout; ++j)
      o << "          ((" << ctype(kp.out_width[j]) << "*)p.out[" << j << "])[pos_] = (" << ctype(kp.out_width[j]) << ")ov" << j << "[r];\n";
    o << "        } else atomicOr(p.err, F_CAPACITY); }\n";
    if (!c2) o << "        }\n";
    o << "    }\n";
  }
  if (kp.early_release) o << "    if (++s == S) { s = 0; ph ^= 1u; }\n  }\n";
  else o << "    __syncwarp();\n    if (lane == 0) mbar_arrive_a(sm0_ + 80u + 8u * (u32)s);\n    if (++s == S) { s = 0; ph ^= 1u; }\n  }\n";
  }  // software pipelining
  if (prof) o << "  if (lane == 0) { p.prof[blockIdx.x * 128 + 8 + warp] = pw_; p.prof[blockIdx.x * 128 + 40 + warp] = clock64() - pl0_; } if (pdv_) atomicAdd((unsigned long long*)&p.prof[blockIdx.x * 128 + 72 + warp], (unsigned long long)pdv_);\n";
  if (kp.a3stage == 2 && sk == 2 && !mp && !we && !c2)  // the rows still in the warp's buffer
    o << "  if (wcnt_ > 0) a3w_flush(p, wb_, wcnt_);\n";
  if (gq) o << "  if (gqn_ > 0) gq_flush(p, sagg, sl0_, gq_, gqn_);  // the updates still queued\n";
  if (kp.a3stage == 1 && sk == 2 && !mp && !we && !c2)  // the last tile's staged rows
    o << "  if (njc > 0) { const int lb_ = (njc - 1) & 1; if (threadIdx.x == 0) s_red[lb_] = (i64)a3pend_; consumer_bar();\n"
      << "    a3_flush(p, s_red[lb_], (int)s_red[2 + lb_], smem + OFF_AGG + lb_ * A3BUF); }\n";
  // ------------------------------------------------------------- sink (end)
  if (mp) {
  } else if (sk == 0 && !c2 && !we) {
    o << "  { u64 c_ = scount_;\n#pragma unroll\n    for (int o_ = 16; o_ > 0; o_ >>= 1) c_ += __shfl_xor_sync(HQ_FULL, c_, o_);\n";
    for (int a = 0; a < kp.naggs; ++a) o << "    const i64 r" << a << " = warp_reduce(AGG_FN[" << a << "], sacc" << a << ");\n";
    o << "    if (lane == 0) { s_red[warp * 9] = (i64)c_;";
    for (int a = 0; a < kp.naggs; ++a) o << " s_red[warp * 9 + " << 1 + a << "] = r" << a << ";";
    o << " }\n    consumer_bar();\n    if (threadIdx.x == 0) { u64 cnt_ = 0;";
    for (int a = 0; a < kp.naggs; ++a) o << " i64 x" << a << " = agg_identity(AGG_FN[" << a << "]);";
    o << "\n      for (int w = 0; w < NW; ++w) { cnt_ += (u64)s_red[w * 9];";
    for (int a = 0; a < kp.naggs; ++a) o << " x" << a << " = agg_combine(AGG_FN[" << a << "], x" << a << ", s_red[w * 9 + " << 1 + a << "]);";
    o << " }\n      if (cnt_) { g_add64(p.gtab, (i64)cnt_);";
    for (int a = 0; a < kp.naggs; ++a) o << " g_agg(AGG_FN[" << a << "], p.gtab + " << 1 + a << ", x" << a << ", cnt_);";
    o << " } } }\n";
  } else if (sk == 1 && kp.smode == SM_LANE) {
    o << "  consumer_bar();\n  { const i64* t_ = (const i64*)sagg;\n"
      << "    for (u32 g = threadIdx.x; g < SMEM_CAP; g += NW * 32) {\n"
      << "      const i64* e_ = t_ + (u64)g * NACC * NW * 32; u64 cnt_ = 0;\n"
      << "      for (int l = 0; l < NW * 32; ++l) cnt_ += (u64)e_[l];\n      if (!cnt_) continue;\n"
      << "      i64 acc_[NACC];\n#pragma unroll\n      for (int a = 1; a < NACC; ++a) { i64 v = agg_identity(ACC_FN[a]);"
      << " for (int l = 0; l < NW * 32; ++l) v = agg_combine(ACC_FN[a], v, e_[a * NW * 32 + l]); acc_[a] = v; }\n"
      << "      i64 vals_[NAGGS > 0 ? NAGGS : 1];\n";
    for (int a = 0; a < kp.naggs; ++a)
      o << "      vals_[" << a << "] = " << (kp.acc_of[a] ? "acc_[" + std::to_string(kp.acc_of[a]) + "]" : std::string("(i64)cnt_")) << ";\n";
    o << "      group_update(p, sagg, sl0_, g, false, cnt_, vals_);\n    } }\n";
  } else if (sk == 1 && kp.smode == SM_DENSE) {
    // the group's entries in every replica are combined first
    o << "  consumer_bar();\n  { const i64* t_ = (const i64*)sagg;\n"
      << "    for (u32 g = threadIdx.x; g < SMEM_CAP; g += NW * 32) { i64 cnt_ = 0; i64 vals_[NAGGS > 0 ? NAGGS : 1];\n"
      << "#pragma unroll\n      for (int a = 0; a < NAGGS; ++a) vals_[a] = agg_identity(AGG_FN[a]);\n"
      << "      for (u32 c_ = 0; c_ < SCOPIES; ++c_) { const i64* e_ = t_ + ((u64)c_ * SMEM_CAP + g) * LVWORDS; cnt_ += e_[0];\n"
      << "#pragma unroll\n        for (int a = 0; a < NAGGS; ++a) if (AGG_FN[a] != F_COUNT) vals_[a] = agg_combine(AGG_FN[a], vals_[a], e_[LCOL[a]]); }\n"
      << "      if (cnt_ != 0) {\n#pragma unroll\n        for (int a = 0; a < NAGGS; ++a) if (AGG_FN[a] == F_COUNT) vals_[a] = cnt_;\n"
      << "        u64 gkey_ = g;\n";
    if (kp.local_keys) {  // narrowed local index -> declared global key
      o << "        { u64 rem_ = g; gkey_ = 0;";
      for (int i = 0; i < kp.nkeys; ++i) {
        const uint64_t* ls = kp.lkey_set[i];
        o << " { const u64 o_ = rem_ / " << kp.lkey_stride[i] << "ull; rem_ -= o_ * " << kp.lkey_stride[i] << "ull;";
        if (ls[0] | ls[1] | ls[2] | ls[3]) {  // rank -> value -> offset in the declared domain
          o << " const long long dv_[] = {";
          int n = 0;
          for (int64_t d = 0; d < 256; ++d)
            if ((ls[d >> 6] >> (d & 63)) & 1ull) o << (n++ ? ", " : "") << (kp.lkey_min[i] + d - kp.key_min[i]) << "LL";
          o << "}; gkey_ += (u64)dv_[o_] * " << kp.key_stride[i] << "ull; }";
        } else {
          o << " gkey_ += (o_ + " << (kp.lkey_min[i] - kp.key_min[i]) << "ull) * " << kp.key_stride[i] << "ull; }";
        }
      }
      o << " }\n";
    }
    o << "        group_update(p, sagg, sl0_, gkey_, false, (u64)cnt_, vals_); } } }\n";
  } else if (sk == 1 && kp.smode == SM_HASH) {
    o << "  consumer_bar();\n  { const u64* k_ = (const u64*)sagg; const i64* t_ = (const i64*)sagg + SMEM_CAP;\n"
      << "    for (u32 h = threadIdx.x; h < SMEM_CAP; h += NW * 32) if (k_[h] != HQ_EMPTY_KEY) { const i64* e_ = t_ + (u64)h * LVWORDS;\n"
      << "      i64 vals_[NAGGS > 0 ? NAGGS : 1];\n#pragma unroll\n      for (int a = 0; a < NAGGS; ++a) vals_[a] = AGG_FN[a] == F_COUNT ? e_[0] : e_[LCOL[a]];\n"
      << "      group_update(p, sagg, sl0_, k_[h], false, (u64)e_[0], vals_); } }\n";
  }
  if (prof) o << "  if (threadIdx.x == 0) { long long t_; asm volatile(\"mov.u64 %0, %%globaltimer;\" : \"=l\"(t_)); p.prof[blockIdx.x * 128] = pt0_; p.prof[blockIdx.x * 128 + 5] = t_;"
              << " unsigned sm_; asm(\"mov.u32 %0, %%smid;\" : \"=r\"(sm_)); p.prof[blockIdx.x * 128 + 6] = sm_; }\n";
  o << "}\n";

  // ---------------------------------------------------------- constants
  std::ostringstream h;
  h << "// generated by libhq (hq_jit.cu) for one fusion operator\n"
    << "#define NW " << kp.nw << "\n#define R " << kp.R << "\n#define T " << kp.tile_rows << "\n#define S " << kp.nstages
    << "\n#define WAIT_NS " << wait_ns << "\n#define STAGE_STRIDE " << kp.stage_stride << "u\n#define STAGE_BYTES " << kp.stage_bytes
    << "u\n#define OFF_AGG " << kp.off_agg << "u\n#define OFF_STAGE " << kp.off_stage << "u\n"
    << "#define NAGGS " << kp.naggs << "\n#define VWORDS " << kp.vwords << "\n#define GMODE " << (int)kp.gmode
    << "\n#define SMODE " << (kp.smode == SM_LANE ? 0 : (int)kp.smode) << "\n#define SMEM_CAP " << kp.smem_cap
    << "u\n#define SCOPIES " << (kp.scopies ? kp.scopies : 1) << "u\n#define SLOG2 " << kp.slog2 << "\n#define NACC " << (kp.nacc > 0 ? kp.nacc : 1) << "\n"
    << "static constexpr __device__ int AGG_FN[" << (kp.naggs > 0 ? kp.naggs : 1) << "] = " << fn_list(kp.agg_fn, kp.naggs)
    << ";\n"
    << "static constexpr __device__ int ACC_FN[" << (kp.nacc > 0 ? kp.nacc : 1) << "] = " << fn_list(kp.acc_fn, kp.nacc) << ";\n"
    << "#define LVWORDS " << kp.lvwords << "\n" << lcol_tables(kp)
    << HQ_STR(HQ_JPARAMS_DEF) << "\n"
    << "#define GQ_CAP " << (gq ? (int)kp.gq_cap : 0) << "u\n"
    << kPrelude << "\n" << a3_flush_fn(kp)
    << (gq ? "// a warp's queued group updates, one per lane (all lanes of the warp call it)\n"
             "__device__ __noinline__ void gq_flush(const JParams& p, char* sagg, u32 sl0, u64* q, int n) {\n"
             "  __syncwarp();\n"
             "  for (int i = (int)(threadIdx.x & 31); i < n; i += 32) { i64 v_[NAGGS > 0 ? NAGGS : 1];\n"
             "#pragma unroll\n    for (int a = 0; a < NAGGS; ++a) v_[a] = (i64)q[(2 + a) * GQ_CAP + i];\n"
             "    group_update(p, sagg, sl0, q[i], false, q[GQ_CAP + i], v_); }\n"
             "  __syncwarp();\n}\n" : "")
    << g.bitmaps.str() << "\n";
  return h.str() + o.str();
}

CUfunction compile(hq_ctx* ctx, const std::string& src) {
  const auto key = std::make_pair(ctx->device, src);
  {
    std::lock_guard<std::mutex> gl(g_mu);
    auto it = g_cache.find(key);
    if (it != g_cache.end()) return it->second;
  }
  // HQ_JIT_DUMP=<dir>: write each generated source there (ncu --resolve-source-file)
  std::string name = "hq_jit_kernel.cu";
  if (const char* dir = getenv("HQ_JIT_DUMP")) {
    name = std::string(dir) + "/hq_jit_" + std::to_string(std::hash<std::string>{}(src) % 1000000007ULL) + ".cu";
    if (FILE* f = fopen(name.c_str(), "w")) {
      fwrite(src.data(), 1, src.size(), f);
      fclose(f);
    }
  }
  nvrtcProgram prog;
  if (nvrtcCreateProgram(&prog, src.c_str(), name.c_str(), 0, nullptr, nullptr) != NVRTC_SUCCESS)
    HQ_THROW(HQ_ERR_CUDA, "nvrtcCreateProgram failed");
  const char* opts[] = {"--gpu-architecture=sm_100a", "-std=c++17", "-lineinfo", "--device-int128"};
  const nvrtcResult rc = nvrtcCompileProgram(prog, 4, opts);
  if (rc != NVRTC_SUCCESS) {
    size_t n = 0;
    nvrtcGetProgramLogSize(prog, &n);
    std::string log(n, '\0');
    nvrtcGetProgramLog(prog, &log[0]);
    nvrtcDestroyProgram(&prog);
    HQ_THROW(HQ_ERR_CUDA, "NVRTC compile failed:\n" + log.substr(0, 4000));
  }
  size_t n = 0;
  nvrtcGetCUBINSize(prog, &n);
  std::string cubin(n, '\0');
  nvrtcGetCUBIN(prog, &cubin[0]);
  nvrtcDestroyProgram(&prog);
  Driver& d = driver();
  CUmodule mod;
  CUfunction fn;
  if (d.modload(&mod, cubin.data()) != CUDA_SUCCESS) HQ_THROW(HQ_ERR_CUDA, "cuModuleLoadData failed");
  if (d.getfn(&fn, mod, "hq_jit_kernel") != CUDA_SUCCESS) HQ_THROW(HQ_ERR_CUDA, "cuModuleGetFunction failed");
  std::lock_guard<std::mutex> gl(g_mu);
  g_cache[key] = fn;
  return fn;
}

}  // namespace

bool hq_jit_enabled() {
  const char* e = getenv("HQ_JIT");
  return !(e && e[0] == '0');
}

std::string hq_jit_source(const KPlan& kp) { return generate(kp); }

namespace {
thread_local CUfunction t_last_fn = nullptr;  // kernel compiled by the last hq_jit_prepare
}

namespace {
// The generated source depends on the plan's shape and constants, not on its
// runtime arguments (pointers, row range): key the kernel cache on the plan
// bytes with pointers reduced to null / non-null, so a repeated query skips
// source generation entirely.
std::string plan_key(const KPlan& kp) {
  KPlan k = kp;
  auto nz = [](const void* p) { return (const char*)(p ? 1 : 0); };
  k.row_begin = k.row_end = 0;
  k.capacity = 0;  // runtime parameters of the launch, not of the source
  k.gmask = 0;
  k.glog2 = 0;
  for (auto& c : k.cols) c.ptr = nz(c.ptr);
  for (auto& pr : k.probes) {
    pr.slots = (const uint32_t*)nz(pr.slots);
    pr.compact = nz(pr.compact);
    pr.pf = (const uint32_t*)nz(pr.pf);
    pr.rpay = (const int32_t*)nz(pr.rpay);
  }
  k.gtab = (long long*)nz(k.gtab);
  for (auto& o : k.out_ptr) o = (void*)nz(o);
  k.counter = (unsigned long long*)nz(k.counter);
  k.err = (int*)nz(k.err);
  return std::string((const char*)&k, sizeof(k));
}
std::map<std::pair<int, std::string>, CUfunction> g_plan_cache;
}  // namespace

void hq_jit_prepare(hq_ctx* ctx, const KPlan& kp, size_t smem) {
  const auto key = std::make_pair(ctx->device, plan_key(kp));
  CUfunction fn = nullptr;
  {
    std::lock_guard<std::mutex> gl(g_mu);
    auto it = g_plan_cache.find(key);
    if (it != g_plan_cache.end()) fn = it->second;
  }
  if (!fn) {
    fn = compile(ctx, generate(kp));
    std::lock_guard<std::mutex> gl(g_mu);
    g_plan_cache[key] = fn;
  }
  if (driver().setattr(fn, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, (int)smem) != CUDA_SUCCESS)
    HQ_THROW(HQ_ERR_CUDA, "cuFuncSetAttribute failed");
  t_last_fn = fn;
}

void hq_jit_launch(hq_ctx* ctx, const KPlan& kp, int grid, size_t smem) {
  CUfunction fn = t_last_fn;
  if (!fn) HQ_THROW(HQ_ERR_STATE, "jit: hq_jit_prepare not called");
  Driver& d = driver();
  JParams jp{};
  jp.row_begin = kp.row_begin;
  jp.row_end = kp.row_end;
  for (int k = 0; k < kp.ncols; ++k) jp.col[k] = kp.cols[k].ptr;
  for (int i = 0; i < MAX_PROBES; ++i) {
    jp.ht[i] = kp.probes[i].slots;
    jp.ctab[i] = kp.probes[i].compact;
    jp.pf[i] = kp.probes[i].pf;
    jp.rpay[i] = kp.probes[i].rpay;
  }
  jp.gtab = kp.gtab;
  jp.gmask = kp.gmask;
  jp.glog2 = kp.glog2;
  for (int j = 0; j < kp.nout; ++j) jp.out[j] = kp.out_ptr[j];
  jp.capacity = kp.capacity;
  jp.counter = kp.counter;
  jp.err = kp.err;
  static long long* prof_buf = nullptr;  // HQ_JIT_PROF (debug) only
  const bool prof = getenv("HQ_JIT_PROF") != nullptr;
  if (prof) {
    if (!prof_buf) HQ_CUDA(cudaMalloc(&prof_buf, 1024 * 128 * sizeof(long long)));
    HQ_CUDA(cudaMemsetAsync(prof_buf, 0, (size_t)grid * 128 * sizeof(long long), ctx->stream));
    jp.prof = prof_buf;
  }
  void* args[] = {&jp};
  ctx->launches++;
  if (d.launch(fn, (unsigned)grid, 1, 1, (unsigned)((kp.nw + 1) * 32), 1, 1, (unsigned)smem, (CUstream)ctx->stream, args,
               nullptr) != CUDA_SUCCESS)
    HQ_THROW(HQ_ERR_CUDA, "cuLaunchKernel failed");
  if (prof) {
    std::vector<long long> h((size_t)grid * 128);
    HQ_CUDA(cudaMemcpyAsync(h.data(), prof_buf, h.size() * 8, cudaMemcpyDeviceToHost, ctx->stream));
    HQ_CUDA(cudaStreamSynchronize(ctx->stream));
    long long t0 = LLONG_MAX, t1 = 0;
    auto dur = [&](int b) { return h[b * 128 + 5] - h[b * 128]; };
    for (int b = 0; b < grid; ++b) { t0 = std::min(t0, h[b * 128]); t1 = std::max(t1, h[b * 128 + 5]); }
    int slow = 0, fast = 0, nslow = 0;
    for (int b = 0; b < grid; ++b) {
      if (dur(b) > dur(slow)) slow = b;
      if (dur(b) < dur(fast)) fast = b;
    }
    for (int b = 0; b < grid; ++b) nslow += dur(b) > dur(fast) * 5 / 4;
    fprintf(stderr, "[hq prof] grid %d span %lld ns, %d CTAs >1.25x the fastest\n", grid, t1 - t0, nslow);
    for (int b : {slow, fast}) {
      fprintf(stderr, "  cta %d sm %lld dur %lld ns producer wait/loop %lld/%lld cyc; warp waits (kcyc):", b, h[b * 128 + 6], dur(b),
              h[b * 128 + 3], h[b * 128 + 4]);
      for (int w = 0; w < kp.nw; ++w) fprintf(stderr, " %lld", h[b * 128 + 8 + w] / 1000);
      fprintf(stderr, "\n    diverged-at-wait lane-iterations per warp:");
      for (int w = 0; w < kp.nw; ++w) fprintf(stderr, " %lld", h[b * 128 + 72 + w]);
      fprintf(stderr, "\n");
    }
  }
}
