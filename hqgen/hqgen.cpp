// hqgen.cpp -- deterministic TPC-H / SSB shaped generator.  See hqgen.h and
// SURVEY.md §8(d.1).  No query arithmetic lives here: only table contents.
#include "hqgen.h"

#include <algorithm>
#include <cmath>
#include <cstring>
#include <map>
#include <memory>
#include <mutex>
#include <thread>
#include <tuple>
#include <vector>

namespace {

inline uint64_t mix64(uint64_t z) {
  z += 0x9e3779b97f4a7c15ULL;
  z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ULL;
  z = (z ^ (z >> 27)) * 0x94d049bb133111ebULL;
  return z ^ (z >> 31);
}
// One independent stream per (table, column); value = f(seed, stream, idx).
inline uint64_t rnd(uint64_t seed, uint32_t stream, uint64_t idx) {
  return mix64(mix64(seed ^ (0xD1B54A32D192ED03ULL * (uint64_t)(stream + 1))) ^ idx);
}
// uniform integer in [lo, hi]
inline int64_t uni(uint64_t seed, uint32_t stream, uint64_t idx, int64_t lo, int64_t hi) {
  uint64_t r = rnd(seed, stream, idx);
  uint64_t span = (uint64_t)(hi - lo + 1);
  return lo + (int64_t)(((unsigned __int128)r * span) >> 64);
}
inline uint32_t S(int table, int col) { return (uint32_t)(table * 64 + col); }
enum { COL_NLINES = 63 };  // private stream for lines-per-order

// ---- calendar ----------------------------------------------------------
// days_from_civil / civil_from_days (proleptic Gregorian), epoch 1992-01-01.
int64_t days_from_civil(int64_t y, unsigned m, unsigned d) {
  y -= m <= 2;
  const int64_t era = (y >= 0 ? y : y - 399) / 400;
  const unsigned yoe = (unsigned)(y - era * 400);
  const unsigned doy = (153 * (m + (m > 2 ? -3 : 9)) + 2) / 5 + d - 1;
  const unsigned doe = yoe * 365 + yoe / 4 - yoe / 100 + doy;
  return era * 146097 + (int64_t)doe - 719468;
}
const int64_t kEpoch = days_from_civil(1992, 1, 1);
void civil_from_day(int32_t day, int* Y, int* M, int* D) {
  int64_t z = day + kEpoch + 719468;
  const int64_t era = (z >= 0 ? z : z - 146096) / 146097;
  const unsigned doe = (unsigned)(z - era * 146097);
  const unsigned yoe = (doe - doe / 1460 + doe / 36524 - doe / 146096) / 365;
  int64_t y = (int64_t)yoe + era * 400;
  const unsigned doy = doe - (365 * yoe + yoe / 4 - yoe / 100);
  const unsigned mp = (5 * doy + 2) / 153;
  const unsigned d = doy - (153 * mp + 2) / 5 + 1;
  const unsigned m = mp + (mp < 10 ? 3 : -9);
  *Y = (int)(y + (m <= 2));
  *M = (int)m;
  *D = (int)d;
}
inline int32_t yyyymmdd(int32_t day) {
  int y, m, d;
  civil_from_day(day, &y, &m, &d);
  return y * 10000 + m * 100 + d;
}
const int32_t kSsbDays = 2557;   // 1992-01-01 .. 1998-12-31
const int32_t kTpchODays = 2406; // o_orderdate: 1992-01-01 .. 1998-08-02
const int32_t kCurrentDay = (int32_t)(days_from_civil(1995, 6, 17) - kEpoch);  // TPC-H CURRENTDATE

// ---- sizes -------------------------------------------------------------
inline int64_t scaled(double base, double sf) {
  int64_t n = (int64_t)std::llround(base * sf);
  return n < 1 ? 1 : n;
}
int64_t ssb_parts(double sf) {
  if (sf >= 1.0) return 200000LL * (1 + (int64_t)std::floor(std::log2(sf)));
  return scaled(200000.0, sf);
}
int64_t n_orders(double sf) { return scaled(1500000.0, sf); }

// region of each nation code (order-preserving alphabetical dictionaries;
// see hqgen/__init__.py NATIONS / REGIONS).
const int8_t kNationRegion[25] = {0, 1, 1, 1, 2, 4, 0, 3, 3, 2, 2, 4, 4,
                                  2, 4, 0, 0, 0, 1, 3, 3, 4, 3, 1, 2};

inline int32_t orderkey(int64_t i) { return (int32_t)(32 * (i / 8) + (i % 8) + 1); }
inline int32_t retailprice(int64_t pk) {  // cents, TPC-H P_RETAILPRICE x 100
  return (int32_t)(90000 + ((pk / 10) % 20001) + 100 * (pk % 1000));
}
inline int nlines(int table, uint64_t seed, int64_t i) {
  return (int)uni(seed, S(table, COL_NLINES), (uint64_t)i, 1, 7);
}

// ---- order -> row index (cached) ----------------------------------------
constexpr int64_t kChunk = 1024;
struct LineIndex {
  int64_t norders = 0, nrows = 0;
  std::vector<int64_t> chunk_off;  // rows before chunk c (size nchunks+1)
};
std::mutex g_mu;
std::map<std::tuple<int, uint64_t, uint64_t>, std::shared_ptr<LineIndex>> g_cache;

int hw_threads(int n) {
  if (n > 0) return n;
  unsigned h = std::thread::hardware_concurrency();
  return h ? (int)h : 1;
}

template <class F>
void parallel_for(int64_t n, int nthreads, F f) {
  nthreads = (int)std::max<int64_t>(1, std::min<int64_t>(nthreads, (n + 65535) / 65536));
  if (nthreads <= 1) { f(0, n); return; }
  std::vector<std::thread> th;
  for (int t = 0; t < nthreads; ++t) {
    int64_t a = n * t / nthreads, b = n * (t + 1) / nthreads;
    th.emplace_back([=] { f(a, b); });
  }
  for (auto& x : th) x.join();
}

std::shared_ptr<LineIndex> line_index(int table, double sf, uint64_t seed, int nthreads) {
  uint64_t sfbits;
  std::memcpy(&sfbits, &sf, 8);
  auto key = std::make_tuple(table, sfbits, seed);
  {
    std::lock_guard<std::mutex> g(g_mu);
    auto it = g_cache.find(key);
    if (it != g_cache.end()) return it->second;
  }
  auto li = std::make_shared<LineIndex>();
  li->norders = n_orders(sf);
  int64_t nch = (li->norders + kChunk - 1) / kChunk;
  std::vector<int64_t> cnt(nch);
  parallel_for(nch, hw_threads(nthreads), [&](int64_t a, int64_t b) {
    for (int64_t c = a; c < b; ++c) {
      int64_t s = 0, e = std::min(li->norders, (c + 1) * kChunk);
      for (int64_t i = c * kChunk; i < e; ++i) s += nlines(table, seed, i);
      cnt[c] = s;
    }
  });
  li->chunk_off.assign(nch + 1, 0);
  for (int64_t c = 0; c < nch; ++c) li->chunk_off[c + 1] = li->chunk_off[c] + cnt[c];
  li->nrows = li->chunk_off[nch];
  std::lock_guard<std::mutex> g(g_mu);
  g_cache[key] = li;
  return li;
}

// ---- per-table row writers ----------------------------------------------
struct Out {
  int ncols;
  const int32_t* cols;
  void* const* outs;
  int64_t base;  // row_begin
};
inline void put(const Out& o, int k, int64_t row, int64_t v, int width) {
  int64_t at = row - o.base;
  switch (width) {
    case 1: ((int8_t*)o.outs[k])[at] = (int8_t)v; break;
    case 4: ((int32_t*)o.outs[k])[at] = (int32_t)v; break;
    default: ((int64_t*)o.outs[k])[at] = v; break;
  }
}

const int kW_LO[LO_NCOLS] = {4, 4, 4, 4, 4, 4, 4, 4, 4, 4, 4, 4};
const int kW_D[D_NCOLS] = {4, 4, 4, 4};
const int kW_C[C_NCOLS] = {4, 1, 1, 4};
const int kW_S[S_NCOLS] = {4, 1, 1, 4};
const int kW_P[P_NCOLS] = {4, 1, 1, 4};
const int kW_L[L_NCOLS] = {4, 4, 8, 8, 8, 8, 1, 1, 4, 4, 4, 4, 4, 1, 1};
const int kW_O[O_NCOLS] = {4, 4, 4, 4, 1, 8, 1};
const int kW_TP[TP_NCOLS] = {4, 1, 1, 4};
const int kW_PS[PS_NCOLS] = {4, 4, 8};
const int kW_TC[TC_NCOLS] = {4, 1, 1};
const int kW_TS[TS_NCOLS] = {4, 1};
const int kW_N[N_NCOLS] = {1, 1};
const int kW_R[R_NCOLS] = {1};

const int* widths(int table, int* ncols) {
  switch (table) {
    case HQG_SSB_LINEORDER: *ncols = LO_NCOLS; return kW_LO;
    case HQG_SSB_DATE: *ncols = D_NCOLS; return kW_D;
    case HQG_SSB_CUSTOMER: *ncols = C_NCOLS; return kW_C;
    case HQG_SSB_SUPPLIER: *ncols = S_NCOLS; return kW_S;
    case HQG_SSB_PART: *ncols = P_NCOLS; return kW_P;
    case HQG_TPCH_LINEITEM: *ncols = L_NCOLS; return kW_L;
    case HQG_TPCH_ORDERS: *ncols = O_NCOLS; return kW_O;
    case HQG_TPCH_CUSTOMER: *ncols = TC_NCOLS; return kW_TC;
    case HQG_TPCH_SUPPLIER: *ncols = TS_NCOLS; return kW_TS;
    case HQG_TPCH_NATION: *ncols = N_NCOLS; return kW_N;
    case HQG_TPCH_REGION: *ncols = R_NCOLS; return kW_R;
    case HQG_TPCH_PART: *ncols = TP_NCOLS; return kW_TP;
    case HQG_TPCH_PARTSUPP: *ncols = PS_NCOLS; return kW_PS;
  }
  *ncols = 0;
  return nullptr;
}

// SSB lineorder line (i = order index, j = line index within order)
void lo_line(const Out& o, double sf, uint64_t seed, int64_t i, int j, int64_t row) {
  const int T = HQG_SSB_LINEORDER;
  const uint64_t q = (uint64_t)i * 8 + (uint64_t)j;
  int64_t pk = -1, qty = -1, disc = -1;
  auto partkey = [&] { if (pk < 0) pk = uni(seed, S(T, LO_PARTKEY), q, 1, ssb_parts(sf)); return pk; };
  auto quantity = [&] { if (qty < 0) qty = uni(seed, S(T, LO_QUANTITY), q, 1, 50); return qty; };
  auto discount = [&] { if (disc < 0) disc = uni(seed, S(T, LO_DISCOUNT), q, 0, 10); return disc; };
  for (int k = 0; k < o.ncols; ++k) {
    int64_t v = 0;
    switch (o.cols[k]) {
      case LO_ORDERKEY: v = orderkey(i); break;
      case LO_LINENUMBER: v = j + 1; break;
      case LO_CUSTKEY: v = uni(seed, S(T, LO_CUSTKEY), (uint64_t)i, 1, scaled(30000.0, sf)); break;
      case LO_PARTKEY: v = partkey(); break;
      case LO_SUPPKEY: v = uni(seed, S(T, LO_SUPPKEY), q, 1, scaled(2000.0, sf)); break;
      case LO_ORDERDATE: v = yyyymmdd((int32_t)uni(seed, S(T, LO_ORDERDATE), (uint64_t)i, 0, kSsbDays - 1)); break;
      case LO_QUANTITY: v = quantity(); break;
      case LO_EXTENDEDPRICE: v = quantity() * retailprice(partkey()); break;
      case LO_DISCOUNT: v = discount(); break;
      case LO_REVENUE: v = quantity() * retailprice(partkey()) * (100 - discount()) / 100; break;
      case LO_SUPPLYCOST: v = uni(seed, S(T, LO_SUPPLYCOST), q, 1, 100000); break;
      case LO_TAX: v = uni(seed, S(T, LO_TAX), q, 0, 8); break;
    }
    put(o, k, row, v, 4);
  }
}

// TPC-H lineitem line values (i = order index, j = line index within order);
// the orders' o_totalprice / o_orderstatus are derived from the same values.
struct TLine {
  double sf;
  uint64_t seed;
  int64_t i;
  uint64_t q;
  int64_t odate;
  int64_t pk = -1, qty = -1, ship = -1, rcpt = -1;
  TLine(double sf_, uint64_t seed_, int64_t i_, int j)
      : sf(sf_), seed(seed_), i(i_), q((uint64_t)i_ * 8 + (uint64_t)j),
        odate(uni(seed_, S(HQG_TPCH_ORDERS, O_ORDERDATE), (uint64_t)i_, 0, kTpchODays - 1)) {}
  static const int T = HQG_TPCH_LINEITEM;
  int64_t partkey() { if (pk < 0) pk = uni(seed, S(T, L_PARTKEY), q, 1, scaled(200000.0, sf)); return pk; }
  int64_t quantity() { if (qty < 0) qty = uni(seed, S(T, L_QUANTITY), q, 1, 50); return qty; }
  int64_t shipday() { if (ship < 0) ship = odate + uni(seed, S(T, L_SHIPDATE), q, 1, 121); return ship; }
  int64_t rcptday() { if (rcpt < 0) rcpt = shipday() + uni(seed, S(T, L_RECEIPTDATE), q, 1, 30); return rcpt; }
  int64_t discount() { return uni(seed, S(T, L_DISCOUNT), q, 0, 10); }
  int64_t tax() { return uni(seed, S(T, L_TAX), q, 0, 8); }
  int64_t extendedprice() { return quantity() * (int64_t)retailprice(partkey()); }
  int64_t suppkey() {  // one of the part's four partsupp suppliers (TPC-H 4.2.3)
    const int64_t ns = scaled(10000.0, sf);
    return ps_supplier(partkey(), uni(seed, S(T, L_SUPPKEY), q, 0, 3), ns);
  }
  static int64_t ps_supplier(int64_t pk, int64_t k, int64_t ns) {
    return (pk + k * (ns / 4 + (pk - 1) / ns)) % ns + 1;
  }
};

void l_line(const Out& o, double sf, uint64_t seed, int64_t i, int j, int64_t row) {
  TLine L(sf, seed, i, j);
  const int T = HQG_TPCH_LINEITEM;
  const uint64_t q = L.q;
  for (int k = 0; k < o.ncols; ++k) {
    int64_t v = 0;
    switch (o.cols[k]) {
      case L_ORDERKEY: v = orderkey(i); break;
      case L_PARTKEY: v = L.partkey(); break;
      case L_QUANTITY: v = L.quantity() * 100; break;  // scale 2
      case L_EXTENDEDPRICE: v = L.extendedprice(); break;  // cents
      case L_DISCOUNT: v = L.discount(); break;  // hundredths
      case L_TAX: v = L.tax(); break;            // hundredths
      case L_RETURNFLAG:  // A=0, N=1, R=2 ; spec 4.2.3: R or A if receipt <= CURRENTDATE
        v = L.rcptday() <= kCurrentDay ? (uni(seed, S(T, L_RETURNFLAG), q, 0, 1) ? 2 : 0) : 1;
        break;
      case L_LINESTATUS: v = L.shipday() > kCurrentDay ? 1 : 0; break;  // F=0, O=1
      case L_SHIPDATE: v = yyyymmdd((int32_t)L.shipday()); break;
      case L_RECEIPTDATE: v = yyyymmdd((int32_t)L.rcptday()); break;
      case L_LINENUMBER: v = j + 1; break;
      case L_SUPPKEY: v = L.suppkey(); break;
      case L_COMMITDATE: v = yyyymmdd((int32_t)(L.odate + uni(seed, S(T, L_COMMITDATE), q, 30, 90))); break;
      case L_SHIPMODE: v = uni(seed, S(T, L_SHIPMODE), q, 0, 6); break;
      case L_SHIPINSTRUCT: v = uni(seed, S(T, L_SHIPINSTRUCT), q, 0, 3); break;
    }
    put(o, k, row, v, kW_L[o.cols[k]]);
  }
}

// o_totalprice (cents) and o_orderstatus (F=0, O=1, P=2) of order i from its lines
void order_lines(double sf, uint64_t seed, int64_t i, int64_t* total, int64_t* status) {
  const int n = nlines(HQG_TPCH_LINEITEM, seed, i);
  int64_t t = 0;
  int nopen = 0;
  for (int j = 0; j < n; ++j) {
    TLine L(sf, seed, i, j);
    t += L.extendedprice() * (100 + L.tax()) * (100 - L.discount()) / 10000;
    nopen += L.shipday() > kCurrentDay;
  }
  *total = t;
  *status = nopen == 0 ? 0 : (nopen == n ? 1 : 2);
}

void gen_lines(int table, double sf, uint64_t seed, int64_t a, int64_t b, const Out& o,
               const LineIndex& li) {
  if (a >= b) return;
  // chunk containing row a
  auto it = std::upper_bound(li.chunk_off.begin(), li.chunk_off.end(), a);
  int64_t c = (int64_t)(it - li.chunk_off.begin()) - 1;
  int64_t off = li.chunk_off[c];
  for (int64_t i = c * kChunk; i < li.norders && off < b; ++i) {
    int n = nlines(table, seed, i);
    if (off + n > a) {
      for (int j = 0; j < n; ++j) {
        int64_t row = off + j;
        if (row < a || row >= b) continue;
        if (table == HQG_SSB_LINEORDER) lo_line(o, sf, seed, i, j, row);
        else l_line(o, sf, seed, i, j, row);
      }
    }
    off += n;
  }
}

void gen_dim(int table, double sf, uint64_t seed, int64_t a, int64_t b, const Out& o) {
  for (int64_t r = a; r < b; ++r) {
    for (int k = 0; k < o.ncols; ++k) {
      int c = o.cols[k];
      int64_t v = 0;
      int w = 4;
      switch (table) {
        case HQG_SSB_DATE: {
          int y, m, d;
          civil_from_day((int32_t)r, &y, &m, &d);
          int64_t doy = r - (days_from_civil(y, 1, 1) - kEpoch) + 1;
          if (c == D_DATEKEY) v = y * 10000 + m * 100 + d;
          else if (c == D_YEAR) v = y;
          else if (c == D_YEARMONTHNUM) v = y * 100 + m;
          else v = (doy - 1) / 7 + 1;
          break;
        }
        case HQG_SSB_CUSTOMER:
        case HQG_SSB_SUPPLIER: {
          int nat = (int)uni(seed, S(table, C_NATION), (uint64_t)r, 0, 24);
          if (c == 0) v = r + 1;
          else if (c == 1) { v = nat; w = 1; }
          else if (c == 2) { v = kNationRegion[nat]; w = 1; }
          else v = nat * 10 + uni(seed, S(table, C_CITY), (uint64_t)r, 0, 9);
          break;
        }
        case HQG_SSB_PART: {
          int mfgr = (int)uni(seed, S(table, P_MFGR), (uint64_t)r, 0, 4);
          int cat = mfgr * 5 + (int)uni(seed, S(table, P_CATEGORY), (uint64_t)r, 0, 4);
          if (c == P_PARTKEY) v = r + 1;
          else if (c == P_MFGR) { v = mfgr; w = 1; }
          else if (c == P_CATEGORY) { v = cat; w = 1; }
          else v = cat * 40 + uni(seed, S(table, P_BRAND1), (uint64_t)r, 0, 39);
          break;
        }
        case HQG_TPCH_ORDERS:
          if (c == O_ORDERKEY) v = orderkey(r);
          else if (c == O_CUSTKEY) v = uni(seed, S(table, O_CUSTKEY), (uint64_t)r, 1, scaled(150000.0, sf));
          else if (c == O_ORDERDATE)
            v = yyyymmdd((int32_t)uni(seed, S(table, O_ORDERDATE), (uint64_t)r, 0, kTpchODays - 1));
          else if (c == O_ORDERPRIORITY) { v = uni(seed, S(table, O_ORDERPRIORITY), (uint64_t)r, 0, 4); w = 1; }
          else if (c == O_TOTALPRICE || c == O_ORDERSTATUS) {
            int64_t tot, st;
            order_lines(sf, seed, r, &tot, &st);
            if (c == O_TOTALPRICE) { v = tot; w = 8; } else { v = st; w = 1; }
          } else v = 0;  // o_shippriority
          break;
        case HQG_TPCH_CUSTOMER:
          if (c == TC_CUSTKEY) v = r + 1;
          else if (c == TC_MKTSEGMENT) { v = uni(seed, S(table, TC_MKTSEGMENT), (uint64_t)r, 0, 4); w = 1; }
          else { v = uni(seed, S(table, TC_NATIONKEY), (uint64_t)r, 0, 24); w = 1; }
          break;
        case HQG_TPCH_SUPPLIER:
          if (c == TS_SUPPKEY) v = r + 1;
          else { v = uni(seed, S(table, TS_NATIONKEY), (uint64_t)r, 0, 24); w = 1; }
          break;
        case HQG_TPCH_NATION:
          v = c == N_NATIONKEY ? r : kNationRegion[r];
          w = 1;
          break;
        case HQG_TPCH_REGION:
          v = r;
          w = 1;
          break;
        case HQG_TPCH_PART:
          if (c == TP_PARTKEY) v = r + 1;
          else if (c == TP_BRAND) {  // Brand#MN: M uniform 1..5, N uniform 1..5
            v = uni(seed, S(table, TP_BRAND), (uint64_t)r, 0, 4) * 5 + uni(seed, S(table, 40), (uint64_t)r, 0, 4);
            w = 1;
          } else if (c == TP_CONTAINER) { v = uni(seed, S(table, TP_CONTAINER), (uint64_t)r, 0, 39); w = 1; }
          else v = uni(seed, S(table, TP_SIZE), (uint64_t)r, 1, 50);
          break;
        case HQG_TPCH_PARTSUPP: {
          const int64_t pk = r / 4 + 1;
          if (c == PS_PARTKEY) v = pk;
          else if (c == PS_SUPPKEY) v = TLine::ps_supplier(pk, r % 4, scaled(10000.0, sf));
          else { v = uni(seed, S(table, PS_SUPPLYCOST), (uint64_t)r, 100, 100000); w = 8; }
          break;
        }
      }
      put(o, k, r, v, w);
    }
  }
}

int64_t dim_rows(int table, double sf) {
  switch (table) {
    case HQG_SSB_DATE: return kSsbDays;
    case HQG_SSB_CUSTOMER: return scaled(30000.0, sf);
    case HQG_SSB_SUPPLIER: return scaled(2000.0, sf);
    case HQG_SSB_PART: return ssb_parts(sf);
    case HQG_TPCH_ORDERS: return n_orders(sf);
    case HQG_TPCH_CUSTOMER: return scaled(150000.0, sf);
    case HQG_TPCH_SUPPLIER: return scaled(10000.0, sf);
    case HQG_TPCH_NATION: return 25;
    case HQG_TPCH_REGION: return 5;
    case HQG_TPCH_PART: return scaled(200000.0, sf);
    case HQG_TPCH_PARTSUPP: return 4 * scaled(200000.0, sf);
  }
  return -1;
}

}  // namespace

extern "C" {

int hqg_table_ncols(int table) {
  int n;
  return widths(table, &n) ? n : -1;
}

int hqg_column_width(int table, int col) {
  int n;
  const int* w = widths(table, &n);
  if (!w || col < 0 || col >= n) return -1;
  return w[col];
}

int64_t hqg_table_rows(int table, double sf, uint64_t seed, int nthreads) {
  if (!(sf > 0)) return -1;
  if (table == HQG_SSB_LINEORDER || table == HQG_TPCH_LINEITEM)
    return line_index(table, sf, seed, nthreads)->nrows;
  return dim_rows(table, sf);
}

int hqg_generate(int table, double sf, uint64_t seed, int64_t a, int64_t b, int ncols,
                 const int32_t* cols, void* const* outs, int nthreads) {
  int n;
  if (!widths(table, &n) || !(sf > 0) || a < 0 || b < a || ncols < 0) return -1;
  for (int k = 0; k < ncols; ++k)
    if (cols[k] < 0 || cols[k] >= n || !outs[k]) return -2;
  int64_t total = hqg_table_rows(table, sf, seed, nthreads);
  if (b > total) return -3;
  Out o{ncols, cols, outs, a};
  int nt = hw_threads(nthreads);
  if (table == HQG_SSB_LINEORDER || table == HQG_TPCH_LINEITEM) {
    auto li = line_index(table, sf, seed, nthreads);
    parallel_for(b - a, nt, [&](int64_t x, int64_t y) { gen_lines(table, sf, seed, a + x, a + y, o, *li); });
  } else {
    parallel_for(b - a, nt, [&](int64_t x, int64_t y) { gen_dim(table, sf, seed, a + x, a + y, o); });
  }
  return 0;
}

int32_t hqg_date_from_day(int32_t d) { return yyyymmdd(d); }

int64_t hqg_line_row_of_order(int table, double sf, uint64_t seed, int64_t order, int nthreads) {
  // first line row of order `order` (== nrows for order == norders): the line tables are
  // generated order by order, so [row_of(a), row_of(b)) holds exactly the lines of orders
  // [a, b) -- a range partition of the line table aligned to one of the order table
  if (!(sf > 0) || (table != HQG_SSB_LINEORDER && table != HQG_TPCH_LINEITEM)) return -1;
  auto li = line_index(table, sf, seed, nthreads);
  if (order < 0 || order > li->norders) return -1;
  if (order == li->norders) return li->nrows;
  int64_t c = order / kChunk, off = li->chunk_off[c];
  for (int64_t i = c * kChunk; i < order; ++i) off += nlines(table, seed, i);
  return off;
}

}  // extern "C"
