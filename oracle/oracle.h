/*
 * oracle.h -- TEST INFRASTRUCTURE ONLY.  A plain, slow, tuple-at-a-time CPU
 * implementation of the SQL results the fused pipeline computes.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load or call this library.  It shares no code,
 * header, helper or constant with the CUDA path (paper_conf_sigmod_funkebnmt18_b200);
 * the only shared module is the input generator hqgen/.
 *
 * What it computes: HorseQC computes exactly the
 * relational result (§5-§6); the only relaxation is the
 * order of materialised rows.  So every function here
 * is the plain SQL definition of one query written out: dimension predicates
 * + std::unordered_map (or nested loops in brute-force mode) for joins, the
 * fact predicates in SQL order, exact integer arithmetic in __int128 with an
 * int64 range check, std::map for GROUP BY, std::sort for ORDER BY.
 *
 * Conventions: every function returns 0 on success; on a duplicate build key
 * -4, on int64 overflow of a result -6, on bad arguments -1.  Results are
 * column-major int64 (icol) and double (fcol) arrays allocated with malloc
 * and released with orc_free.  `nthreads` > 1 splits the fact table into
 * contiguous ranges whose integer partial aggregates are merged exactly
 * (SURVEY.md §8(c.2) step 6).  `brute` != 0 replaces the hash joins with
 * nested loops over the dimension arrays (step 5).
 */
#ifndef HQ_ORACLE_H
#define HQ_ORACLE_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

typedef struct {
  int64_t nrows;      /* rows of the full (pre-LIMIT) result */
  int32_t ni, nf;     /* number of int64 / double columns */
  int64_t* icol;      /* ni * nrows, column-major */
  double* fcol;       /* nf * nrows, column-major */
  int64_t qualifying; /* rows that reached the sink (COUNT(*)) */
} orc_result;

/* SSB lineorder (int32 columns; NULL for columns a query does not read) */
typedef struct {
  int64_t n;
  const int32_t *orderkey, *custkey, *partkey, *suppkey, *orderdate, *quantity,
      *extendedprice, *discount, *revenue, *supplycost, *tax;
} orc_lineorder;
typedef struct { int64_t n; const int32_t *datekey, *year, *yearmonthnum, *weeknuminyear; } orc_date;
/* SSB customer or supplier */
typedef struct { int64_t n; const int32_t* key; const int8_t *nation, *region; const int32_t* city; } orc_ssb_dim;
typedef struct { int64_t n; const int32_t* partkey; const int8_t *mfgr, *category; const int32_t* brand1; } orc_part;
/* TPC-H lineitem: DECIMALs are int64 fixed point, scale 2 */
typedef struct {
  int64_t n;
  const int32_t* orderkey;
  const int64_t *quantity, *extendedprice, *discount, *tax;
  const int8_t *returnflag, *linestatus;
  const int32_t* shipdate;
  const int32_t* suppkey;
  const int32_t *partkey, *commitdate, *receiptdate;
  const int8_t *shipmode, *shipinstruct;
} orc_lineitem;
typedef struct {
  int64_t n;
  const int32_t *orderkey, *custkey, *orderdate, *shippriority;
  const int8_t* orderpriority;
  const int64_t* totalprice;
  const int8_t* orderstatus;
} orc_orders;
/* TPC-H partsupp (4 rows per part): supplycost int64 cents */
typedef struct { int64_t n; const int32_t *partkey, *suppkey; const int64_t* supplycost; } orc_partsupp;
/* TPC-H part: brand 'Brand#MN' = (M-1)*5 + N-1; container = code in string order (hqgen) */
typedef struct { int64_t n; const int32_t* partkey; const int8_t *brand, *container; const int32_t* size; } orc_tpch_part;
typedef struct { int64_t n; const int32_t* custkey; const int8_t *mktsegment, *nationkey; } orc_tpch_customer;
typedef struct { int64_t n; const int32_t* suppkey; const int8_t* nationkey; } orc_tpch_supplier;
typedef struct { int64_t n; const int8_t *nationkey, *regionkey; } orc_nation;
typedef struct { int64_t n; const int8_t* regionkey; } orc_region;

/* TPC-H Q6 -> 1 row: [revenue (scale 4), count] */
int orc_tpch_q6(const orc_lineitem* li, int nthreads, orc_result* out);
/* TPC-H Q1 -> rows [rf, ls, sum_qty, sum_base_price, sum_disc_price(s4), sum_charge(s6), count]
 *            + f [avg_qty, avg_price, avg_disc], ORDER BY rf, ls */
int orc_tpch_q1(const orc_lineitem* li, int nthreads, orc_result* out);
/* SSB Q1.1 / Q1.2 / Q1.3 (variant 1..3) -> 1 row: [revenue, count] */
int orc_ssb_q1(int variant, const orc_lineorder* lo, const orc_date* d, int brute, int nthreads,
               orc_result* out);
/* SSB Q3.1 (Fig 23) -> rows [c_nation, s_nation, d_year, revenue, count]
 * ORDER BY d_year asc, revenue desc, c_nation, s_nation */
int orc_ssb_q31(const orc_lineorder* lo, const orc_ssb_dim* c, const orc_ssb_dim* s,
                const orc_date* d, int brute, int nthreads, orc_result* out);
/* SSB Q3.1 materialised join result -> rows [c_nation, s_nation, d_year, lo_revenue],
 * sorted lexicographically (a multiset: P:1203-1210) */
int orc_ssb_q31_mat(const orc_lineorder* lo, const orc_ssb_dim* c, const orc_ssb_dim* s,
                    const orc_date* d, int brute, int nthreads, orc_result* out);
/* SSB Q4.1 -> rows [d_year, c_nation, profit, count], ORDER BY d_year, c_nation */
int orc_ssb_q41(const orc_lineorder* lo, const orc_date* d, const orc_ssb_dim* c,
                const orc_ssb_dim* s, const orc_part* p, int brute, int nthreads, orc_result* out);
/* SSB flight 2 (variant 1..3: Q2.1 p_category = 'MFGR#12', s_region = 'AMERICA'; Q2.2 p_brand1
 * BETWEEN 'MFGR#2221' AND 'MFGR#2228', s_region = 'ASIA'; Q2.3 p_brand1 = 'MFGR#2239',
 * s_region = 'EUROPE') -> rows [d_year, p_brand1, revenue, count] ORDER BY d_year, p_brand1 */
int orc_ssb_q2(int variant, const orc_lineorder* lo, const orc_date* d, const orc_part* p,
               const orc_ssb_dim* s, int brute, int nthreads, orc_result* out);
/* SSB flight 3 (variant 2..4: Q3.2 c_nation = s_nation = 'UNITED STATES', d_year 1992..1997;
 * Q3.3 c_city, s_city IN ('UNITED KI1', 'UNITED KI5'), d_year 1992..1997; Q3.4 the same cities,
 * d_yearmonth = 'Dec1997') -> rows [c_city, s_city, d_year, revenue, count]
 * ORDER BY d_year asc, revenue desc, c_city, s_city */
int orc_ssb_q3(int variant, const orc_lineorder* lo, const orc_ssb_dim* c, const orc_ssb_dim* s,
               const orc_date* d, int brute, int nthreads, orc_result* out);
/* SSB flight 4 (variant 2..3): Q4.2 c_region = s_region = 'AMERICA', d_year IN (1997, 1998),
 * p_mfgr IN ('MFGR#1', 'MFGR#2') -> rows [d_year, s_nation, p_category, profit, count];
 * Q4.3 c_region = 'AMERICA', s_nation = 'UNITED STATES', d_year IN (1997, 1998),
 * p_category = 'MFGR#14' -> rows [d_year, s_city, p_brand1, profit, count]; ORDER BY the keys */
int orc_ssb_q4(int variant, const orc_lineorder* lo, const orc_date* d, const orc_ssb_dim* c,
               const orc_ssb_dim* s, const orc_part* p, int brute, int nthreads, orc_result* out);
/* TPC-H Q3 -> rows [l_orderkey, revenue(s4), o_orderdate, o_shippriority, count],
 * ORDER BY revenue desc, o_orderdate asc, l_orderkey asc (full result; caller applies LIMIT 10) */
int orc_tpch_q3(const orc_tpch_customer* c, const orc_orders* o, const orc_lineitem* li, int brute,
                int nthreads, orc_result* out);
/* TPC-H Q5 (region 'ASIA', order year 1994) -> rows [n_name (nation code), revenue (scale 4),
 * count] ORDER BY revenue desc, n_name */
int orc_tpch_q5(const orc_tpch_customer* c, const orc_orders* o, const orc_lineitem* li,
                const orc_tpch_supplier* s, const orc_nation* n, const orc_region* r, int brute, int nthreads,
                orc_result* out);
/* TPC-H Q10 (returned items; order quarter 1993-10-01 .. 1993-12-31, l_returnflag = 'R') ->
 * rows [c_custkey, n_name, revenue (scale 4), count] ORDER BY revenue desc, c_custkey (full
 * result; the caller applies LIMIT 20).  c_name, c_acctbal, c_phone, c_address, c_comment are
 * functionally dependent on c_custkey and not generated (R18). */
int orc_tpch_q10(const orc_tpch_customer* c, const orc_orders* o, const orc_lineitem* li, const orc_nation* n,
                 int brute, int nthreads, orc_result* out);
/* TPC-H Q7 (volume shipping between FRANCE and GERMANY, ship years 1995-1996) ->
 * rows [supp_nation, cust_nation, l_year, revenue (scale 4), count]
 * ORDER BY supp_nation, cust_nation, l_year (n_name = the nation's code, R18) */
int orc_tpch_q7(const orc_tpch_customer* c, const orc_orders* o, const orc_lineitem* li,
                const orc_tpch_supplier* s, const orc_nation* n, int brute, int nthreads, orc_result* out);
/* PAPER.md Fig 16 "Query 1": revenue = lo_extendedprice*lo_discount+lo_tax
 * where lo_quantity between 25-x and 25+x -> rows [revenue] sorted (a multiset) */
int orc_micro_select(const orc_lineorder* lo, int32_t x, int nthreads, orc_result* out);
/* App G.1: sum(revenue) of the same selection -> 1 row [sum, count] */
int orc_micro_sum(const orc_lineorder* lo, int32_t x, int nthreads, orc_result* out);
/* Fig 26: select sum(lo_extendedprice), lo_orderkey % x group by lo_orderkey % x
 * -> rows [lo_orderkey % x, sum, count] ORDER BY key */
int orc_micro_groupby(const orc_lineorder* lo, int32_t x, int nthreads, orc_result* out);

/* TPC-H Q4 (order priority checking) -> rows [o_orderpriority, order_count] ORDER BY
 * o_orderpriority; qualifying = orders counted */
int orc_tpch_q4(const orc_orders* o, const orc_lineitem* li, int brute, int nthreads, orc_result* out);
/* TPC-H Q13 without the o_comment LIKE (App F) -> rows [c_count,
 * custdist] ORDER BY custdist desc, c_count desc; qualifying = customers */
int orc_tpch_q13(const orc_tpch_customer* c, const orc_orders* o, int brute, orc_result* out);
/* TPC-H Q17, the correlated subquery unnested (App F) -> 1 row [sum_extendedprice
 * (cents), count]; avg_yearly = sum_extendedprice / 7.0 (R19) */
int orc_tpch_q17(const orc_tpch_part* p, const orc_lineitem* li, int brute, orc_result* out);
/* TPC-H Q18 (large volume customer) -> rows [c_custkey, o_orderkey, o_orderdate, o_totalprice,
 * sum_qty (scale 2), count] ORDER BY o_totalprice desc, o_orderdate, o_orderkey (full result;
 * the caller applies LIMIT 100); c_name depends on c_custkey (R18) */
int orc_tpch_q18(const orc_tpch_customer* c, const orc_orders* o, const orc_lineitem* li, int brute,
                 orc_result* out);
/* TPC-H Q19 (discounted revenue) -> 1 row [revenue (scale 4), count] */
int orc_tpch_q19(const orc_tpch_part* p, const orc_lineitem* li, int brute, int nthreads, orc_result* out);
/* TPC-H Q21 (suppliers who kept orders waiting; variant 0: the TPC-H text, the third
 * subquery NOT EXISTS; variant 1: PAPER.md App F's EXISTS) -> rows
 * [s_suppkey, numwait] ORDER BY numwait desc, s_suppkey (s_name depends on s_suppkey, R18) */
int orc_tpch_q21(int variant, const orc_tpch_supplier* s, const orc_orders* o, const orc_lineitem* li,
                 const orc_nation* n, int brute, orc_result* out);

/* TPC-H Q9 (product type profit) with PAPER.md App F's rewrite of p_name like '%green%' as a
 * filter on p_partkey (R19: p_partkey <= pmax) -> rows [nation, o_year,
 * sum_profit (scale 4), count] ORDER BY nation, o_year desc */
int orc_tpch_q9(const orc_tpch_part* p, const orc_tpch_supplier* s, const orc_lineitem* li, const orc_partsupp* ps,
                const orc_orders* o, const orc_nation* n, int32_t pmax, int brute, int nthreads, orc_result* out);

void orc_free(orc_result* r);

#ifdef __cplusplus
}
#endif
#endif
