/*
 * hqgen.h -- deterministic TPC-H / SSB shaped data generator (C ABI).
 *
 * This module is the ONLY thing the oracle (oracle/) and the CUDA path
 * (paper_conf_sigmod_funkebnmt18_b200/) share: it produces the input columns
 * both consume and holds none of the query arithmetic.  Recipe: SURVEY.md
 * §8(d.1); DESIGN.md "Input recipe".
 *
 * Every value is a pure function of (seed, scale factor, table, column, row):
 * a counter-based splitmix64 stream, so any row range can be generated
 * independently (partition invariance) and by any number of threads.
 *
 * Types: keys, dates (yyyymmdd) and SSB measures are int32; TPC-H DECIMAL
 * columns are int64 fixed point with scale 2; strings are order-preserving
 * int8 dictionary codes (dictionaries in hqgen/__init__.py).
 *
 * Errors: functions return 0 on success, a negative value on a bad argument.
 * Ownership: output buffers belong to the caller; the library keeps a small
 * per-(table, sf, seed) cache of order->row offsets, guarded by a mutex.
 */
#ifndef HQGEN_H
#define HQGEN_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

#define HQG_DEFAULT_SEED 20180610ULL

/* tables */
enum {
  HQG_SSB_LINEORDER = 1,
  HQG_SSB_DATE = 2,
  HQG_SSB_CUSTOMER = 3,
  HQG_SSB_SUPPLIER = 4,
  HQG_SSB_PART = 5,
  HQG_TPCH_LINEITEM = 11,
  HQG_TPCH_ORDERS = 12,
  HQG_TPCH_CUSTOMER = 13,
  HQG_TPCH_SUPPLIER = 14,
  HQG_TPCH_NATION = 15,
  HQG_TPCH_REGION = 16,
  HQG_TPCH_PART = 17,
  HQG_TPCH_PARTSUPP = 18
};

/* SSB lineorder columns (all int32) */
enum {
  LO_ORDERKEY = 0, LO_LINENUMBER, LO_CUSTKEY, LO_PARTKEY, LO_SUPPKEY, LO_ORDERDATE,
  LO_QUANTITY, LO_EXTENDEDPRICE, LO_DISCOUNT, LO_REVENUE, LO_SUPPLYCOST, LO_TAX,
  LO_NCOLS
};
/* SSB date (int32) */
enum { D_DATEKEY = 0, D_YEAR, D_YEARMONTHNUM, D_WEEKNUMINYEAR, D_NCOLS };
/* SSB customer: custkey i32, nation i8, region i8, city i32 */
enum { C_CUSTKEY = 0, C_NATION, C_REGION, C_CITY, C_NCOLS };
/* SSB supplier: suppkey i32, nation i8, region i8, city i32 */
enum { S_SUPPKEY = 0, S_NATION, S_REGION, S_CITY, S_NCOLS };
/* SSB part: partkey i32, mfgr i8, category i8, brand1 i32 */
enum { P_PARTKEY = 0, P_MFGR, P_CATEGORY, P_BRAND1, P_NCOLS };
/* TPC-H lineitem */
enum {
  L_ORDERKEY = 0, L_PARTKEY, L_QUANTITY, L_EXTENDEDPRICE, L_DISCOUNT, L_TAX,
  L_RETURNFLAG, L_LINESTATUS, L_SHIPDATE, L_RECEIPTDATE, L_LINENUMBER, L_SUPPKEY,
  L_COMMITDATE,   /* i32 yyyymmdd: o_orderdate + U[30, 90] (TPC-H 4.2.3) */
  L_SHIPMODE,     /* i8 code of AIR, FOB, MAIL, RAIL, REG AIR, SHIP, TRUCK (uniform) */
  L_SHIPINSTRUCT, /* i8 code of COLLECT COD, DELIVER IN PERSON, NONE, TAKE BACK RETURN (uniform) */
  L_NCOLS
};
/* TPC-H orders */
enum {
  O_ORDERKEY = 0, O_CUSTKEY, O_ORDERDATE, O_SHIPPRIORITY,
  O_ORDERPRIORITY, /* i8 code of 1-URGENT .. 5-LOW (uniform) */
  O_TOTALPRICE,    /* i64 cents: sum over the order's lines of l_extendedprice*(100+l_tax)*(100-l_discount)/10^4 */
  O_ORDERSTATUS,   /* i8 code of F, O, P: all lines F / all lines O / mixed (TPC-H 4.2.3) */
  O_NCOLS
};
/* TPC-H customer */
enum { TC_CUSTKEY = 0, TC_MKTSEGMENT, TC_NATIONKEY, TC_NCOLS };
/* TPC-H supplier (10 K * SF rows): suppkey i32, nationkey i8 (uniform over the 25 nations) */
enum { TS_SUPPKEY = 0, TS_NATIONKEY, TS_NCOLS };
/* TPC-H nation (25 rows): nationkey i8 = the name's dictionary code, regionkey i8 */
enum { N_NATIONKEY = 0, N_REGIONKEY, N_NCOLS };
/* TPC-H region (5 rows): regionkey i8 = the name's dictionary code */
enum { R_REGIONKEY = 0, R_NCOLS };
/* TPC-H part (200 K * SF rows): partkey i32, brand i8 ('Brand#MN' = (M-1)*5 + N-1, M, N in 1..5),
 * container i8 (code of the 40 'SIZE TYPE' strings in string order), size i32 (1..50) */
enum { TP_PARTKEY = 0, TP_BRAND, TP_CONTAINER, TP_SIZE, TP_NCOLS };
/* TPC-H partsupp (4 rows per part): partkey i32, suppkey i32 (TPC-H 4.2.3: the part's
 * i-th supplier (partkey + i*(S/4 + (partkey-1)/S)) mod S + 1), supplycost i64 cents 100..100000.
 * l_suppkey is one of its l_partkey's four suppliers, chosen uniformly. */
enum { PS_PARTKEY = 0, PS_SUPPKEY, PS_SUPPLYCOST, PS_NCOLS };

/* Number of rows of a table at scale factor sf (lineorder/lineitem count
 * the 1..7 lines of every order, computed once and cached). <0 on error. */
int64_t hqg_table_rows(int table, double sf, uint64_t seed, int nthreads);
/* Byte width of a column (1, 4 or 8); <0 on error. */
int hqg_column_width(int table, int col);
/* Number of columns of a table; <0 on error. */
int hqg_table_ncols(int table);
/* Generate rows [row_begin, row_end) of the given columns into outs[i]
 * (outs[i] must hold (row_end-row_begin)*width bytes).  nthreads<=0 means
 * hardware concurrency. */
int hqg_generate(int table, double sf, uint64_t seed, int64_t row_begin, int64_t row_end,
                 int ncols, const int32_t* cols, void* const* outs, int nthreads);
/* yyyymmdd of day d counted from 1992-01-01 (d=0). */
int32_t hqg_date_from_day(int32_t d);

/* First row of the lines of order `order` in a line table (SSB lineorder / TPC-H
 * lineitem; order == number of orders gives the row count).  The line tables are
 * generated order by order, so rows [row_of(a), row_of(b)) hold exactly the lines of
 * orders [a, b): a partition of the line table co-aligned with one of the order
 * table (multi-GPU co-partitioning by orderkey).  -1 on a bad table / sf / order. */
int64_t hqg_line_row_of_order(int table, double sf, uint64_t seed, int64_t order, int nthreads);

#ifdef __cplusplus
}
#endif
#endif
