"""Plan builders for the benchmark queries.

Each query is written as its fusion operators: hash builds (pipeline breakers,
filtered dimension scans) followed by ONE probe pipeline over the fact table
(the compound kernel), exactly as PAPER.md §4.1/§7 describes a plan with
explicit fusion operators.  Constants are the SQL
constants folded to the storage encoding (readings R2, R4, R5):
decimals in hundredths, dates as yyyymmdd, strings as order-preserving
dictionary codes from ``hqgen``.

Predicate/probe order inside a pipeline is result-invariant (R14):
cheap and selective first.
"""
from __future__ import annotations

from typing import Callable, Dict, List, Optional

import hqgen

from . import hq
from .engine import Engine, PlanBuilder, QueryResult, fetch

ASIA = hqgen.code(hqgen.REGIONS, "ASIA")
AMERICA = hqgen.code(hqgen.REGIONS, "AMERICA")
BUILDING = hqgen.code(hqgen.MKTSEGMENTS, "BUILDING")
MFGR1 = hqgen.code(hqgen.MFGRS, "MFGR#1")
MFGR2 = hqgen.code(hqgen.MFGRS, "MFGR#2")
EUROPE = hqgen.code(hqgen.REGIONS, "EUROPE")
UNITED_STATES = hqgen.code(hqgen.NATIONS, "UNITED STATES")
UNITED_KI1, UNITED_KI5 = hqgen.city_code("UNITED KI1"), hqgen.city_code("UNITED KI5")


class Query:
    """A query: fact table, referenced columns per table, and run(E) which
    builds the hash tables and returns (final Result, final PlanBuilder)."""

    def __init__(self, name: str, bench: str, fact: str, columns: Dict[str, List[str]], run: Callable,
                 copart: Optional[str] = None):
        self.name, self.bench, self.fact, self.columns, self._run = name, bench, fact, columns, run
        # copart: the order table partitioned together with the fact (line) table by order
        # for multi-GPU runs (hqgen.copartition; the final GROUP BY contains the orderkey)
        self.copart = copart

    def run(self, E: Engine, **kw):
        return self._run(E, **kw)

    def execute(self, E: Engine, **kw) -> QueryResult:
        res, pb = self._run(E, **kw)
        return fetch(res, pb.result_names)

    def fact_bytes_per_row(self) -> int:
        """Algorithmic bytes per fact row: widths of the referenced fact columns."""
        schema = dict(hqgen.SCHEMAS[hqgen.TABLE_NAMES[self.fact]])
        return sum(int(schema[c][1]) for c in self.columns[self.fact])


# ---------------------------------------------------------------- TPC-H Q6
def _tpch_q6(E: Engine, **_):
    pb = E.plan("lineitem")
    pb.filter("l_shipdate", "between", 19940101, 19950101 - 1)  # >= 1994-01-01 and < 1995-01-01
    pb.filter("l_discount", "between", 5, 7)                     # 0.06 +- 0.01 in hundredths
    pb.filter("l_quantity", "<", 2400)                           # < 24 in hundredths
    pb.compute("rev", [("load", "l_extendedprice"), ("mul", "l_discount")])  # scale 4
    pb.aggregate(aggs=[("sum", "rev"), ("count", None)], agg_names=["revenue", "count"])
    return E.run(pb), pb


# ---------------------------------------------------------------- TPC-H Q1
def _tpch_q1(E: Engine, **_):
    pb = E.plan("lineitem")
    pb.filter("l_shipdate", "<=", 19980902)  # 1998-12-01 - 90 days
    pb.compute("disc_price", [("load", "l_discount"), ("rsub", 100), ("mul", "l_extendedprice")])  # scale 4
    pb.compute("charge", [("load", "l_tax"), ("add", 100), ("mul", "disc_price")])                 # scale 6
    pb.aggregate(keys=[("l_returnflag", 0, 3), ("l_linestatus", 0, 2)],
                 aggs=[("sum", "l_quantity"), ("sum", "l_extendedprice"), ("sum", "disc_price"),
                       ("sum", "charge"), ("avg", "l_quantity", 2), ("avg", "l_extendedprice", 2),
                       ("avg", "l_discount", 2), ("count", None)],
                 agg_names=["sum_qty", "sum_base_price", "sum_disc_price", "sum_charge", "avg_qty",
                            "avg_price", "avg_disc", "count_order"])
    return E.run(pb), pb


# ---------------------------------------------------------------- SSB Q1.x
_Q1X = {
    1: ([("d_year", "=", 1993)], ("lo_quantity", "<", 25, 0), (1, 3)),
    2: ([("d_yearmonthnum", "=", 199401)], ("lo_quantity", "between", 26, 35), (4, 6)),
    3: ([("d_weeknuminyear", "=", 6), ("d_year", "=", 1994)], ("lo_quantity", "between", 26, 35), (5, 7)),
}


def _ssb_q1(v: int):
    def run(E: Engine, **_):
        dpreds, qf, (dlo, dhi) = _Q1X[v]
        hd = E.hash("date", "d_datekey", preds=dpreds)  # semi-join table of qualifying dates
        pb = E.plan("lineorder")
        pb.filter(qf[0], qf[1], qf[2], qf[3])
        pb.filter("lo_discount", "between", dlo, dhi)
        pb.probe(hd, "lo_orderdate", "semi")
        pb.compute("rev", [("load", "lo_extendedprice"), ("mul", "lo_discount")])
        pb.aggregate(aggs=[("sum", "rev"), ("count", None)], agg_names=["revenue", "count"])
        return E.run(pb), pb
    return run


# ---------------------------------------------------------------- SSB Q3.1
def _ssb_q31_probes(E: Engine, porder: str = "scd") -> PlanBuilder:
    hc, hs, hd = E.hashes([
        dict(table="customer", key="c_custkey", payload=["c_nation"], preds=[("c_region", "=", ASIA)]),
        dict(table="supplier", key="s_suppkey", payload=["s_nation"], preds=[("s_region", "=", ASIA)]),
        dict(table="date", key="d_datekey", payload=["d_year"], preds=[("d_year", "between", 1992, 1997)])])
    pb = E.plan("lineorder")
    probes = {"s": (hs, "lo_suppkey", ["s_nation"]), "c": (hc, "lo_custkey", ["c_nation"]),
              "d": (hd, "lo_orderdate", ["d_year"])}
    for k in porder:  # probe order (result-invariant, R14)
        h, key, pay = probes[k]
        pb.probe(h, key, "inner", pay)
    return pb


def _ssb_q31(E: Engine, porder: str = "scd", **_):
    pb = _ssb_q31_probes(E, porder)
    pb.aggregate(keys=[("c_nation", 0, 25), ("s_nation", 0, 25), ("d_year", 1992, 7)],
                 aggs=[("sum", "lo_revenue"), ("count", None)],
                 order=[("d_year", False), ("revenue", True)], agg_names=["revenue", "count"])
    return E.run(pb), pb


def _ssb_q31_mat(E: Engine, capacity: int = 0, **_):
    pb = _ssb_q31_probes(E)
    pb.materialise([("c_nation", "i32"), ("s_nation", "i32"), ("d_year", "i32"), ("lo_revenue", "i32")],
                   capacity=capacity)
    return E.run(pb), pb


# ---------------------------------------------------------------- SSB Q4.1
def _ssb_q41(E: Engine, **_):
    hs, hc, hp, hd = E.hashes([
        dict(table="supplier", key="s_suppkey", preds=[("s_region", "=", AMERICA)]),
        dict(table="customer", key="c_custkey", payload=["c_nation"], preds=[("c_region", "=", AMERICA)]),
        dict(table="part", key="p_partkey", preds=[("p_mfgr", "in", [MFGR1, MFGR2])]),
        dict(table="date", key="d_datekey", payload=["d_year"])])
    pb = E.plan("lineorder")
    pb.probe(hs, "lo_suppkey", "semi")
    pb.probe(hc, "lo_custkey", "inner", ["c_nation"])
    pb.probe(hp, "lo_partkey", "semi")
    pb.probe(hd, "lo_orderdate", "inner", ["d_year"])
    pb.compute("profit", [("load", "lo_revenue"), ("sub", "lo_supplycost")])
    pb.aggregate(keys=[("d_year", 1992, 7), ("c_nation", 0, 25)],
                 aggs=[("sum", "profit"), ("count", None)], agg_names=["profit", "count"])
    return E.run(pb), pb


# ------------------------------------------------------- SSB flight 2
# select sum(lo_revenue), d_year, p_brand1 from lineorder, date, part, supplier
# where <joins> and <part predicate> and s_region = <r> group by d_year, p_brand1
# order by d_year, p_brand1
_Q2X = {
    1: ([("p_category", "=", hqgen.category_code("MFGR#12"))], AMERICA),
    2: ([("p_brand1", "between", hqgen.brand_code("MFGR#2221"), hqgen.brand_code("MFGR#2228"))],
        hqgen.code(hqgen.REGIONS, "ASIA")),
    3: ([("p_brand1", "=", hqgen.brand_code("MFGR#2239"))], EUROPE),
}


def _ssb_q2(v: int):
    def run(E: Engine, **_):
        ppreds, region = _Q2X[v]
        hp, hs, hd = E.hashes([
            dict(table="part", key="p_partkey", payload=["p_brand1"], preds=ppreds),
            dict(table="supplier", key="s_suppkey", preds=[("s_region", "=", region)]),
            dict(table="date", key="d_datekey", payload=["d_year"])])
        pb = E.plan("lineorder")
        pb.probe(hs, "lo_suppkey", "semi")                  # 1/5, a bitmap staged in shared memory
        pb.probe(hp, "lo_partkey", "inner", ["p_brand1"])   # 1/25 .. 1/1000, a byte map in L2
        pb.probe(hd, "lo_orderdate", "inner", ["d_year"])
        pb.aggregate(keys=[("d_year", 1992, 7), ("p_brand1", 0, 1000)],
                     aggs=[("sum", "lo_revenue"), ("count", None)], agg_names=["revenue", "count"])
        return E.run(pb), pb
    return run


# ------------------------------------------------------- SSB flight 3 (Q3.2-Q3.4)
# select c_city, s_city, d_year, sum(lo_revenue) as revenue from customer, lineorder,
# supplier, date where <joins> and <customer, supplier, date predicates>
# group by c_city, s_city, d_year order by d_year asc, revenue desc
_CITIES = ("in", [UNITED_KI1, UNITED_KI5])
_Q3X = {
    2: ([("c_nation", "=", UNITED_STATES)], [("s_nation", "=", UNITED_STATES)], [("d_year", "between", 1992, 1997)]),
    3: ([("c_city",) + _CITIES], [("s_city",) + _CITIES], [("d_year", "between", 1992, 1997)]),
    4: ([("c_city",) + _CITIES], [("s_city",) + _CITIES], [("d_yearmonthnum", "=", 199712)]),  # 'Dec1997'
}


def _ssb_q3(v: int):
    def run(E: Engine, **_):
        cpreds, spreds, dpreds = _Q3X[v]
        hc, hs, hd = E.hashes([
            dict(table="customer", key="c_custkey", payload=["c_city"], preds=cpreds),
            dict(table="supplier", key="s_suppkey", payload=["s_city"], preds=spreds),
            dict(table="date", key="d_datekey", payload=["d_year"], preds=dpreds)])
        pb = E.plan("lineorder")
        pb.probe(hs, "lo_suppkey", "inner", ["s_city"])
        pb.probe(hc, "lo_custkey", "inner", ["c_city"])
        pb.probe(hd, "lo_orderdate", "inner", ["d_year"])
        pb.aggregate(keys=[("c_city", 0, 250), ("s_city", 0, 250), ("d_year", 1992, 7)],
                     aggs=[("sum", "lo_revenue"), ("count", None)],
                     order=[("d_year", False), ("revenue", True)], agg_names=["revenue", "count"],
                     group_capacity=4096)  # declared 437,500 city pairs x years; <= 600 occur
        return E.run(pb), pb
    return run


# ------------------------------------------------------- SSB flight 4 (Q4.2, Q4.3)
# select d_year, <s_nation | s_city>, <p_category | p_brand1>, sum(lo_revenue - lo_supplycost)
# from date, customer, supplier, part, lineorder where <joins> and c_region = 'AMERICA'
# and <supplier predicate> and d_year in (1997, 1998) and <part predicate>
# group by / order by the three keys
def _ssb_q4(v: int):
    def run(E: Engine, **_):
        if v == 2:
            sdesc = dict(table="supplier", key="s_suppkey", payload=["s_nation"], preds=[("s_region", "=", AMERICA)])
            pdesc = dict(table="part", key="p_partkey", payload=["p_category"], preds=[("p_mfgr", "in", [MFGR1, MFGR2])])
            skey, pkey = ("s_nation", 0, 25), ("p_category", 0, 25)
        else:
            sdesc = dict(table="supplier", key="s_suppkey", payload=["s_city"], preds=[("s_nation", "=", UNITED_STATES)])
            pdesc = dict(table="part", key="p_partkey", payload=["p_brand1"],
                         preds=[("p_category", "=", hqgen.category_code("MFGR#14"))])
            skey, pkey = ("s_city", 0, 250), ("p_brand1", 0, 1000)
        hc, hs, hp, hd = E.hashes([
            dict(table="customer", key="c_custkey", preds=[("c_region", "=", AMERICA)]), sdesc, pdesc,
            dict(table="date", key="d_datekey", payload=["d_year"],
                 preds=[("d_year", "between", 1997, 1998)])])  # d_year = 1997 or d_year = 1998
        pb = E.plan("lineorder")
        pb.probe(hd, "lo_orderdate", "inner", ["d_year"])   # 2/7
        pb.probe(hs, "lo_suppkey", "inner", [skey[0]])        # 1/5 or 1/25
        pb.probe(hc, "lo_custkey", "semi")                    # 1/5
        pb.probe(hp, "lo_partkey", "inner", [pkey[0]])        # 2/5 or 1/25
        pb.compute("profit", [("load", "lo_revenue"), ("sub", "lo_supplycost")])
        pb.aggregate(keys=[("d_year", 1992, 7), skey, pkey],
                     aggs=[("sum", "profit"), ("count", None)], agg_names=["profit", "count"],
                     group_capacity=4096)  # Q4.3: declared 1.75 M keys, <= 800 occur
        return E.run(pb), pb
    return run


# ---------------------------------------------------------------- TPC-H Q3
def _tpch_q3(E: Engine, limit: int = 10, **_):
    # pipeline 1: customer filter -> build (semi)
    hc = E.hash("tpch_customer", "c_custkey", preds=[("c_mktsegment", "=", BUILDING)])
    # pipeline 2: orders filter -> probe customer -> materialise -> build
    ro = None
    if E.builds_here:  # build side: only the root of a DistributedEngine holds the dimensions
        po = E.plan("orders")
        po.filter("o_orderdate", "<", 19950315)
        po.probe(hc, "o_custkey", "semi")
        po.materialise([("o_orderkey", "i32"), ("o_orderdate", "i32"), ("o_shippriority", "i32")])
        ro = E.run(po, partitioned=False)
    ho = E.hash_from(ro, ["o_orderkey", "o_orderdate", "o_shippriority"], "o_orderkey",
                     ["o_orderdate", "o_shippriority"])
    nk = max(int(ho.meta().nkeys), 0)
    # pipeline 3: lineitem filter -> probe orders -> group by orderkey
    pl = E.plan("lineitem")
    pl.filter("l_shipdate", ">", 19950315)
    pl.probe(ho, "l_orderkey", "inner", ["o_orderdate", "o_shippriority"])
    pl.compute("rev", [("load", "l_discount"), ("rsub", 100), ("mul", "l_extendedprice")])  # scale 4
    pl.aggregate(keys=[("l_orderkey", 0, 1 << 31), ("o_orderdate", 19920101, 70000), ("o_shippriority", 0, 8)],
                 aggs=[("sum", "rev"), ("count", None)],
                 order=[("revenue", True), ("o_orderdate", False)], limit=limit,
                 # expected groups: the qualifying orders with a line shipped after the date,
                 # ~8 % of them on the synthetic data (libhq sizes the table at 2x, power of two;
                 # an underestimate costs one re-run with a larger table, never a wrong row)
                 group_capacity=max(1024, nk // 12), agg_names=["revenue", "count"])
    res = E.run(pl)
    pl.keep += [ro, ho]
    return res, pl


# ---------------------------------------------------------------- TPC-H Q5
# select n_name, sum(l_extendedprice * (1 - l_discount)) as revenue
# from customer, orders, lineitem, supplier, nation, region
# where c_custkey = o_custkey and l_orderkey = o_orderkey and l_suppkey = s_suppkey
#   and c_nationkey = s_nationkey and s_nationkey = n_nationkey and n_regionkey = r_regionkey
#   and r_name = 'ASIA' and o_orderdate >= '1994-01-01' and o_orderdate < '1995-01-01'
# group by n_name order by revenue desc
def _tpch_q5(E: Engine, **_):
    asia = hqgen.code(hqgen.REGIONS, "ASIA")  # r_name = 'ASIA' (region key = its name's code)
    # pipeline 1: region filter -> build; pipeline 2: nation -> probe region -> materialise -> build
    hr = E.hash("region", "r_regionkey", preds=[("r_regionkey", "=", asia)])
    hc, hs = E.hashes([dict(table="tpch_customer", key="c_custkey", payload=["c_nationkey"]),
                       dict(table="tpch_supplier", key="s_suppkey", payload=["s_nationkey"])])
    rn = ro = None
    if E.builds_here:  # build side: only the root of a DistributedEngine holds the dimensions
        pn = E.plan("nation")
        pn.probe(hr, "n_regionkey", "semi")
        pn.materialise([("n_nationkey", "i32")])
        rn = E.run(pn, partitioned=False)
        # pipeline 3: orders filter -> probe customer -> materialise -> build
        po = E.plan("orders")
        po.filter("o_orderdate", "between", 19940101, 19950101 - 1)
        po.probe(hc, "o_custkey", "inner", ["c_nationkey"])
        po.materialise([("o_orderkey", "i32"), ("c_nationkey", "i32")])
        ro = E.run(po, partitioned=False)
    hn = E.hash_from(rn, ["n_nationkey"], "n_nationkey")
    ho = E.hash_from(ro, ["o_orderkey", "c_nationkey"], "o_orderkey", ["c_nationkey"])
    # pipeline 4: lineitem -> probe orders, supplier -> c_nationkey = s_nationkey -> probe nation -> group
    pl = E.plan("lineitem")
    pl.probe(ho, "l_orderkey", "inner", ["c_nationkey"])   # ~1/7 of the rows (order year)
    pl.probe(hs, "l_suppkey", "inner", ["s_nationkey"])
    pl.compute("dn", [("load", "c_nationkey"), ("sub", "s_nationkey")])
    pl.filter("dn", "=", 0)                                # c_nationkey = s_nationkey
    pl.probe(hn, "s_nationkey", "semi")                    # the nation is in ASIA
    pl.compute("n_name", [("load", "s_nationkey")])        # n_name = the nation's code
    pl.compute("rev", [("load", "l_discount"), ("rsub", 100), ("mul", "l_extendedprice")])  # scale 4
    pl.aggregate(keys=[("n_name", 0, 25)], aggs=[("sum", "rev"), ("count", None)],
                 order=[("revenue", True)], agg_names=["revenue", "count"])
    res = E.run(pl)
    pl.keep += [rn, ro, hn, ho]
    return res, pl


# ---------------------------------------------------------------- TPC-H Q7
# select supp_nation, cust_nation, l_year, sum(volume) as revenue
# from (select n1.n_name as supp_nation, n2.n_name as cust_nation, extract(year from l_shipdate) as l_year,
#              l_extendedprice * (1 - l_discount) as volume
#       from supplier, lineitem, orders, customer, nation n1, nation n2
#       where s_suppkey = l_suppkey and o_orderkey = l_orderkey and c_custkey = o_custkey
#         and s_nationkey = n1.n_nationkey and c_nationkey = n2.n_nationkey
#         and ((n1.n_name = 'FRANCE' and n2.n_name = 'GERMANY') or (n1.n_name = 'GERMANY' and n2.n_name = 'FRANCE'))
#         and l_shipdate between date '1995-01-01' and date '1996-12-31') as shipping
# group by supp_nation, cust_nation, l_year order by supp_nation, cust_nation, l_year
# The disjunction is (n1, n2 both in {FRANCE, GERMANY}) and n1 != n2; each half is pushed
# into its build (n_name = nation key, R18), the inequality stays in the pipeline.
def _tpch_q7(E: Engine, **_):
    pair = ("in", [hqgen.code(hqgen.NATIONS, "FRANCE"), hqgen.code(hqgen.NATIONS, "GERMANY")])
    hs, hc, hn = E.hashes([dict(table="tpch_supplier", key="s_suppkey", payload=["s_nationkey"],
                                preds=[("s_nationkey",) + pair]),
                           dict(table="tpch_customer", key="c_custkey", payload=["c_nationkey"],
                                preds=[("c_nationkey",) + pair]),
                           dict(table="nation", key="n_nationkey", preds=[("n_nationkey",) + pair])])
    ro = None
    if E.builds_here:
        po = E.plan("orders")
        po.probe(hc, "o_custkey", "inner", ["c_nationkey"])   # 2/25 of the orders
        po.materialise([("o_orderkey", "i32"), ("c_nationkey", "i32")])
        ro = E.run(po, partitioned=False)
    ho = E.hash_from(ro, ["o_orderkey", "c_nationkey"], "o_orderkey", ["c_nationkey"])
    pl = E.plan("lineitem")
    pl.filter("l_shipdate", "between", 19950101, 19961231)  # ~30 %
    pl.probe(hs, "l_suppkey", "inner", ["s_nationkey"])     # 2/25
    pl.probe(ho, "l_orderkey", "inner", ["c_nationkey"])    # 2/25
    pl.compute("dn", [("load", "s_nationkey"), ("sub", "c_nationkey")])
    pl.filter("dn", "!=", 0)                                # FRANCE -> GERMANY or GERMANY -> FRANCE
    pl.probe(hn, "s_nationkey", "semi")                     # n1
    pl.probe(hn, "c_nationkey", "semi")                     # n2
    pl.compute("l_year", [("load", "l_shipdate"), ("div", 10000)])
    pl.compute("rev", [("load", "l_discount"), ("rsub", 100), ("mul", "l_extendedprice")])  # scale 4
    pl.aggregate(keys=[("s_nationkey", 0, 25), ("c_nationkey", 0, 25), ("l_year", 1995, 2)],
                 aggs=[("sum", "rev"), ("count", None)],
                 order=[("s_nationkey", False), ("c_nationkey", False), ("l_year", False)],
                 agg_names=["revenue", "count"])
    pb_names = ["supp_nation", "cust_nation", "l_year", "revenue", "count"]
    res = E.run(pl)
    pl.result_names = pb_names
    pl.keep += [ro, ho]
    return res, pl


# ---------------------------------------------------------------- TPC-H Q10
# select c_custkey, c_name, sum(l_extendedprice * (1 - l_discount)) as revenue, c_acctbal,
#   n_name, c_address, c_phone, c_comment from customer, orders, lineitem, nation
# where c_custkey = o_custkey and l_orderkey = o_orderkey and o_orderdate >= '1993-10-01'
#   and o_orderdate < '1994-01-01' and l_returnflag = 'R' and c_nationkey = n_nationkey
# group by c_custkey, c_name, c_acctbal, c_phone, n_name, c_address, c_comment
# order by revenue desc limit 20
# (R18: the customer attributes besides c_custkey and n_name depend on c_custkey)
def _tpch_q10(E: Engine, limit: int = 20, **_):
    hc, hn = E.hashes([dict(table="tpch_customer", key="c_custkey", payload=["c_nationkey"]),
                       dict(table="nation", key="n_nationkey")])
    ro = None
    if E.builds_here:
        po = E.plan("orders")
        po.filter("o_orderdate", "between", 19931001, 19940101 - 1)
        po.probe(hc, "o_custkey", "inner", ["c_nationkey"])
        po.materialise([("o_orderkey", "i32"), ("o_custkey", "i32"), ("c_nationkey", "i32")])
        ro = E.run(po, partitioned=False)
    ho = E.hash_from(ro, ["o_orderkey", "o_custkey", "c_nationkey"], "o_orderkey", ["o_custkey", "c_nationkey"])
    nk = max(int(ho.meta().nkeys), 0)
    pl = E.plan("lineitem")
    pl.filter("l_returnflag", "=", hqgen.code(hqgen.RETURNFLAGS, "R"))
    pl.probe(ho, "l_orderkey", "inner", ["o_custkey", "c_nationkey"])
    pl.probe(hn, "c_nationkey", "semi")
    pl.compute("c_custkey", [("load", "o_custkey")])
    pl.compute("n_name", [("load", "c_nationkey")])
    pl.compute("rev", [("load", "l_discount"), ("rsub", 100), ("mul", "l_extendedprice")])  # scale 4
    pl.aggregate(keys=[("c_custkey", 0, 1 << 31), ("n_name", 0, 25)], aggs=[("sum", "rev"), ("count", None)],
                 order=[("revenue", True)], limit=limit, group_capacity=max(1024, nk),
                 agg_names=["revenue", "count"])
    res = E.run(pl)
    pl.keep += [ro, ho]
    return res, pl


# ------------------------------------------------------- TPC-H Q4, Q13, Q17, Q18, Q19, Q21
# Correlated and nested subqueries become pipelines whose aggregation results feed
# builds or further pipelines (pipeline breakers); functionally dependent
# attributes (R18) ride along as MIN aggregates of their group.  Multi-GPU (DESIGN.md
# §7): fact pipelines run over each rank's range partition; E.gather completes an
# intermediate GROUP BY on the root (an order split by the partition is merged there),
# whose builds are broadcast; root-side pipelines finish the query on the root.
_KEY32 = 1 << 31


class _RootOnly:
    """What a non-root rank returns for a query the root finishes alone."""
    root_only = True

    def __init__(self, names):
        self.result_names, self.keep = list(names), []


def _orders_estimate(E: Engine) -> int:
    return max(1024, E.table("lineitem").nrows // 4)  # 1..7 lines per order, 4 on average


# select o_orderpriority, count(*) as order_count from orders
# where o_orderdate >= date '1993-07-01' and o_orderdate < date '1993-10-01'
#   and exists (select * from lineitem where l_orderkey = o_orderkey and l_commitdate < l_receiptdate)
# group by o_orderpriority order by o_orderpriority
def _tpch_q4(E: Engine, **_):
    # the quarter's orders -> build (3.8 % of the orders, payload o_orderpriority)
    ho = E.hash("orders", "o_orderkey", payload=["o_orderpriority"],
                preds=[("o_orderdate", "between", 19930701, 19931001 - 1)])
    nk = max(int(ho.meta().nkeys), 0)
    # lineitem: late lines probe the quarter's orders; GROUP BY l_orderkey = the EXISTS (one row per order)
    pl = E.plan("lineitem")
    pl.compute("late", [("load", "l_receiptdate"), ("sub", "l_commitdate")])
    pl.filter("late", ">", 0)                                   # l_commitdate < l_receiptdate
    pl.probe(ho, "l_orderkey", "inner", ["o_orderpriority"])
    pl.aggregate(keys=[("l_orderkey", 0, _KEY32), ("o_orderpriority", 0, 5)], aggs=[("count", None)],
                 group_capacity=max(1024, nk), agg_names=["lines"])
    rl = E.gather(E.run(pl), pl)
    if rl is None:  # non-root rank: the root finishes the query
        return None, _RootOnly(["o_orderpriority", "order_count"])
    # orders per priority over the distinct order keys
    pg = E.plan_over(rl, ["l_orderkey", "o_orderpriority", "lines"])
    pg.aggregate(keys=[("o_orderpriority", 0, 5)], aggs=[("count", None)],
                 order=[("o_orderpriority", False)], agg_names=["order_count"])
    return E.run(pg, partitioned=False), pg


# select c_count, count(*) as custdist
# from (select c_custkey, count(o_orderkey) from customer left outer join orders on c_custkey = o_custkey
#       group by c_custkey) as c_orders (c_custkey, c_count)
# group by c_count order by custdist desc, c_count desc            (App F: no o_comment LIKE)
def _tpch_q13(E: Engine, **_):
    po = E.plan("orders")
    po.aggregate(keys=[("o_custkey",) + E.key_domain("orders", "o_custkey")], aggs=[("count", None)],
                 group_capacity=max(1024, E.table("orders").nrows // 4), agg_names=["n"])
    ro = E.gather(E.run(po), po)
    hn = E.hash_from(ro, ["o_custkey", "n"], "o_custkey", ["n"])
    maxn = max(int(hn.meta().pay_max), 0)
    if not E.builds_here:  # the customer table (the outer join's preserved side) is on the root
        return None, _RootOnly(["c_count", "custdist"])
    pc = E.plan("tpch_customer")
    pc.probe(hn, "c_custkey", "outer", ["c_count"])            # LEFT OUTER JOIN: 0 orders -> 0
    pc.aggregate(keys=[("c_count", 0, maxn + 1)], aggs=[("count", None)],
                 order=[("custdist", True), ("c_count", True)], agg_names=["custdist"])
    res = E.run(pc, partitioned=False)
    pc.keep += [ro, hn]
    return res, pc


# select sum(l_extendedprice) / 7.0 as avg_yearly from lineitem, part
# where p_partkey = l_partkey and p_brand = 'Brand#23' and p_container = 'MED BOX'
#   and l_quantity < (select 0.2 * avg(l_quantity) from lineitem where l_partkey = p_partkey)
# unnested (App F): pipeline 1 aggregates the subquery per selected part, pipeline 2
# tests l_quantity < 0.2 * sum / cnt as 5 * l_quantity * cnt - sum < 0 (exact integers, R19).
def _tpch_q17(E: Engine, **_):
    hp = E.hash("tpch_part", "p_partkey", preds=[("p_brand", "=", hqgen.code(hqgen.BRANDS, "Brand#23")),
                                                 ("p_container", "=", hqgen.code(hqgen.CONTAINERS, "MED BOX"))])
    p1 = E.plan("lineitem")
    p1.probe(hp, "l_partkey", "semi")
    p1.aggregate(keys=[("l_partkey",) + E.key_domain("lineitem", "l_partkey")],
                 aggs=[("sum", "l_quantity"), ("count", None)],
                 group_capacity=max(1024, int(hp.meta().nkeys)), agg_names=["sum_qty", "cnt"])
    r1 = E.gather(E.run(p1), p1)
    ha = E.hash_from(r1, ["l_partkey", "sum_qty", "cnt"], "l_partkey", ["sum_qty", "cnt"])
    p2 = E.plan("lineitem")
    p2.probe(ha, "l_partkey", "inner", ["sum_qty", "cnt"])
    p2.compute("d", [("load", "l_quantity"), ("mul", 5), ("mul", "cnt"), ("sub", "sum_qty")])
    p2.filter("d", "<", 0)
    p2.aggregate(aggs=[("sum", "l_extendedprice"), ("count", None)], agg_names=["sum_extendedprice", "count"])
    res = E.run(p2)
    p2.keep += [r1, hp]
    return res, p2


# select c_name, c_custkey, o_orderkey, o_orderdate, o_totalprice, sum(l_quantity)
# from customer, orders, lineitem
# where o_orderkey in (select l_orderkey from lineitem group by l_orderkey having sum(l_quantity) > 300)
#   and c_custkey = o_custkey and o_orderkey = l_orderkey
# group by c_name, c_custkey, o_orderkey, o_orderdate, o_totalprice
# order by o_totalprice desc, o_orderdate limit 100
def _tpch_q18(E: Engine, limit: int = 100, **_):
    # the IN subquery: GROUP BY l_orderkey over all of lineitem, HAVING as the build predicate
    p1 = E.plan("lineitem")
    p1.aggregate(keys=[("l_orderkey",) + E.key_domain("lineitem", "l_orderkey")], aggs=[("sum", "l_quantity")],
                 group_capacity=_orders_estimate(E), agg_names=["sum_qty"])
    r1 = E.gather(E.run(p1), p1)
    hb = E.hash_from(r1, ["l_orderkey", "sum_qty"], "l_orderkey", preds=[("sum_qty", ">", 30000)])
    hc = E.hash("tpch_customer", "c_custkey")
    ro = None
    if E.builds_here:  # build side: the orders pipeline runs where the dimensions are
        po = E.plan("orders")
        po.probe(hb, "o_orderkey", "semi")
        po.probe(hc, "o_custkey", "semi")
        po.materialise([("o_orderkey", "i32"), ("o_custkey", "i32"), ("o_orderdate", "i32"), ("o_totalprice", "i64")])
        ro = E.run(po, partitioned=False)
    ho = E.hash_from(ro, ["o_orderkey", "o_custkey", "o_orderdate", "o_totalprice"], "o_orderkey",
                     ["o_custkey", "o_orderdate", "o_totalprice"])
    pl = E.plan("lineitem")
    pl.probe(ho, "l_orderkey", "inner", ["o_custkey", "o_orderdate", "o_totalprice"])
    pl.aggregate(keys=[("l_orderkey", 0, _KEY32)],
                 aggs=[("min", "o_custkey"), ("min", "o_orderdate"), ("min", "o_totalprice"),
                       ("sum", "l_quantity"), ("count", None)],
                 order=[("o_totalprice", True), ("o_orderdate", False)], limit=limit,
                 group_capacity=max(1024, int(ho.meta().nkeys)),
                 agg_names=["c_custkey", "o_orderdate", "o_totalprice", "sum_qty", "count"])
    res = E.run(pl)
    pl.result_names = ["o_orderkey"] + pl.result_names[1:]
    pl.keep += [r1, hb, ro, ho]
    return res, pl


# select sum(l_extendedprice * (1 - l_discount)) as revenue from lineitem, part
# where (p_partkey = l_partkey and p_brand = 'Brand#12' and p_container in ('SM CASE', 'SM BOX', 'SM PACK', 'SM PKG')
#        and l_quantity >= 1 and l_quantity <= 1 + 10 and p_size between 1 and 5
#        and l_shipmode in ('AIR', 'AIR REG') and l_shipinstruct = 'DELIVER IN PERSON')
#    or (... 'Brand#23' ... ('MED BAG', 'MED BOX', 'MED PKG', 'MED PACK') ... 10 .. 20 ... size 1 .. 10 ...)
#    or (... 'Brand#34' ... ('LG CASE', 'LG BOX', 'LG PACK', 'LG PKG') ... 20 .. 30 ... size 1 .. 15 ...)
# The conjuncts common to the three disjuncts are filters / the part build's superset
# predicate; each disjunct is one predicate expression over the probe payloads (HQ_I_AND_*).
_Q19 = [("Brand#12", ["SM CASE", "SM BOX", "SM PACK", "SM PKG"], 1, 5),
        ("Brand#23", ["MED BAG", "MED BOX", "MED PKG", "MED PACK"], 10, 10),
        ("Brand#34", ["LG CASE", "LG BOX", "LG PACK", "LG PKG"], 20, 15)]


def _tpch_q19(E: Engine, **_):
    brands = [hqgen.code(hqgen.BRANDS, b) for b, *_ in _Q19]
    conts = [[hqgen.code(hqgen.CONTAINERS, c) for c in cs] for _, cs, *_ in _Q19]
    hp = E.hash("tpch_part", "p_partkey", payload=["p_brand", "p_container", "p_size"],
                preds=[("p_brand", "in", brands), ("p_container", "in", sum(conts, [])),
                       ("p_size", "between", 1, 15)])
    modes = [hqgen.code(hqgen.SHIPMODES, m) for m in ("AIR", "AIR REG") if m in hqgen.SHIPMODES]  # R19
    pl = E.plan("lineitem")
    pl.filter("l_shipinstruct", "=", hqgen.code(hqgen.SHIPINSTRUCTS, "DELIVER IN PERSON"))
    pl.filter("l_shipmode", "in", modes)
    pl.filter("l_quantity", "between", 100, 3000)               # the union of the three ranges
    pl.probe(hp, "l_partkey", "inner", ["p_brand", "p_container", "p_size"])
    for k, (brand, cs, (_, _, qlo, size)) in enumerate(zip(brands, conts, _Q19)):
        code = [("load", 1), ("and_eq", "p_brand", brand), ("and_in", "p_container", cs),
                ("and_ge", "l_quantity", qlo * 100), ("and_le", "l_quantity", (qlo + 10) * 100),
                ("and_ge", "p_size", 1), ("and_le", "p_size", size)]
        code += [("or", f"b{j}") for j in range(k)]
        pl.compute(f"b{k}", code)
    pl.filter("b2", "!=", 0)
    pl.compute("rev", [("load", "l_discount"), ("rsub", 100), ("mul", "l_extendedprice")])  # scale 4
    pl.aggregate(aggs=[("sum", "rev"), ("count", None)], agg_names=["revenue", "count"])
    return E.run(pl), pl


# select s_name, count(*) as numwait from supplier, lineitem l1, orders, nation
# where s_suppkey = l1.l_suppkey and o_orderkey = l1.l_orderkey and o_orderstatus = 'F'
#   and l1.l_receiptdate > l1.l_commitdate
#   and exists (select * from lineitem l2 where l2.l_orderkey = l1.l_orderkey and l2.l_suppkey <> l1.l_suppkey)
#   and not exists (select * from lineitem l3 where l3.l_orderkey = l1.l_orderkey
#                   and l3.l_suppkey <> l1.l_suppkey and l3.l_receiptdate > l3.l_commitdate)
#   and s_nationkey = n_nationkey and n_name = 'SAUDI ARABIA'
# group by s_name order by numwait desc, s_name limit 100
# variant 1: App F's EXISTS for the third subquery.  l1's supplier belongs to
# both subqueries' supplier sets, so "another supplier exists" <=> min(l_suppkey) <> max(l_suppkey)
# over the order's lines (l2) / late lines (l3): two GROUP BY l_orderkey pipelines (R20).
def _tpch_q21(E: Engine, variant: int = 0, limit: int = 100, **_):
    saudi = hqgen.code(hqgen.NATIONS, "SAUDI ARABIA")
    hs, hn, ho = E.hashes([dict(table="tpch_supplier", key="s_suppkey", payload=["s_nationkey"],
                                preds=[("s_nationkey", "=", saudi)]),
                           dict(table="nation", key="n_nationkey", preds=[("n_nationkey", "=", saudi)]),
                           dict(table="orders", key="o_orderkey",
                                preds=[("o_orderstatus", "=", hqgen.code(hqgen.ORDERSTATUS, "F"))])])
    sets = []
    okeys = E.key_domain("lineitem", "l_orderkey")
    for late in (False, True):  # l2: all lines of the order; l3: its late lines
        pb = E.plan("lineitem")
        if late:
            pb.compute("late", [("load", "l_receiptdate"), ("sub", "l_commitdate")])
            pb.filter("late", ">", 0)
        pb.aggregate(keys=[("l_orderkey",) + okeys], aggs=[("min", "l_suppkey"), ("max", "l_suppkey")],
                     group_capacity=_orders_estimate(E), agg_names=["smin", "smax"])
        r = E.gather(E.run(pb), pb)
        mat = None
        if r is not None:  # the derived predicate runs on the merged groups (root)
            pm = E.plan_over(r, ["l_orderkey", "smin", "smax"])
            pm.compute("d", [("load", "smax"), ("sub", "smin")])
            pm.filter("d", "=" if (late and variant == 0) else "!=", 0)
            pm.materialise([("l_orderkey", "i32")])
            mat = E.run(pm, partitioned=False)
        sets.append(E.hash_from(mat, ["l_orderkey"], "l_orderkey"))
    h2, h3 = sets
    pl = E.plan("lineitem")
    pl.compute("late", [("load", "l_receiptdate"), ("sub", "l_commitdate")])
    pl.filter("late", ">", 0)                                   # l1.l_receiptdate > l1.l_commitdate
    pl.probe(hs, "l_suppkey", "inner", ["s_nationkey"])         # 1/25
    pl.probe(hn, "s_nationkey", "semi")
    pl.probe(ho, "l_orderkey", "semi")                          # o_orderstatus = 'F'
    pl.probe(h2, "l_orderkey", "semi")                          # exists l2
    pl.probe(h3, "l_orderkey", "semi")                          # not exists l3 (variant 1: exists)
    ms = hs.meta()  # the surviving rows' suppliers are the build's keys (same meta on every rank)
    pl.aggregate(keys=[("l_suppkey", int(ms.key_min), max(int(ms.key_max) - int(ms.key_min) + 1, 1))],
                 aggs=[("count", None)],
                 order=[("numwait", True), ("l_suppkey", False)], limit=limit, agg_names=["numwait"])
    res = E.run(pl)
    pl.result_names = ["s_suppkey", "numwait"]
    pl.keep += sets
    return res, pl


# select nation, o_year, sum(amount) as sum_profit
# from (select n_name as nation, extract(year from o_orderdate) as o_year,
#              l_extendedprice * (1 - l_discount) - ps_supplycost * l_quantity as amount
#       from part, supplier, lineitem, partsupp, orders, nation
#       where s_suppkey = l_suppkey and ps_suppkey = l_suppkey and ps_partkey = l_partkey
#         and p_partkey = l_partkey and o_orderkey = l_orderkey and s_nationkey = n_nationkey
#         and p_name like '%green%') as profit
# group by nation, o_year order by nation, o_year desc
# App F: the LIKE becomes a filter on p_partkey, p_partkey <= |part| * 5 // 92 (R19),
# pushed into the partsupp build through p_partkey = ps_partkey.  partsupp is joined on its
# two-column key (ps_partkey, ps_suppkey): a composite hash table (hq_build_desc::composite).
def _tpch_q9(E: Engine, pmax: Optional[int] = None, **_):
    if pmax is None:  # only the ranks that build need it (non-root ranks hold no dimension tables)
        pmax = E.table("tpch_part").nrows * 5 // 92 if E.builds_here else 0
    hp, hps, hs, hn, ho = E.hashes([
        dict(table="tpch_part", key="p_partkey", preds=[("p_partkey", "<=", pmax)]),
        dict(table="partsupp", key="ps_partkey", key2="ps_suppkey", payload=["ps_supplycost"],
             preds=[("ps_partkey", "<=", pmax)]),
        dict(table="tpch_supplier", key="s_suppkey", payload=["s_nationkey"]),
        dict(table="nation", key="n_nationkey"),
        dict(table="orders", key="o_orderkey", payload=["o_orderdate"])])
    pl = E.plan("lineitem")
    pl.probe(hp, "l_partkey", "semi")                                           # 5/92
    pl.probe(hps, "l_partkey", "inner", ["ps_supplycost"], key2="l_suppkey")
    pl.probe(hs, "l_suppkey", "inner", ["s_nationkey"])
    pl.probe(hn, "s_nationkey", "semi")
    pl.probe(ho, "l_orderkey", "inner", ["o_orderdate"])
    pl.compute("o_year", [("load", "o_orderdate"), ("div", 10000)])
    pl.compute("cost", [("load", "ps_supplycost"), ("mul", "l_quantity")])   # scale 4
    pl.compute("amount", [("load", "l_discount"), ("rsub", 100), ("mul", "l_extendedprice"), ("sub", "cost")])
    pl.aggregate(keys=[("s_nationkey", 0, 25), ("o_year", 1992, 7)], aggs=[("sum", "amount"), ("count", None)],
                 order=[("s_nationkey", False), ("o_year", True)], agg_names=["sum_profit", "count"])
    res = E.run(pl)
    pl.result_names = ["nation"] + pl.result_names[1:]
    return res, pl


# ------------------------------------------------ paper micro queries (f2)
def _micro_select(E: Engine, x: int = 5, resolution=None, **_):
    """PAPER.md Fig 16 'Query 1': selection + projection, materialised."""
    pb = E.plan("lineorder")
    pb.filter("lo_quantity", "between", 25 - x, 25 + x)
    pb.compute("revenue", [("load", "lo_extendedprice"), ("mul", "lo_discount"), ("add", "lo_tax")])
    pb.materialise([("revenue", "i64")])
    return E.run(pb), pb


def _micro_sum(E: Engine, x: int = 5, **_):
    """App G.1: single-tuple aggregation of Query 1."""
    pb = E.plan("lineorder")
    pb.filter("lo_quantity", "between", 25 - x, 25 + x)
    pb.compute("revenue", [("load", "lo_extendedprice"), ("mul", "lo_discount"), ("add", "lo_tax")])
    pb.aggregate(aggs=[("sum", "revenue"), ("count", None)], agg_names=["revenue", "count"])
    return E.run(pb), pb


def _micro_groupby(E: Engine, x: int = 16, **_):
    """Fig 26: sum(lo_extendedprice) group by lo_orderkey % x."""
    pb = E.plan("lineorder")
    pb.compute("k", [("load", "lo_orderkey"), ("mod", x)])
    pb.aggregate(keys=[("k", 0, x)], aggs=[("sum", "lo_extendedprice"), ("count", None)],
                 agg_names=["sum", "count"])
    return E.run(pb), pb


QUERIES: Dict[str, Query] = {q.name: q for q in [
    Query("tpch_q6", "tpch", "lineitem",
          {"lineitem": ["l_shipdate", "l_discount", "l_quantity", "l_extendedprice"]}, _tpch_q6),
    Query("tpch_q1", "tpch", "lineitem",
          {"lineitem": ["l_shipdate", "l_returnflag", "l_linestatus", "l_quantity", "l_extendedprice",
                        "l_discount", "l_tax"]}, _tpch_q1),
    Query("ssb_q11", "ssb", "lineorder",
          {"lineorder": ["lo_orderdate", "lo_quantity", "lo_discount", "lo_extendedprice"],
           "date": ["d_datekey", "d_year", "d_yearmonthnum", "d_weeknuminyear"]}, _ssb_q1(1)),
    Query("ssb_q12", "ssb", "lineorder",
          {"lineorder": ["lo_orderdate", "lo_quantity", "lo_discount", "lo_extendedprice"],
           "date": ["d_datekey", "d_year", "d_yearmonthnum", "d_weeknuminyear"]}, _ssb_q1(2)),
    Query("ssb_q13", "ssb", "lineorder",
          {"lineorder": ["lo_orderdate", "lo_quantity", "lo_discount", "lo_extendedprice"],
           "date": ["d_datekey", "d_year", "d_yearmonthnum", "d_weeknuminyear"]}, _ssb_q1(3)),
    Query("ssb_q31", "ssb", "lineorder",
          {"lineorder": ["lo_custkey", "lo_suppkey", "lo_orderdate", "lo_revenue"],
           "customer": ["c_custkey", "c_nation", "c_region"], "supplier": ["s_suppkey", "s_nation", "s_region"],
           "date": ["d_datekey", "d_year"]}, _ssb_q31),
    Query("ssb_q31_mat", "ssb", "lineorder",
          {"lineorder": ["lo_custkey", "lo_suppkey", "lo_orderdate", "lo_revenue"],
           "customer": ["c_custkey", "c_nation", "c_region"], "supplier": ["s_suppkey", "s_nation", "s_region"],
           "date": ["d_datekey", "d_year"]}, _ssb_q31_mat),
    Query("ssb_q41", "ssb", "lineorder",
          {"lineorder": ["lo_custkey", "lo_suppkey", "lo_partkey", "lo_orderdate", "lo_revenue", "lo_supplycost"],
           "customer": ["c_custkey", "c_nation", "c_region"], "supplier": ["s_suppkey", "s_region"],
           "part": ["p_partkey", "p_mfgr"], "date": ["d_datekey", "d_year"]}, _ssb_q41),
    *[Query(f"ssb_q2{v}", "ssb", "lineorder",
            {"lineorder": ["lo_partkey", "lo_suppkey", "lo_orderdate", "lo_revenue"],
             "part": ["p_partkey", "p_category", "p_brand1"], "supplier": ["s_suppkey", "s_region"],
             "date": ["d_datekey", "d_year"]}, _ssb_q2(v)) for v in (1, 2, 3)],
    *[Query(f"ssb_q3{v}", "ssb", "lineorder",
            {"lineorder": ["lo_custkey", "lo_suppkey", "lo_orderdate", "lo_revenue"],
             "customer": ["c_custkey", "c_nation", "c_city"], "supplier": ["s_suppkey", "s_nation", "s_city"],
             "date": ["d_datekey", "d_year", "d_yearmonthnum"]}, _ssb_q3(v)) for v in (2, 3, 4)],
    *[Query(f"ssb_q4{v}", "ssb", "lineorder",
            {"lineorder": ["lo_custkey", "lo_suppkey", "lo_partkey", "lo_orderdate", "lo_revenue", "lo_supplycost"],
             "customer": ["c_custkey", "c_region"], "supplier": ["s_suppkey", "s_nation", "s_region", "s_city"],
             "part": ["p_partkey", "p_mfgr", "p_category", "p_brand1"], "date": ["d_datekey", "d_year"]},
            _ssb_q4(v)) for v in (2, 3)],
    Query("tpch_q3", "tpch", "lineitem",
          {"lineitem": ["l_orderkey", "l_shipdate", "l_extendedprice", "l_discount"],
           "orders": ["o_orderkey", "o_custkey", "o_orderdate", "o_shippriority"],
           "tpch_customer": ["c_custkey", "c_mktsegment"]}, _tpch_q3, copart="orders"),
    Query("tpch_q5", "tpch", "lineitem",
          {"lineitem": ["l_orderkey", "l_suppkey", "l_extendedprice", "l_discount"],
           "orders": ["o_orderkey", "o_custkey", "o_orderdate"], "tpch_customer": ["c_custkey", "c_nationkey"],
           "tpch_supplier": ["s_suppkey", "s_nationkey"], "nation": ["n_nationkey", "n_regionkey"],
           "region": ["r_regionkey"]}, _tpch_q5),
    Query("tpch_q7", "tpch", "lineitem",
          {"lineitem": ["l_orderkey", "l_suppkey", "l_shipdate", "l_extendedprice", "l_discount"],
           "orders": ["o_orderkey", "o_custkey"], "tpch_customer": ["c_custkey", "c_nationkey"],
           "tpch_supplier": ["s_suppkey", "s_nationkey"], "nation": ["n_nationkey"]}, _tpch_q7),
    Query("tpch_q10", "tpch", "lineitem",
          {"lineitem": ["l_orderkey", "l_returnflag", "l_extendedprice", "l_discount"],
           "orders": ["o_orderkey", "o_custkey", "o_orderdate"], "tpch_customer": ["c_custkey", "c_nationkey"],
           "nation": ["n_nationkey"]}, _tpch_q10),
    Query("tpch_q4", "tpch", "lineitem",
          {"lineitem": ["l_orderkey", "l_commitdate", "l_receiptdate"],
           "orders": ["o_orderkey", "o_orderdate", "o_orderpriority"]}, _tpch_q4),
    Query("tpch_q9", "tpch", "lineitem",
          {"lineitem": ["l_orderkey", "l_partkey", "l_suppkey", "l_quantity", "l_extendedprice", "l_discount"],
           "orders": ["o_orderkey", "o_orderdate"], "tpch_part": ["p_partkey"],
           "partsupp": ["ps_partkey", "ps_suppkey", "ps_supplycost"], "tpch_supplier": ["s_suppkey", "s_nationkey"],
           "nation": ["n_nationkey"]}, _tpch_q9),
    Query("tpch_q13", "tpch", "orders",
          {"orders": ["o_custkey"], "tpch_customer": ["c_custkey"]}, _tpch_q13),
    Query("tpch_q17", "tpch", "lineitem",
          {"lineitem": ["l_partkey", "l_quantity", "l_extendedprice"],
           "tpch_part": ["p_partkey", "p_brand", "p_container"]}, _tpch_q17),
    Query("tpch_q18", "tpch", "lineitem",
          {"lineitem": ["l_orderkey", "l_quantity"],
           "orders": ["o_orderkey", "o_custkey", "o_orderdate", "o_totalprice"],
           "tpch_customer": ["c_custkey"]}, _tpch_q18),
    Query("tpch_q19", "tpch", "lineitem",
          {"lineitem": ["l_partkey", "l_quantity", "l_extendedprice", "l_discount", "l_shipmode", "l_shipinstruct"],
           "tpch_part": ["p_partkey", "p_brand", "p_container", "p_size"]}, _tpch_q19),
    Query("tpch_q21", "tpch", "lineitem",
          {"lineitem": ["l_orderkey", "l_suppkey", "l_commitdate", "l_receiptdate"],
           "orders": ["o_orderkey", "o_orderstatus"], "tpch_supplier": ["s_suppkey", "s_nationkey"],
           "nation": ["n_nationkey"]}, _tpch_q21),
    Query("micro_select", "ssb", "lineorder",
          {"lineorder": ["lo_quantity", "lo_extendedprice", "lo_discount", "lo_tax"]}, _micro_select),
    Query("micro_sum", "ssb", "lineorder",
          {"lineorder": ["lo_quantity", "lo_extendedprice", "lo_discount", "lo_tax"]}, _micro_sum),
    Query("micro_groupby", "ssb", "lineorder",
          {"lineorder": ["lo_orderkey", "lo_extendedprice"]}, _micro_groupby),
]}


def load_tables(ctx: hq.Context, query: Query, sf: float, seed: int = hqgen.DEFAULT_SEED,
                fact_range: Optional[tuple] = None, host: Optional[Dict[str, Dict]] = None,
                skip_dims: bool = False, stream_fact: bool = False,
                copart_range: Optional[tuple] = None) -> Dict[str, hq.Table]:
    """Generate (or take from ``host``) the referenced columns and load them onto
    the context's device.  fact_range: rows of the fact table to load (a range
    partition).  skip_dims: load only the fact table (non-root ranks).  stream_fact:
    leave the fact table in host memory (HQ_HOST_STREAM, batch processing).
    copart_range: rows of ``query.copart`` (the order table co-partitioned with the
    fact table, hqgen.copartition)."""
    tables = {}
    for t, cols in query.columns.items():
        if skip_dims and t != query.fact and t != query.copart:
            continue
        if host is not None and t in host:
            data = {c: host[t][c] for c in cols}
        else:
            rr = fact_range if t == query.fact else (copart_range if t == query.copart else None)
            data = hqgen.generate(t, sf, seed, columns=cols, row_range=rr)
        tables[t] = ctx.load_columns(data, stream=stream_fact and t == query.fact)
    return tables
