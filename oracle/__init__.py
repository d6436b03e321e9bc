"""oracle -- TEST INFRASTRUCTURE ONLY.

A plain tuple-at-a-time CPU oracle (C++17, ``oracle.cpp``) for the queries of
SURVEY.md §8(c.1).  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py`` (its ``cpu_baseline`` leg and ``--impl reference``) may import
this package.  It shares no code with the CUDA path
(``paper_conf_sigmod_funkebnmt18_b200``); the only common module is the input
generator ``hqgen``.

Pins (tests/test_oracle.py): hand-computed fixtures F1-F6 (tests/golden/),
brute-force nested-loop joins, numpy library cross-checks, invariants
(COUNT(*) = qualifying rows, sum of group counts = total, sum of group sums =
scalar sum) and the generator's closed-form selectivities.  No function is
"parity unpinned".

Each function takes dicts of numpy columns named as in ``hqgen.SCHEMAS`` and
returns an :class:`OracleResult` with named int64 / float64 columns.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass, field
from typing import Dict, List

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_SRC = os.path.join(_HERE, "oracle.cpp")

P_I32 = ctypes.POINTER(ctypes.c_int32)
P_I64 = ctypes.POINTER(ctypes.c_int64)
P_I8 = ctypes.POINTER(ctypes.c_int8)


class _Result(ctypes.Structure):
    _fields_ = [("nrows", ctypes.c_int64), ("ni", ctypes.c_int32), ("nf", ctypes.c_int32),
                ("icol", P_I64), ("fcol", ctypes.POINTER(ctypes.c_double)),
                ("qualifying", ctypes.c_int64)]


class _Lineorder(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64)] + [(c, P_I32) for c in (
        "orderkey", "custkey", "partkey", "suppkey", "orderdate", "quantity", "extendedprice",
        "discount", "revenue", "supplycost", "tax")]


class _Date(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("datekey", P_I32), ("year", P_I32),
                ("yearmonthnum", P_I32), ("weeknuminyear", P_I32)]


class _SsbDim(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("key", P_I32), ("nation", P_I8), ("region", P_I8), ("city", P_I32)]


class _Part(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("partkey", P_I32), ("mfgr", P_I8), ("category", P_I8), ("brand1", P_I32)]


class _Lineitem(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("orderkey", P_I32), ("quantity", P_I64),
                ("extendedprice", P_I64), ("discount", P_I64), ("tax", P_I64),
                ("returnflag", P_I8), ("linestatus", P_I8), ("shipdate", P_I32), ("suppkey", P_I32),
                ("partkey", P_I32), ("commitdate", P_I32), ("receiptdate", P_I32),
                ("shipmode", P_I8), ("shipinstruct", P_I8)]


class _Orders(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("orderkey", P_I32), ("custkey", P_I32),
                ("orderdate", P_I32), ("shippriority", P_I32), ("orderpriority", P_I8),
                ("totalprice", P_I64), ("orderstatus", P_I8)]


class _Partsupp(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("partkey", P_I32), ("suppkey", P_I32), ("supplycost", P_I64)]


class _TPart(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("partkey", P_I32), ("brand", P_I8), ("container", P_I8), ("size", P_I32)]


class _TCustomer(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("custkey", P_I32), ("mktsegment", P_I8), ("nationkey", P_I8)]


class _TSupplier(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("suppkey", P_I32), ("nationkey", P_I8)]


class _Nation(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("nationkey", P_I8), ("regionkey", P_I8)]


class _Region(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("regionkey", P_I8)]


class OracleError(RuntimeError):
    def __init__(self, rc: int):
        super().__init__({-4: "duplicate build key", -6: "int64 overflow", -1: "bad argument"}.get(rc, str(rc)))
        self.rc = rc


@dataclass
class OracleResult:
    columns: Dict[str, np.ndarray] = field(default_factory=dict)
    qualifying: int = 0

    @property
    def nrows(self) -> int:
        return len(next(iter(self.columns.values()))) if self.columns else 0

    def rows(self, names: List[str] = None) -> List[tuple]:
        names = names or list(self.columns)
        return list(zip(*[self.columns[n].tolist() for n in names]))


_lib = None


def build() -> str:
    subprocess.check_call(["g++", "-O2", "-std=c++17", "-shared", "-fPIC", "-pthread", "-o", _SO, _SRC])
    return _SO


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
            build()
        L = ctypes.CDLL(_SO)
        P = ctypes.POINTER
        sig = {
            "orc_tpch_q6": [P(_Lineitem), ctypes.c_int],
            "orc_tpch_q1": [P(_Lineitem), ctypes.c_int],
            "orc_ssb_q1": [ctypes.c_int, P(_Lineorder), P(_Date), ctypes.c_int, ctypes.c_int],
            "orc_ssb_q31": [P(_Lineorder), P(_SsbDim), P(_SsbDim), P(_Date), ctypes.c_int, ctypes.c_int],
            "orc_ssb_q31_mat": [P(_Lineorder), P(_SsbDim), P(_SsbDim), P(_Date), ctypes.c_int, ctypes.c_int],
            "orc_ssb_q41": [P(_Lineorder), P(_Date), P(_SsbDim), P(_SsbDim), P(_Part), ctypes.c_int, ctypes.c_int],
            "orc_tpch_q3": [P(_TCustomer), P(_Orders), P(_Lineitem), ctypes.c_int, ctypes.c_int],
            "orc_tpch_q9": [P(_TPart), P(_TSupplier), P(_Lineitem), P(_Partsupp), P(_Orders), P(_Nation),
                            ctypes.c_int32, ctypes.c_int, ctypes.c_int],
            "orc_tpch_q4": [P(_Orders), P(_Lineitem), ctypes.c_int, ctypes.c_int],
            "orc_tpch_q13": [P(_TCustomer), P(_Orders), ctypes.c_int],
            "orc_tpch_q17": [P(_TPart), P(_Lineitem), ctypes.c_int],
            "orc_tpch_q18": [P(_TCustomer), P(_Orders), P(_Lineitem), ctypes.c_int],
            "orc_tpch_q19": [P(_TPart), P(_Lineitem), ctypes.c_int, ctypes.c_int],
            "orc_tpch_q21": [ctypes.c_int, P(_TSupplier), P(_Orders), P(_Lineitem), P(_Nation), ctypes.c_int],
            "orc_tpch_q7": [P(_TCustomer), P(_Orders), P(_Lineitem), P(_TSupplier), P(_Nation),
                            ctypes.c_int, ctypes.c_int],
            "orc_tpch_q10": [P(_TCustomer), P(_Orders), P(_Lineitem), P(_Nation), ctypes.c_int, ctypes.c_int],
            "orc_tpch_q5": [P(_TCustomer), P(_Orders), P(_Lineitem), P(_TSupplier), P(_Nation), P(_Region),
                            ctypes.c_int, ctypes.c_int],
            "orc_ssb_q2": [ctypes.c_int, P(_Lineorder), P(_Date), P(_Part), P(_SsbDim), ctypes.c_int, ctypes.c_int],
            "orc_ssb_q3": [ctypes.c_int, P(_Lineorder), P(_SsbDim), P(_SsbDim), P(_Date), ctypes.c_int, ctypes.c_int],
            "orc_ssb_q4": [ctypes.c_int, P(_Lineorder), P(_Date), P(_SsbDim), P(_SsbDim), P(_Part), ctypes.c_int,
                           ctypes.c_int],
            "orc_micro_select": [P(_Lineorder), ctypes.c_int32, ctypes.c_int],
            "orc_micro_sum": [P(_Lineorder), ctypes.c_int32, ctypes.c_int],
            "orc_micro_groupby": [P(_Lineorder), ctypes.c_int32, ctypes.c_int],
        }
        for name, args in sig.items():
            f = getattr(L, name)
            f.restype = ctypes.c_int
            f.argtypes = args + [P(_Result)]
        L.orc_free.restype = None
        L.orc_free.argtypes = [P(_Result)]
        _lib = L
    return _lib


def _ptr(arr, ctype, keep):
    if arr is None:
        return None
    a = np.ascontiguousarray(arr, dtype={P_I32: np.int32, P_I64: np.int64, P_I8: np.int8}[ctype])
    keep.append(a)
    return a.ctypes.data_as(ctype)


def _n(cols) -> int:
    return len(next(iter(cols.values())))


def _lineorder(t, keep):
    s = _Lineorder()
    s.n = _n(t)
    for f in ("orderkey", "custkey", "partkey", "suppkey", "orderdate", "quantity", "extendedprice",
              "discount", "revenue", "supplycost", "tax"):
        setattr(s, f, _ptr(t.get("lo_" + f), P_I32, keep))
    return s


def _date(t, keep):
    s = _Date()
    s.n = _n(t)
    for f in ("datekey", "year", "yearmonthnum", "weeknuminyear"):
        setattr(s, f, _ptr(t.get("d_" + f), P_I32, keep))
    return s


def _dim(t, prefix, keep):
    s = _SsbDim()
    s.n = _n(t)
    s.key = _ptr(t[prefix + ("custkey" if prefix == "c_" else "suppkey")], P_I32, keep)
    s.nation = _ptr(t.get(prefix + "nation"), P_I8, keep)
    s.region = _ptr(t.get(prefix + "region"), P_I8, keep)
    s.city = _ptr(t.get(prefix + "city"), P_I32, keep)
    return s


def _part(t, keep):
    s = _Part()
    s.n = _n(t)
    s.partkey = _ptr(t["p_partkey"], P_I32, keep)
    s.mfgr = _ptr(t.get("p_mfgr"), P_I8, keep)
    s.category = _ptr(t.get("p_category"), P_I8, keep)
    s.brand1 = _ptr(t.get("p_brand1"), P_I32, keep)
    return s


def _lineitem(t, keep):
    s = _Lineitem()
    s.n = _n(t)
    s.orderkey = _ptr(t.get("l_orderkey"), P_I32, keep)
    for f in ("quantity", "extendedprice", "discount", "tax"):
        setattr(s, f, _ptr(t.get("l_" + f), P_I64, keep))
    s.returnflag = _ptr(t.get("l_returnflag"), P_I8, keep)
    s.linestatus = _ptr(t.get("l_linestatus"), P_I8, keep)
    s.shipdate = _ptr(t.get("l_shipdate"), P_I32, keep)
    s.suppkey = _ptr(t.get("l_suppkey"), P_I32, keep)
    for f in ("partkey", "commitdate", "receiptdate"):
        setattr(s, f, _ptr(t.get("l_" + f), P_I32, keep))
    s.shipmode = _ptr(t.get("l_shipmode"), P_I8, keep)
    s.shipinstruct = _ptr(t.get("l_shipinstruct"), P_I8, keep)
    return s


def _orders(t, keep):
    s = _Orders()
    s.n = _n(t)
    for f in ("orderkey", "custkey", "orderdate", "shippriority"):
        setattr(s, f, _ptr(t.get("o_" + f), P_I32, keep))
    s.orderpriority = _ptr(t.get("o_orderpriority"), P_I8, keep)
    s.totalprice = _ptr(t.get("o_totalprice"), P_I64, keep)
    s.orderstatus = _ptr(t.get("o_orderstatus"), P_I8, keep)
    return s


def _tpart(t, keep):
    s = _TPart()
    s.n = _n(t)
    s.partkey = _ptr(t["p_partkey"], P_I32, keep)
    s.brand = _ptr(t.get("p_brand"), P_I8, keep)
    s.container = _ptr(t.get("p_container"), P_I8, keep)
    s.size = _ptr(t.get("p_size"), P_I32, keep)
    return s


def _tcust(t, keep):
    s = _TCustomer()
    s.n = _n(t)
    s.custkey = _ptr(t["c_custkey"], P_I32, keep)
    s.mktsegment = _ptr(t.get("c_mktsegment"), P_I8, keep)
    s.nationkey = _ptr(t.get("c_nationkey"), P_I8, keep)
    return s


def _tsupp(t, keep):
    s = _TSupplier()
    s.n = _n(t)
    s.suppkey = _ptr(t["s_suppkey"], P_I32, keep)
    s.nationkey = _ptr(t.get("s_nationkey"), P_I8, keep)
    return s


def _nation(t, keep):
    s = _Nation()
    s.n = _n(t)
    s.nationkey = _ptr(t["n_nationkey"], P_I8, keep)
    s.regionkey = _ptr(t.get("n_regionkey"), P_I8, keep)
    return s


def _region(t, keep):
    s = _Region()
    s.n = _n(t)
    s.regionkey = _ptr(t["r_regionkey"], P_I8, keep)
    return s


def _call(fname, args, icols, fcols=()):
    r = _Result()
    rc = getattr(lib(), fname)(*args, ctypes.byref(r))
    if rc != 0:
        raise OracleError(rc)
    try:
        n = r.nrows
        out = OracleResult(qualifying=int(r.qualifying))
        if n > 0:
            ia = np.ctypeslib.as_array(r.icol, shape=(r.ni * n,)).reshape(r.ni, n).copy() if r.ni else None
            fa = np.ctypeslib.as_array(r.fcol, shape=(r.nf * n,)).reshape(r.nf, n).copy() if r.nf else None
        for k, name in enumerate(icols):
            out.columns[name] = ia[k] if n > 0 else np.zeros(0, np.int64)
        for k, name in enumerate(fcols):
            out.columns[name] = fa[k] if n > 0 else np.zeros(0, np.float64)
        return out
    finally:
        lib().orc_free(ctypes.byref(r))


def tpch_q6(lineitem, nthreads=1) -> OracleResult:
    keep = []
    return _call("orc_tpch_q6", [ctypes.byref(_lineitem(lineitem, keep)), nthreads], ["revenue", "count"])


def tpch_q1(lineitem, nthreads=1) -> OracleResult:
    keep = []
    return _call("orc_tpch_q1", [ctypes.byref(_lineitem(lineitem, keep)), nthreads],
                 ["l_returnflag", "l_linestatus", "sum_qty", "sum_base_price", "sum_disc_price",
                  "sum_charge", "count_order"], ["avg_qty", "avg_price", "avg_disc"])


def ssb_q1(variant, lineorder, date, brute=False, nthreads=1) -> OracleResult:
    keep = []
    return _call("orc_ssb_q1", [variant, ctypes.byref(_lineorder(lineorder, keep)),
                                ctypes.byref(_date(date, keep)), int(brute), nthreads],
                 ["revenue", "count"])


def ssb_q31(lineorder, customer, supplier, date, brute=False, nthreads=1) -> OracleResult:
    keep = []
    return _call("orc_ssb_q31", [ctypes.byref(_lineorder(lineorder, keep)),
                                 ctypes.byref(_dim(customer, "c_", keep)),
                                 ctypes.byref(_dim(supplier, "s_", keep)),
                                 ctypes.byref(_date(date, keep)), int(brute), nthreads],
                 ["c_nation", "s_nation", "d_year", "revenue", "count"])


def ssb_q31_mat(lineorder, customer, supplier, date, brute=False, nthreads=1) -> OracleResult:
    keep = []
    return _call("orc_ssb_q31_mat", [ctypes.byref(_lineorder(lineorder, keep)),
                                     ctypes.byref(_dim(customer, "c_", keep)),
                                     ctypes.byref(_dim(supplier, "s_", keep)),
                                     ctypes.byref(_date(date, keep)), int(brute), nthreads],
                 ["c_nation", "s_nation", "d_year", "lo_revenue"])


def ssb_q41(lineorder, date, customer, supplier, part, brute=False, nthreads=1) -> OracleResult:
    keep = []
    return _call("orc_ssb_q41", [ctypes.byref(_lineorder(lineorder, keep)),
                                 ctypes.byref(_date(date, keep)),
                                 ctypes.byref(_dim(customer, "c_", keep)),
                                 ctypes.byref(_dim(supplier, "s_", keep)),
                                 ctypes.byref(_part(part, keep)), int(brute), nthreads],
                 ["d_year", "c_nation", "profit", "count"])


def ssb_q2(variant, lineorder, date, part, supplier, brute=False, nthreads=1) -> OracleResult:
    """SSB Q2.1-Q2.3 -> [d_year, p_brand1, revenue, count] ORDER BY d_year, p_brand1."""
    keep = []
    return _call("orc_ssb_q2", [variant, ctypes.byref(_lineorder(lineorder, keep)), ctypes.byref(_date(date, keep)),
                                ctypes.byref(_part(part, keep)), ctypes.byref(_dim(supplier, "s_", keep)),
                                int(brute), nthreads],
                 ["d_year", "p_brand1", "revenue", "count"])


def ssb_q3(variant, lineorder, customer, supplier, date, brute=False, nthreads=1) -> OracleResult:
    """SSB Q3.2-Q3.4 -> [c_city, s_city, d_year, revenue, count] ORDER BY d_year, revenue desc."""
    keep = []
    return _call("orc_ssb_q3", [variant, ctypes.byref(_lineorder(lineorder, keep)),
                                ctypes.byref(_dim(customer, "c_", keep)), ctypes.byref(_dim(supplier, "s_", keep)),
                                ctypes.byref(_date(date, keep)), int(brute), nthreads],
                 ["c_city", "s_city", "d_year", "revenue", "count"])


def ssb_q4(variant, lineorder, date, customer, supplier, part, brute=False, nthreads=1) -> OracleResult:
    """SSB Q4.2 -> [d_year, s_nation, p_category, profit, count]; Q4.3 -> [d_year, s_city,
    p_brand1, profit, count]; ORDER BY the three keys."""
    keep = []
    k1, k2 = ("s_nation", "p_category") if variant == 2 else ("s_city", "p_brand1")
    return _call("orc_ssb_q4", [variant, ctypes.byref(_lineorder(lineorder, keep)), ctypes.byref(_date(date, keep)),
                                ctypes.byref(_dim(customer, "c_", keep)), ctypes.byref(_dim(supplier, "s_", keep)),
                                ctypes.byref(_part(part, keep)), int(brute), nthreads],
                 ["d_year", k1, k2, "profit", "count"])


def tpch_q3(customer, orders, lineitem, brute=False, nthreads=1) -> OracleResult:
    keep = []
    return _call("orc_tpch_q3", [ctypes.byref(_tcust(customer, keep)),
                                 ctypes.byref(_orders(orders, keep)),
                                 ctypes.byref(_lineitem(lineitem, keep)), int(brute), nthreads],
                 ["l_orderkey", "revenue", "o_orderdate", "o_shippriority", "count"])


def tpch_q5(customer, orders, lineitem, supplier, nation, region, brute=False, nthreads=1) -> OracleResult:
    """TPC-H Q5 -> [n_name, revenue (scale 4), count] ORDER BY revenue desc."""
    keep = []
    return _call("orc_tpch_q5", [ctypes.byref(_tcust(customer, keep)), ctypes.byref(_orders(orders, keep)),
                                 ctypes.byref(_lineitem(lineitem, keep)), ctypes.byref(_tsupp(supplier, keep)),
                                 ctypes.byref(_nation(nation, keep)), ctypes.byref(_region(region, keep)),
                                 int(brute), nthreads],
                 ["n_name", "revenue", "count"])


def tpch_q7(customer, orders, lineitem, supplier, nation, brute=False, nthreads=1) -> OracleResult:
    """TPC-H Q7 -> [supp_nation, cust_nation, l_year, revenue (scale 4), count]
    ORDER BY supp_nation, cust_nation, l_year."""
    keep = []
    return _call("orc_tpch_q7", [ctypes.byref(_tcust(customer, keep)), ctypes.byref(_orders(orders, keep)),
                                 ctypes.byref(_lineitem(lineitem, keep)), ctypes.byref(_tsupp(supplier, keep)),
                                 ctypes.byref(_nation(nation, keep)), int(brute), nthreads],
                 ["supp_nation", "cust_nation", "l_year", "revenue", "count"])


def _partsupp(t, keep):
    s = _Partsupp()
    s.n = _n(t)
    s.partkey = _ptr(t["ps_partkey"], P_I32, keep)
    s.suppkey = _ptr(t["ps_suppkey"], P_I32, keep)
    s.supplycost = _ptr(t["ps_supplycost"], P_I64, keep)
    return s


def q9_pmax(nparts: int) -> int:
    """DESIGN.md R19: App F's p_partkey filter for p_name like '%green%' keeps the LIKE's
    selectivity, 5 of 92 colour words: p_partkey <= |part| * 5 // 92."""
    return int(nparts) * 5 // 92


def tpch_q9(part, supplier, lineitem, partsupp, orders, nation, pmax=None, brute=False, nthreads=1) -> OracleResult:
    """TPC-H Q9 (App F) -> [nation, o_year, sum_profit (scale 4), count] ORDER BY nation, o_year desc."""
    keep = []
    pmax = q9_pmax(_n(part)) if pmax is None else int(pmax)
    return _call("orc_tpch_q9", [ctypes.byref(_tpart(part, keep)), ctypes.byref(_tsupp(supplier, keep)),
                                 ctypes.byref(_lineitem(lineitem, keep)), ctypes.byref(_partsupp(partsupp, keep)),
                                 ctypes.byref(_orders(orders, keep)), ctypes.byref(_nation(nation, keep)), pmax,
                                 int(brute), nthreads], ["nation", "o_year", "sum_profit", "count"])


def tpch_q4(orders, lineitem, brute=False, nthreads=1) -> OracleResult:
    """TPC-H Q4 -> [o_orderpriority, order_count] ORDER BY o_orderpriority."""
    keep = []
    return _call("orc_tpch_q4", [ctypes.byref(_orders(orders, keep)), ctypes.byref(_lineitem(lineitem, keep)),
                                 int(brute), nthreads], ["o_orderpriority", "order_count"])


def tpch_q13(customer, orders, brute=False) -> OracleResult:
    """TPC-H Q13 (App F: no LIKE) -> [c_count, custdist] ORDER BY custdist desc, c_count desc."""
    keep = []
    return _call("orc_tpch_q13", [ctypes.byref(_tcust(customer, keep)), ctypes.byref(_orders(orders, keep)),
                                  int(brute)], ["c_count", "custdist"])


def tpch_q17(part, lineitem, brute=False) -> OracleResult:
    """TPC-H Q17 (unnested) -> 1 row [sum_extendedprice (cents), count]; avg_yearly = sum / 7.0."""
    keep = []
    return _call("orc_tpch_q17", [ctypes.byref(_tpart(part, keep)), ctypes.byref(_lineitem(lineitem, keep)),
                                  int(brute)], ["sum_extendedprice", "count"])


def tpch_q18(customer, orders, lineitem, brute=False) -> OracleResult:
    """TPC-H Q18 -> [c_custkey, o_orderkey, o_orderdate, o_totalprice, sum_qty, count]
    ORDER BY o_totalprice desc, o_orderdate, o_orderkey (full result)."""
    keep = []
    return _call("orc_tpch_q18", [ctypes.byref(_tcust(customer, keep)), ctypes.byref(_orders(orders, keep)),
                                  ctypes.byref(_lineitem(lineitem, keep)), int(brute)],
                 ["c_custkey", "o_orderkey", "o_orderdate", "o_totalprice", "sum_qty", "count"])


def tpch_q19(part, lineitem, brute=False, nthreads=1) -> OracleResult:
    """TPC-H Q19 -> 1 row [revenue (scale 4), count]."""
    keep = []
    return _call("orc_tpch_q19", [ctypes.byref(_tpart(part, keep)), ctypes.byref(_lineitem(lineitem, keep)),
                                  int(brute), nthreads], ["revenue", "count"])


def tpch_q21(supplier, orders, lineitem, nation, variant=0, brute=False) -> OracleResult:
    """TPC-H Q21 -> [s_suppkey, numwait] ORDER BY numwait desc, s_suppkey (full result);
    variant 1 = PAPER.md App F's EXISTS in place of NOT EXISTS."""
    keep = []
    return _call("orc_tpch_q21", [int(variant), ctypes.byref(_tsupp(supplier, keep)),
                                  ctypes.byref(_orders(orders, keep)), ctypes.byref(_lineitem(lineitem, keep)),
                                  ctypes.byref(_nation(nation, keep)), int(brute)], ["s_suppkey", "numwait"])


def tpch_q10(customer, orders, lineitem, nation, brute=False, nthreads=1) -> OracleResult:
    """TPC-H Q10 -> [c_custkey, n_name, revenue (scale 4), count] ORDER BY revenue desc (full result)."""
    keep = []
    return _call("orc_tpch_q10", [ctypes.byref(_tcust(customer, keep)), ctypes.byref(_orders(orders, keep)),
                                  ctypes.byref(_lineitem(lineitem, keep)), ctypes.byref(_nation(nation, keep)),
                                  int(brute), nthreads],
                 ["c_custkey", "n_name", "revenue", "count"])


def micro_select(lineorder, x, nthreads=1) -> OracleResult:
    keep = []
    return _call("orc_micro_select", [ctypes.byref(_lineorder(lineorder, keep)), int(x), nthreads], ["revenue"])


def micro_sum(lineorder, x, nthreads=1) -> OracleResult:
    keep = []
    return _call("orc_micro_sum", [ctypes.byref(_lineorder(lineorder, keep)), int(x), nthreads], ["revenue", "count"])


def micro_groupby(lineorder, x, nthreads=1) -> OracleResult:
    keep = []
    return _call("orc_micro_groupby", [ctypes.byref(_lineorder(lineorder, keep)), int(x), nthreads],
                 ["key", "sum", "count"])
