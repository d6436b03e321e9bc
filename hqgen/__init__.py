"""hqgen -- deterministic TPC-H / SSB shaped input generator (Python side).

The single module shared by the oracle (``oracle/``) and the CUDA path
(``paper_conf_sigmod_funkebnmt18_b200``).  It generates columns only; it holds
none of the query arithmetic.  Recipe: SURVEY.md §8(d.1), DESIGN.md "Input
recipe".  Values are pure functions of (seed, sf, table, column, row), so any
row range is generated independently (partition invariance, used for the
multi-GPU range partitioning of SURVEY.md §8(e)).

Strings are order-preserving int8 dictionary codes:
the code order equals the string order, so equality/IN/range predicates on
strings become integer predicates on codes.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from typing import Dict, Iterable, Optional, Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libhqgen.so")

DEFAULT_SEED = 20180610

# ---- order-preserving dictionaries ---------------------------------------
REGIONS = ["AFRICA", "AMERICA", "ASIA", "EUROPE", "MIDDLE EAST"]
NATIONS = [
    "ALGERIA", "ARGENTINA", "BRAZIL", "CANADA", "CHINA", "EGYPT", "ETHIOPIA",
    "FRANCE", "GERMANY", "INDIA", "INDONESIA", "IRAN", "IRAQ", "JAPAN", "JORDAN",
    "KENYA", "MOROCCO", "MOZAMBIQUE", "PERU", "ROMANIA", "RUSSIA", "SAUDI ARABIA",
    "UNITED KINGDOM", "UNITED STATES", "VIETNAM",
]
NATION_REGION = [0, 1, 1, 1, 2, 4, 0, 3, 3, 2, 2, 4, 4, 2, 4, 0, 0, 0, 1, 3, 3, 4, 3, 1, 2]
MFGRS = ["MFGR#1", "MFGR#2", "MFGR#3", "MFGR#4", "MFGR#5"]
MKTSEGMENTS = ["AUTOMOBILE", "BUILDING", "FURNITURE", "HOUSEHOLD", "MACHINERY"]
RETURNFLAGS = ["A", "N", "R"]
LINESTATUS = ["F", "O"]
ORDERSTATUS = ["F", "O", "P"]
ORDERPRIORITIES = ["1-URGENT", "2-HIGH", "3-MEDIUM", "4-NOT SPECIFIED", "5-LOW"]
SHIPMODES = ["AIR", "FOB", "MAIL", "RAIL", "REG AIR", "SHIP", "TRUCK"]
SHIPINSTRUCTS = ["COLLECT COD", "DELIVER IN PERSON", "NONE", "TAKE BACK RETURN"]
# TPC-H p_brand 'Brand#MN' (M, N in 1..5) = (M-1)*5 + N-1; p_container = the 40
# 'SIZE TYPE' strings (TPC-H 4.2.2.13) in string order
BRANDS = [f"Brand#{m}{n}" for m in range(1, 6) for n in range(1, 6)]
CONTAINERS = sorted(f"{a} {b}" for a in ["SM", "LG", "MED", "JUMBO", "WRAP"]
                    for b in ["CASE", "BOX", "BAG", "JAR", "PKG", "PACK", "CAN", "DRUM"])


def code(dictionary: Sequence[str], s: str) -> int:
    return list(dictionary).index(s)


# SSB strings with generated codes (hqgen.cpp): city = nation * 10 + digit, the
# city name being the nation's first 9 characters (space padded) + the digit;
# p_category 'MFGR#mc' = (m-1)*5 + (c-1); p_brand1 'MFGR#mcbb' = category*40 + bb-1.
# City and category code orders equal the string orders; brand codes follow
# (category, brand number) -- the string order differs only where a one-digit
# and a two-digit brand number of one category meet ('MFGR#222' < 'MFGR#2221'),
# which no SSB predicate here compares (Q2.2's BETWEEN spans brands 21..28).
def city_name(c: int) -> str:
    return NATIONS[c // 10][:9].ljust(9) + str(c % 10)


def city_code(s: str) -> int:
    for n, name in enumerate(NATIONS):
        if name[:9].ljust(9) == s[:9]:
            return n * 10 + int(s[9])
    raise KeyError(s)


def category_name(c: int) -> str:
    return f"MFGR#{c // 5 + 1}{c % 5 + 1}"


def category_code(s: str) -> int:
    return (int(s[5]) - 1) * 5 + int(s[6]) - 1


def brand_name(b: int) -> str:
    return f"{category_name(b // 40)}{b % 40 + 1}"


def brand_code(s: str) -> int:
    return category_code(s[:7]) * 40 + int(s[7:]) - 1


# ---- table schemas (mirror hqgen.h) ---------------------------------------
SSB_LINEORDER, SSB_DATE, SSB_CUSTOMER, SSB_SUPPLIER, SSB_PART = 1, 2, 3, 4, 5
TPCH_LINEITEM, TPCH_ORDERS, TPCH_CUSTOMER, TPCH_SUPPLIER, TPCH_NATION, TPCH_REGION = 11, 12, 13, 14, 15, 16
TPCH_PART, TPCH_PARTSUPP = 17, 18

SCHEMAS: Dict[int, list] = {
    SSB_LINEORDER: [("lo_orderkey", "i4"), ("lo_linenumber", "i4"), ("lo_custkey", "i4"),
                    ("lo_partkey", "i4"), ("lo_suppkey", "i4"), ("lo_orderdate", "i4"),
                    ("lo_quantity", "i4"), ("lo_extendedprice", "i4"), ("lo_discount", "i4"),
                    ("lo_revenue", "i4"), ("lo_supplycost", "i4"), ("lo_tax", "i4")],
    SSB_DATE: [("d_datekey", "i4"), ("d_year", "i4"), ("d_yearmonthnum", "i4"),
               ("d_weeknuminyear", "i4")],
    SSB_CUSTOMER: [("c_custkey", "i4"), ("c_nation", "i1"), ("c_region", "i1"), ("c_city", "i4")],
    SSB_SUPPLIER: [("s_suppkey", "i4"), ("s_nation", "i1"), ("s_region", "i1"), ("s_city", "i4")],
    SSB_PART: [("p_partkey", "i4"), ("p_mfgr", "i1"), ("p_category", "i1"), ("p_brand1", "i4")],
    TPCH_LINEITEM: [("l_orderkey", "i4"), ("l_partkey", "i4"), ("l_quantity", "i8"),
                    ("l_extendedprice", "i8"), ("l_discount", "i8"), ("l_tax", "i8"),
                    ("l_returnflag", "i1"), ("l_linestatus", "i1"), ("l_shipdate", "i4"),
                    ("l_receiptdate", "i4"), ("l_linenumber", "i4"), ("l_suppkey", "i4"),
                    ("l_commitdate", "i4"), ("l_shipmode", "i1"), ("l_shipinstruct", "i1")],
    TPCH_ORDERS: [("o_orderkey", "i4"), ("o_custkey", "i4"), ("o_orderdate", "i4"),
                  ("o_shippriority", "i4"), ("o_orderpriority", "i1"), ("o_totalprice", "i8"),
                  ("o_orderstatus", "i1")],
    TPCH_CUSTOMER: [("c_custkey", "i4"), ("c_mktsegment", "i1"), ("c_nationkey", "i1")],
    TPCH_SUPPLIER: [("s_suppkey", "i4"), ("s_nationkey", "i1")],
    TPCH_NATION: [("n_nationkey", "i1"), ("n_regionkey", "i1")],
    TPCH_REGION: [("r_regionkey", "i1")],
    TPCH_PART: [("p_partkey", "i4"), ("p_brand", "i1"), ("p_container", "i1"), ("p_size", "i4")],
    TPCH_PARTSUPP: [("ps_partkey", "i4"), ("ps_suppkey", "i4"), ("ps_supplycost", "i8")],
}
TABLE_NAMES = {
    "lineorder": SSB_LINEORDER, "date": SSB_DATE, "customer": SSB_CUSTOMER,
    "supplier": SSB_SUPPLIER, "part": SSB_PART, "lineitem": TPCH_LINEITEM,
    "orders": TPCH_ORDERS, "tpch_customer": TPCH_CUSTOMER, "tpch_supplier": TPCH_SUPPLIER,
    "nation": TPCH_NATION, "region": TPCH_REGION, "tpch_part": TPCH_PART, "partsupp": TPCH_PARTSUPP,
}
SSB_TABLES = ["lineorder", "date", "customer", "supplier", "part"]
TPCH_TABLES = ["lineitem", "orders", "tpch_customer", "tpch_supplier", "nation", "region", "tpch_part", "partsupp"]


def _build() -> None:
    src = os.path.join(_HERE, "hqgen.cpp")
    subprocess.check_call(["g++", "-O2", "-std=c++17", "-shared", "-fPIC", "-pthread",
                           "-o", _SO, src])


_lib = None


def lib():
    global _lib
    if _lib is None:
        src = os.path.join(_HERE, "hqgen.cpp")
        if not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(src):
            _build()
        L = ctypes.CDLL(_SO)
        L.hqg_table_rows.restype = ctypes.c_int64
        L.hqg_table_rows.argtypes = [ctypes.c_int, ctypes.c_double, ctypes.c_uint64, ctypes.c_int]
        L.hqg_generate.restype = ctypes.c_int
        L.hqg_generate.argtypes = [ctypes.c_int, ctypes.c_double, ctypes.c_uint64, ctypes.c_int64,
                                   ctypes.c_int64, ctypes.c_int, ctypes.POINTER(ctypes.c_int32),
                                   ctypes.POINTER(ctypes.c_void_p), ctypes.c_int]
        L.hqg_date_from_day.restype = ctypes.c_int32
        L.hqg_date_from_day.argtypes = [ctypes.c_int32]
        L.hqg_line_row_of_order.restype = ctypes.c_int64
        L.hqg_line_row_of_order.argtypes = [ctypes.c_int, ctypes.c_double, ctypes.c_uint64, ctypes.c_int64,
                                            ctypes.c_int]
        _lib = L
    return _lib


def table_id(table) -> int:
    return TABLE_NAMES[table] if isinstance(table, str) else int(table)


def table_rows(table, sf: float, seed: int = DEFAULT_SEED, nthreads: int = 0) -> int:
    n = lib().hqg_table_rows(table_id(table), float(sf), int(seed), int(nthreads))
    if n < 0:
        raise ValueError(f"bad table/sf {table} {sf}")
    return int(n)


def line_row_of_order(table, sf: float, order: int, seed: int = DEFAULT_SEED, nthreads: int = 0) -> int:
    """First row of order `order`'s lines in a line table (lineorder / lineitem)."""
    r = lib().hqg_line_row_of_order(table_id(table), float(sf), int(seed), int(order), int(nthreads))
    if r < 0:
        raise ValueError(f"bad line table / sf / order {table} {sf} {order}")
    return int(r)


def copartition(line_table, order_table, sf: float, rank: int, world: int, seed: int = DEFAULT_SEED):
    """Rank `rank`'s share of a line table and its order table partitioned together by
    order (orderkey): ((order rows a, b), (line rows la, lb)) with the lines of orders
    [a, b) exactly the line rows [la, lb)."""
    no = table_rows(order_table, sf, seed)
    a, b = no * rank // world, no * (rank + 1) // world
    return (a, b), (line_row_of_order(line_table, sf, a, seed), line_row_of_order(line_table, sf, b, seed))


def column_names(table) -> list:
    return [c for c, _ in SCHEMAS[table_id(table)]]


def generate(table, sf: float, seed: int = DEFAULT_SEED, columns: Optional[Iterable[str]] = None,
             row_range: Optional[tuple] = None, nthreads: int = 0,
             out: Optional[Dict[str, np.ndarray]] = None) -> Dict[str, np.ndarray]:
    """Generate columns of `table` for rows [a, b) (default: all rows).

    Returns {column name: numpy array}.  ``out`` may supply preallocated
    (e.g. pinned) numpy arrays to fill in place.
    """
    tid = table_id(table)
    schema = SCHEMAS[tid]
    names = [c for c, _ in schema]
    cols = list(columns) if columns is not None else names
    n = table_rows(tid, sf, seed, nthreads)
    a, b = (0, n) if row_range is None else (int(row_range[0]), int(row_range[1]))
    if not (0 <= a <= b <= n):
        raise ValueError(f"row range {a, b} outside [0, {n}]")
    res: Dict[str, np.ndarray] = {}
    ids, ptrs = [], []
    for c in cols:
        k = names.index(c)
        dt = np.dtype(schema[k][1])
        arr = out[c] if out is not None and c in out else np.empty(b - a, dtype=dt)
        assert arr.dtype == dt and arr.shape == (b - a,) and arr.flags.c_contiguous
        res[c] = arr
        ids.append(k)
        ptrs.append(arr.ctypes.data)
    if cols and b > a:
        ids_c = (ctypes.c_int32 * len(ids))(*ids)
        ptr_c = (ctypes.c_void_p * len(ptrs))(*ptrs)
        rc = lib().hqg_generate(tid, float(sf), int(seed), a, b, len(ids), ids_c, ptr_c, int(nthreads))
        if rc != 0:
            raise RuntimeError(f"hqg_generate failed rc={rc}")
    return res


def date_from_day(d: int) -> int:
    return int(lib().hqg_date_from_day(int(d)))
