"""Generator tests (CPU): determinism, partition invariance, closed-form
distributions.  SURVEY.md §4.2 layer 1, §8(d.1)."""
import datetime

import numpy as np
import pytest

import hqgen

EPOCH = datetime.date(1992, 1, 1)


def ymd(day):
    d = EPOCH + datetime.timedelta(days=int(day))
    return d.year * 10000 + d.month * 100 + d.day


@pytest.mark.parametrize("table", ["lineorder", "lineitem", "orders", "customer", "part", "date"])
def test_deterministic(table):
    a = hqgen.generate(table, 0.01, seed=7)
    b = hqgen.generate(table, 0.01, seed=7, nthreads=3)
    c = hqgen.generate(table, 0.01, seed=8)
    for k in a:
        np.testing.assert_array_equal(a[k], b[k])
    if table != "date":
        assert any(not np.array_equal(a[k], c[k]) for k in a)


@pytest.mark.parametrize("table", ["lineorder", "lineitem", "orders", "tpch_customer", "supplier", "tpch_part", "partsupp"])
def test_partition_invariance(table):
    full = hqgen.generate(table, 0.01)
    n = hqgen.table_rows(table, 0.01)
    rng = np.random.default_rng(0)
    cuts = sorted(set([0, n] + rng.integers(0, n, 6).tolist()))
    for a, b in zip(cuts[:-1], cuts[1:]):
        part = hqgen.generate(table, 0.01, row_range=(a, b))
        for k in full:
            np.testing.assert_array_equal(part[k], full[k][a:b])


def test_row_counts_and_keys():
    assert hqgen.table_rows("date", 1) == 2557
    assert hqgen.table_rows("customer", 1) == 30000
    assert hqgen.table_rows("supplier", 10) == 20000
    assert hqgen.table_rows("part", 10) == 200000 * (1 + 3)
    assert hqgen.table_rows("orders", 0.01) == 15000
    lo = hqgen.generate("lineorder", 0.01, columns=["lo_orderkey", "lo_linenumber"])
    # 1..7 lines per order, mean 4 -> ~6M*SF rows
    n = len(lo["lo_orderkey"])
    assert abs(n / 15000 - 4.0) < 0.1
    assert lo["lo_linenumber"].min() == 1 and lo["lo_linenumber"].max() == 7
    # sparse TPC-H order keys 32*(i/8)+(i%8)+1
    keys = np.unique(lo["lo_orderkey"])
    i = np.arange(15000)
    np.testing.assert_array_equal(keys, 32 * (i // 8) + (i % 8) + 1)


def test_date_dimension_matches_calendar():
    d = hqgen.generate("date", 1)
    days = np.arange(2557)
    np.testing.assert_array_equal(d["d_datekey"], [ymd(x) for x in days])
    assert d["d_datekey"][-1] == 19981231
    np.testing.assert_array_equal(d["d_year"], d["d_datekey"] // 10000)
    np.testing.assert_array_equal(d["d_yearmonthnum"], d["d_datekey"] // 100)
    # week 6 of every year = 7 days (SURVEY.md §8(c.4) Q1.3 closed form 7/2557)
    assert ((d["d_weeknuminyear"] == 6) & (d["d_year"] == 1994)).sum() == 7


def test_dictionaries():
    assert sorted(hqgen.NATIONS) == hqgen.NATIONS and sorted(hqgen.REGIONS) == hqgen.REGIONS
    for r in range(5):
        assert hqgen.NATION_REGION.count(r) == 5
    c = hqgen.generate("customer", 1)
    np.testing.assert_array_equal(c["c_region"], np.asarray(hqgen.NATION_REGION)[c["c_nation"]])


def _within(k, n, p, design=1.0, sig=5.0):
    sd = np.sqrt(p * (1 - p) / n * design)
    return abs(k / n - p) <= sig * sd


def test_ssb_selectivities_closed_form():
    """Q1.1 365/2557*3/11*24/50, Q3.1 1/5*1/5*2192/2557, Q4.1 1/5*1/5*2/5."""
    sf = 1
    lo = hqgen.generate("lineorder", sf, columns=["lo_orderdate", "lo_quantity", "lo_discount",
                                                  "lo_custkey", "lo_suppkey", "lo_partkey"])
    c = hqgen.generate("customer", sf)
    s = hqgen.generate("supplier", sf)
    p = hqgen.generate("part", sf)
    n = len(lo["lo_orderdate"])
    year = lo["lo_orderdate"] // 10000
    # orderdate is shared by the 1..7 lines of an order: design effect E[k^2]/E[k] = 5
    q11 = ((year == 1993) & (lo["lo_discount"] >= 1) & (lo["lo_discount"] <= 3) & (lo["lo_quantity"] < 25)).sum()
    assert _within(q11, n, 365 / 2557 * 3 / 11 * 24 / 50, design=5)
    # dimension region/mfgr shares are binomial samples around 1/5 and 2/5 ...
    fc = (c["c_region"] == 2).mean()
    fs = (s["s_region"] == 2).mean()
    assert _within(fc * len(c["c_region"]), len(c["c_region"]), 0.2)
    assert _within(fs * len(s["s_region"]), len(s["s_region"]), 0.2)
    assert _within((p["p_mfgr"] <= 1).sum(), len(p["p_mfgr"]), 0.4)
    # ... and foreign keys are uniform, so the star-join selectivity is their product
    creg = c["c_region"][lo["lo_custkey"] - 1]
    sreg = s["s_region"][lo["lo_suppkey"] - 1]
    q31 = ((creg == 2) & (sreg == 2) & (year <= 1997)).sum()
    assert _within(q31, n, fc * fs * 2192 / 2557, design=5, sig=6)
    pm = p["p_mfgr"][lo["lo_partkey"] - 1]
    q41 = ((creg == 1) & (sreg == 1) & (pm <= 1)).sum()
    p41 = (c["c_region"] == 1).mean() * (s["s_region"] == 1).mean() * (p["p_mfgr"] <= 1).mean()
    assert _within(q41, n, p41, design=5, sig=6)


def test_tpch_lineitem_rules():
    li = hqgen.generate("lineitem", 0.1)
    o = hqgen.generate("orders", 0.1)
    n = len(li["l_orderkey"])
    # l_shipdate = o_orderdate + U[1,121]; receipt = ship + U[1,30]
    okey_to_date = dict(zip(o["o_orderkey"].tolist(), o["o_orderdate"].tolist()))
    to_day = lambda v: (datetime.date(v // 10000, v // 100 % 100, v % 100) - EPOCH).days
    idx = np.random.default_rng(1).integers(0, n, 2000)
    for i in idx:
        od = to_day(okey_to_date[int(li["l_orderkey"][i])])
        sd = to_day(int(li["l_shipdate"][i]))
        rd = to_day(int(li["l_receiptdate"][i]))
        assert 1 <= sd - od <= 121 and 1 <= rd - sd <= 30
        cur = to_day(19950617)
        rf, ls = int(li["l_returnflag"][i]), int(li["l_linestatus"][i])
        assert (rf == 1) == (rd > cur)
        assert (ls == 1) == (sd > cur)
    assert li["l_quantity"].min() == 100 and li["l_quantity"].max() == 5000
    assert li["l_discount"].max() == 10 and li["l_tax"].max() == 8
    # extendedprice = quantity * retailprice(partkey) in cents
    pk = li["l_partkey"].astype(np.int64)
    rp = 90000 + (pk // 10) % 20001 + 100 * (pk % 1000)
    np.testing.assert_array_equal(li["l_extendedprice"], li["l_quantity"] // 100 * rp)
    # group mix vs TPC-H answer set shares (approximate)
    key = li["l_returnflag"].astype(int) * 2 + li["l_linestatus"]
    share = np.bincount(key, minlength=6) / n
    assert abs(share[0] - 0.246) < 0.02 and abs(share[4] - 0.246) < 0.02   # A/F, R/F
    assert abs(share[3] - 0.487) < 0.03                                     # N/O
    assert share[2] < 0.03                                                  # N/F


def test_tpch_derived_columns():
    """Columns of the TPC-H Q4/Q9/Q13/Q17/Q18/Q19/Q21 plans (TPC-H 4.2.3 rules as
    DESIGN.md §3 states them), checked against the lines with pandas."""
    import pandas as pd
    sf = 0.05
    li = pd.DataFrame(hqgen.generate("lineitem", sf))
    o = pd.DataFrame(hqgen.generate("orders", sf))
    p = pd.DataFrame(hqgen.generate("tpch_part", sf))
    ps = pd.DataFrame(hqgen.generate("partsupp", sf))
    ns = hqgen.table_rows("tpch_supplier", sf)
    to_day = lambda v: (pd.to_datetime(v.astype(str), format="%Y%m%d") - pd.Timestamp(EPOCH)).dt.days
    j = li.merge(o, left_on="l_orderkey", right_on="o_orderkey")
    d = to_day(j.l_commitdate) - to_day(j.o_orderdate)
    assert d.min() == 30 and d.max() == 90
    # o_totalprice = sum of the lines' extendedprice * (1 + tax) * (1 - discount), per line in cents
    j = j.assign(charge=j.l_extendedprice * (100 + j.l_tax) * (100 - j.l_discount) // 10000,
                 open=(j.l_linestatus == 1).astype(int), one=1)
    g = j.groupby("o_orderkey").agg(tp=("charge", "sum"), op=("open", "sum"), n=("one", "sum"),
                                    o_totalprice=("o_totalprice", "first"), st=("o_orderstatus", "first"))
    assert (g.tp == g.o_totalprice).all()
    exp = np.where(g.op == 0, 0, np.where(g.op == g.n, 1, 2))            # F, O, P
    assert (g.st.values == exp).all()
    assert len(g) == len(o)                                             # every order has lines
    assert set(o.o_orderpriority) == set(range(5)) and set(li.l_shipmode) == set(range(7))
    assert set(li.l_shipinstruct) == set(range(4))
    # part: brand / container / size domains; partsupp: 4 distinct suppliers per part, and
    # every (l_partkey, l_suppkey) is one partsupp row
    assert set(p.p_brand) == set(range(25)) and set(p.p_container) == set(range(40))
    assert p.p_size.min() == 1 and p.p_size.max() == 50 and (p.p_partkey == np.arange(1, len(p) + 1)).all()
    assert len(ps) == 4 * len(p) and (ps.groupby("ps_partkey").ps_suppkey.nunique() == 4).all()
    assert ps.ps_suppkey.between(1, ns).all() and ps.ps_supplycost.between(100, 100000).all()
    m = li.merge(ps, left_on=["l_partkey", "l_suppkey"], right_on=["ps_partkey", "ps_suppkey"])
    assert len(m) == len(li)
    assert hqgen.BRANDS[hqgen.code(hqgen.BRANDS, "Brand#23")] == "Brand#23" and hqgen.BRANDS == sorted(hqgen.BRANDS)
    assert len(hqgen.CONTAINERS) == 40 and hqgen.CONTAINERS == sorted(hqgen.CONTAINERS)


@pytest.mark.parametrize("line,order", [("lineitem", "orders"), ("lineorder", None)])
def test_copartition_by_order(line, order):
    """hqgen.copartition: rank r's line rows are exactly the lines of its orders (the
    ranks' line ranges tile the table; every line's orderkey is one of its rank's
    orders), and line_row_of_order is the first row carrying the order's key."""
    sf = 0.01
    key = "l_orderkey" if line == "lineitem" else "lo_orderkey"
    lk = hqgen.generate(line, sf, columns=[key])[key]
    first = {}
    for i, k in enumerate(lk.tolist()):
        first.setdefault(k, i)
    ks = sorted(first)
    for j in (0, 1, 7, 8, 9, len(ks) // 2, len(ks) - 1):
        assert hqgen.line_row_of_order(line, sf, j) == first[ks[j]]
    assert hqgen.line_row_of_order(line, sf, len(ks)) == len(lk)
    if order is None:
        return
    ok = hqgen.generate(order, sf, columns=["o_orderkey"])["o_orderkey"]
    for world in (1, 2, 3, 8):
        end = 0
        for r in range(world):
            (a, b), (la, lb) = hqgen.copartition(line, order, sf, r, world)
            assert la == end
            end = lb
            assert np.isin(lk[la:lb], ok[a:b]).all()
            assert set(ok[a:b].tolist()) >= set(lk[la:lb].tolist())
        assert end == len(lk)
