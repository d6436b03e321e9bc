"""Resolution:WE (App C "Work-Efficient Reduction", Fig 24; Table 4
A3/B3/C3 with work-efficient local resolution): the generated fused kernel's per-tile
Blelloch trees (B3-WE reduce, A3-WE exclusive scan, C3-WE bitonic sort + segmented
scan + atomic hash reduce) give the oracle's results, element by element."""
import numpy as np
import pytest

import hqgen
import oracle
from paper_conf_sigmod_funkebnmt18_b200 import hq
from paper_conf_sigmod_funkebnmt18_b200.engine import Engine, PlanBuilder
from paper_conf_sigmod_funkebnmt18_b200.queries import QUERIES

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ctx():
    import torch
    assert torch.cuda.is_available(), "gpu tests need a CUDA device"
    c = hq.Context(0)
    yield c
    c.close()


@pytest.fixture(scope="module", params=[0.01, 1.0])
def data(request):
    sf = request.param
    return sf, {t: hqgen.generate(t, sf) for t in hqgen.SSB_TABLES}, {t: hqgen.generate(t, sf) for t in hqgen.TPCH_TABLES}


def run(ctx, qname, host, resolution=hq.RES_WE, **kw):
    q = QUERIES[qname]
    tables = {t: ctx.load_columns({c: host[t][c] for c in cols}) for t, cols in q.columns.items()}
    return q.execute(Engine(ctx, tables, resolution=resolution), **kw)


COLS = {"ssb_q41": ["d_year", "c_nation", "profit", "count"],
        "ssb_q31": ["c_nation", "s_nation", "d_year", "revenue", "count"],
        "ssb_q11": ["revenue", "count"], "tpch_q6": ["revenue", "count"],
        "tpch_q1": ["l_returnflag", "l_linestatus", "sum_qty", "sum_base_price", "sum_disc_price", "sum_charge",
                    "count_order"],
        "tpch_q3": ["l_orderkey", "o_orderdate", "o_shippriority", "revenue", "count"]}


@pytest.mark.parametrize("qname", list(COLS))
def test_we_queries_match_oracle(ctx, data, qname):
    sf, ssb, tpch = data
    nt = 8
    o = {"ssb_q41": lambda: oracle.ssb_q41(ssb["lineorder"], ssb["date"], ssb["customer"], ssb["supplier"], ssb["part"],
                                           nthreads=nt),
         "ssb_q31": lambda: oracle.ssb_q31(ssb["lineorder"], ssb["customer"], ssb["supplier"], ssb["date"], nthreads=nt),
         "ssb_q11": lambda: oracle.ssb_q1(1, ssb["lineorder"], ssb["date"], nthreads=nt),
         "tpch_q6": lambda: oracle.tpch_q6(tpch["lineitem"], nthreads=nt),
         "tpch_q1": lambda: oracle.tpch_q1(tpch["lineitem"], nthreads=nt),
         "tpch_q3": lambda: oracle.tpch_q3(tpch["tpch_customer"], tpch["orders"], tpch["lineitem"], nthreads=nt)}[qname]()
    host = ssb if QUERIES[qname].bench == "ssb" else tpch
    g = run(ctx, qname, host, **({"limit": 0} if qname == "tpch_q3" else {}))
    assert g.rows(COLS[qname]) == o.rows(COLS[qname])
    assert g.qualifying == o.qualifying
    if qname == "tpch_q1":
        for c in ("avg_qty", "avg_price", "avg_disc"):
            np.testing.assert_allclose(g.columns[c], o.columns[c], rtol=1e-9, atol=0)


def test_we_materialise_matches_oracle(ctx, data):
    """A3-WE: the joined tuples of SSB Q3.1 as a multiset (reading R1), and the write
    positions dense (every slot written once: the sorted multiset has the oracle's size)."""
    sf, ssb, _ = data
    g = run(ctx, "ssb_q31_mat", ssb)
    o = oracle.ssb_q31_mat(ssb["lineorder"], ssb["customer"], ssb["supplier"], ssb["date"], nthreads=8)
    assert sorted(g.rows(["c_nation", "s_nation", "d_year", "lo_revenue"])) == o.rows()


def test_we_micro_queries(ctx):
    """Exp 1 / App G.1 / Exp 2 query shapes (Fig 16, Fig 26) under WE against the oracle,
    including MIN / MAX in the C3-WE segmented scan and a hash group-by."""
    ssb = {t: hqgen.generate(t, 0.1) for t in ("lineorder",)}
    lo = ssb["lineorder"]
    for x in (0, 5, 25):
        g = run(ctx, "micro_select", ssb, x=x)
        np.testing.assert_array_equal(np.sort(g.columns["revenue"]), oracle.micro_select(lo, x).columns["revenue"])
        s = run(ctx, "micro_sum", ssb, x=x)
        assert s.rows(["revenue", "count"]) == oracle.micro_sum(lo, x).rows(["revenue", "count"])
    for x in (2, 7, 1000, 16384):
        g = run(ctx, "micro_groupby", ssb, x=x)
        assert g.rows(["k", "sum", "count"]) == oracle.micro_groupby(lo, x).rows(["key", "sum", "count"])


def test_we_min_max_hash_groups(ctx):
    """C3-WE with MIN / MAX aggregates into a global hash table (TPC-H Q18's first
    pipeline shape): min/max per group against numpy over the same rows."""
    rng = np.random.default_rng(5)
    n = 300_000
    k = rng.integers(0, 5000, n).astype(np.int32)
    v = rng.integers(-10**9, 10**9, n).astype(np.int64)
    t = ctx.load_columns({"k": k, "v": v})
    pb = PlanBuilder(t)
    pb.aggregate(keys=[("k", 0, 1 << 31)], aggs=[("min", "v"), ("max", "v"), ("sum", "v"), ("count", None)],
                 order=[("k", False)], group_capacity=8192, agg_names=["mn", "mx", "s", "c"])
    pb.plan.resolution = hq.RES_WE
    cols = ctx.run(pb.plan, keep=pb.keep).fetch()
    keys = np.unique(k)
    order = np.argsort(k, kind="stable")
    ks, vs = k[order], v[order]
    starts = np.r_[0, np.nonzero(np.diff(ks))[0] + 1]
    np.testing.assert_array_equal(cols[0], keys)
    np.testing.assert_array_equal(cols[1], np.minimum.reduceat(vs, starts))
    np.testing.assert_array_equal(cols[2], np.maximum.reduceat(vs, starts))
    np.testing.assert_array_equal(cols[3], np.add.reduceat(vs, starts))
    np.testing.assert_array_equal(cols[4], np.diff(np.r_[starts, n]))


def test_we_only_fused(ctx):
    ssb = {t: hqgen.generate(t, 0.01) for t in hqgen.SSB_TABLES}
    q = QUERIES["ssb_q11"]
    tables = {t: ctx.load_columns({c: ssb[t][c] for c in cols}) for t, cols in q.columns.items()}
    for em in (hq.EXEC_FUSED_INTERP, hq.EXEC_MULTIPASS):
        with pytest.raises(hq.HQError) as e:
            q.execute(Engine(ctx, tables, exec_mode=em, resolution=hq.RES_WE))
        assert e.value.code == hq.HQ_ERR_UNSUPPORTED
