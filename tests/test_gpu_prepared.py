"""Prepared queries (CUDA graphs, include/hq.h): a query step recorded once and replayed
re-executes all of its device work -- a change of the input between launches shows
in the next result -- and every launch equals the oracle."""
import numpy as np
import pytest

import hqgen
import oracle
from paper_conf_sigmod_funkebnmt18_b200 import hq
from paper_conf_sigmod_funkebnmt18_b200.engine import Engine
from paper_conf_sigmod_funkebnmt18_b200.queries import QUERIES

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ctx():
    import torch
    assert torch.cuda.is_available(), "gpu tests need a CUDA device"
    c = hq.Context(0)
    yield c
    c.close()


def _oracle(qname, t):
    return {"ssb_q41": lambda: oracle.ssb_q41(t["lineorder"], t["date"], t["customer"], t["supplier"], t["part"], nthreads=8),
            "ssb_q31": lambda: oracle.ssb_q31(t["lineorder"], t["customer"], t["supplier"], t["date"], nthreads=8),
            "ssb_q11": lambda: oracle.ssb_q1(1, t["lineorder"], t["date"], nthreads=8),
            "ssb_q13": lambda: oracle.ssb_q1(3, t["lineorder"], t["date"], nthreads=8),
            "tpch_q6": lambda: oracle.tpch_q6(t["lineitem"], nthreads=8),
            "tpch_q3": lambda: oracle.tpch_q3(t["tpch_customer"], t["orders"], t["lineitem"]),
            "tpch_q1": lambda: oracle.tpch_q1(t["lineitem"], nthreads=8)}[qname]()


COLS = {"ssb_q41": ["d_year", "c_nation", "profit", "count"],
        "ssb_q31": ["c_nation", "s_nation", "d_year", "revenue", "count"],
        "ssb_q11": ["revenue", "count"], "ssb_q13": ["revenue", "count"], "tpch_q6": ["revenue", "count"],
        "tpch_q3": ["l_orderkey", "o_orderdate", "o_shippriority", "revenue", "count"],
        "tpch_q1": ["l_returnflag", "l_linestatus", "sum_qty", "sum_base_price", "sum_disc_price", "sum_charge",
                    "count_order"]}


@pytest.mark.parametrize("sf", [0.01, 1.0])
@pytest.mark.parametrize("qname", list(COLS))
def test_prepared_matches_oracle(ctx, qname, sf):
    q = QUERIES[qname]
    tabs = hqgen.SSB_TABLES if q.bench == "ssb" else hqgen.TPCH_TABLES
    host = {t: hqgen.generate(t, sf, columns=q.columns[t]) for t in q.columns if t in tabs}
    E = Engine(ctx, {t: ctx.load_columns(host[t]) for t in q.columns})
    o = _oracle(qname, host)
    pq = E.prepare(q)
    want = o.rows(COLS[qname])[:10] if qname == "tpch_q3" else o.rows(COLS[qname])
    for _ in range(3):
        l0 = ctx.launches()
        g = pq.execute()
        assert g.rows(COLS[qname]) == want
        if qname != "tpch_q3":  # (Q3's qualifying = lineitem rows reaching its GROUP BY)
            assert g.qualifying == o.qualifying
        assert ctx.launches() - l0 >= 2  # the builds, the pipeline and the finalize ran again
    if qname == "tpch_q1":
        np.testing.assert_allclose(g.columns["avg_disc"], o.columns["avg_disc"], rtol=1e-9, atol=0)
    pq.close()


def test_prepared_reexecutes_on_new_input(ctx):
    """The graph reads the borrowed fact columns at every launch: values changed in
    place between launches change the next result exactly as the oracle says."""
    import torch
    sf = 0.1
    host = {t: hqgen.generate(t, sf) for t in hqgen.SSB_TABLES}
    q = QUERIES["ssb_q41"]
    dev = {c: torch.from_numpy(host["lineorder"][c]).cuda() for c in q.columns["lineorder"]}
    tabs = {t: ctx.load_columns({c: host[t][c] for c in cs}) for t, cs in q.columns.items() if t != "lineorder"}
    tabs["lineorder"] = ctx.load_columns(dev)
    E = Engine(ctx, tabs)
    pq = E.prepare(q)
    cols = COLS["ssb_q41"]
    for k in range(3):
        g = pq.execute()
        lo = {c: v.cpu().numpy() for c, v in dev.items()}
        o = oracle.ssb_q41(lo, host["date"], host["customer"], host["supplier"], host["part"], nthreads=8)
        assert g.rows(cols) == o.rows(), k
        dev["lo_revenue"].add_(1000 * (k + 1))  # a new input for the next launch
        torch.cuda.synchronize()
    pq.close()


def test_not_capturable_query_raises_and_context_recovers(ctx):
    """Multi-pass execution reads its qualifying count on the host between its kernels:
    the capture fails with HQ_ERR_STATE and the context keeps working eagerly."""
    sf = 0.01
    host = {t: hqgen.generate(t, sf) for t in hqgen.TPCH_TABLES}
    q = QUERIES["tpch_q3"]
    Em = Engine(ctx, {t: ctx.load_columns({c: host[t][c] for c in cs}) for t, cs in q.columns.items()},
                exec_mode=hq.EXEC_MULTIPASS)
    with pytest.raises(hq.HQError) as e:
        Em.prepare(q)
    assert e.value.code == hq.HQ_ERR_STATE
    E = Engine(ctx, Em.tables)
    o = oracle.tpch_q3(host["tpch_customer"], host["orders"], host["lineitem"])
    g = q.execute(E)
    assert g.rows(["l_orderkey", "o_orderdate", "o_shippriority", "revenue", "count"]) == \
        o.rows(["l_orderkey", "o_orderdate", "o_shippriority", "revenue", "count"])[:10]


def test_prepared_tpch_q3_detects_a_changed_result_count(ctx):
    """TPC-H Q3's captured step views the materialised orders side with its row count
    cached from the eager run: when the orders change in place so that the count differs,
    the next launch raises HQ_ERR_STATE (the build checks the device count) instead of
    answering from a wrong view; an eager run afterwards is exact again."""
    import torch
    sf = 0.01
    host = {t: hqgen.generate(t, sf) for t in ("lineitem", "orders", "tpch_customer")}
    q = QUERIES["tpch_q3"]
    dev = {c: torch.from_numpy(host["orders"][c]).cuda() for c in q.columns["orders"]}
    tabs = {t: ctx.load_columns({c: host[t][c] for c in cs}) for t, cs in q.columns.items() if t != "orders"}
    tabs["orders"] = ctx.load_columns(dev)
    E = Engine(ctx, tabs)
    cols = COLS["tpch_q3"]
    pq = E.prepare(q)
    o = oracle.tpch_q3(host["tpch_customer"], host["orders"], host["lineitem"])
    assert pq.execute().rows(cols) == o.rows(cols)[:10]
    dev["o_orderdate"][:200] = 19920101  # more orders pass o_orderdate < 1995-03-15
    torch.cuda.synchronize()
    with pytest.raises(hq.HQError) as e:
        pq.execute()
    assert e.value.code == hq.HQ_ERR_STATE
    pq.close()
    ho = {c: dev[c].cpu().numpy() for c in dev}
    o2 = oracle.tpch_q3(host["tpch_customer"], ho, host["lineitem"])
    for _ in range(2):  # the stale entries were dropped: counted afresh, then cached again
        assert q.execute(E).rows(cols) == o2.rows(cols)[:10]
