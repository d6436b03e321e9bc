"""GPU parity of batch processing (SURVEY.md §8(f) f4 i; §3, Exp 5
P:1708-1732): the fact table stays in (pinned) host memory and streams through the
compound kernel in blocks over a double-buffered device ring.  The result must equal
the oracle element by element for every sink kind, for block sizes that leave a
ragged last block, one block, and many blocks."""
import numpy as np
import pytest

import hqgen
import oracle
from paper_conf_sigmod_funkebnmt18_b200 import hq
from paper_conf_sigmod_funkebnmt18_b200.engine import Engine
from paper_conf_sigmod_funkebnmt18_b200.queries import QUERIES

pytestmark = pytest.mark.gpu

SF = 0.01


@pytest.fixture(scope="module")
def ctx():
    import torch
    assert torch.cuda.is_available(), "gpu tests need a CUDA device"
    c = hq.Context(0)
    yield c
    c.close()


@pytest.fixture(scope="module")
def data():
    return {**{t: hqgen.generate(t, SF) for t in hqgen.SSB_TABLES}, **{t: hqgen.generate(t, SF) for t in hqgen.TPCH_TABLES}}


def pinned(a):
    import torch
    t = torch.empty(a.shape[0], dtype={np.int8: torch.int8, np.int32: torch.int32, np.int64: torch.int64}[a.dtype.type],
                    pin_memory=True)
    t.numpy()[:] = a
    return t


def run_streamed(ctx, qname, host, block, exec_mode=hq.EXEC_FUSED, pin=True, **kw):
    q = QUERIES[qname]
    tables = {}
    for t, cols in q.columns.items():
        if t == q.fact:
            tables[t] = ctx.load_columns({c: (pinned(host[t][c]) if pin else host[t][c]) for c in cols}, stream=True)
        else:
            tables[t] = ctx.load_columns({c: host[t][c] for c in cols})
    E = Engine(ctx, tables, exec_mode=exec_mode, stream_block=block)
    return q.execute(E, **kw)


def expected(qname, t):
    if qname == "tpch_q6":
        return oracle.tpch_q6(t["lineitem"]), ["revenue", "count"]
    if qname == "tpch_q1":
        return oracle.tpch_q1(t["lineitem"]), ["l_returnflag", "l_linestatus", "sum_qty", "sum_base_price",
                                               "sum_disc_price", "sum_charge", "count_order"]
    if qname == "ssb_q41":
        return (oracle.ssb_q41(t["lineorder"], t["date"], t["customer"], t["supplier"], t["part"]),
                ["d_year", "c_nation", "profit", "count"])
    if qname == "tpch_q3":
        return (oracle.tpch_q3(t["tpch_customer"], t["orders"], t["lineitem"]),
                ["l_orderkey", "o_orderdate", "o_shippriority", "revenue", "count"])
    raise KeyError(qname)


BLOCKS = [4096, 50000, None]  # many blocks (rounded up to the tile), a ragged last block, one block


@pytest.mark.parametrize("qname", ["tpch_q6", "tpch_q1", "ssb_q41", "tpch_q3"])
@pytest.mark.parametrize("block", BLOCKS)
def test_streamed_parity(ctx, data, qname, block):
    o, cols = expected(qname, data)
    kw = {"limit": 0} if qname == "tpch_q3" else {}
    for em in (hq.EXEC_FUSED, hq.EXEC_FUSED_INTERP):
        g = run_streamed(ctx, qname, data, block, exec_mode=em, **kw)
        assert g.rows(cols) == o.rows(cols), (qname, block, em)
        assert g.qualifying == o.qualifying
    if qname == "tpch_q1":
        np.testing.assert_allclose(g.columns["avg_qty"], o.columns["avg_qty"], rtol=1e-9, atol=0)


@pytest.mark.parametrize("block", [4096, None])
def test_streamed_materialise(ctx, data, block):
    """A3 materialisation: the output counter carries over the blocks (a multiset)."""
    o = oracle.ssb_q31_mat(data["lineorder"], data["customer"], data["supplier"], data["date"])
    g = run_streamed(ctx, "ssb_q31_mat", data, block)
    names = ["c_nation", "s_nation", "d_year", "lo_revenue"]
    assert sorted(g.rows(names)) == o.rows() and g.qualifying == o.nrows


def test_streamed_pageable_and_unsupported(ctx, data):
    """Pageable host arrays still give the exact result (copies do not overlap);
    operator-at-a-time / multi-pass and builds refuse host-streamed tables."""
    o, cols = expected("tpch_q6", data)
    g = run_streamed(ctx, "tpch_q6", data, 8192, pin=False)
    assert g.rows(cols) == o.rows(cols)
    for em in (hq.EXEC_OAAT, hq.EXEC_MULTIPASS):
        with pytest.raises(hq.HQError):
            run_streamed(ctx, "tpch_q6", data, 8192, exec_mode=em)
    t = ctx.load_columns({"c_custkey": data["tpch_customer"]["c_custkey"]}, stream=True)
    with pytest.raises(hq.HQError):
        ctx.build_hash(t, 0)
