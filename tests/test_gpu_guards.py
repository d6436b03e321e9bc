"""GPU tests of the sink mechanisms the query-level parity cannot force by itself:
the int64 guard of the aggregation sinks, the shared-memory hash table's spill to
global memory (C3 -> C2) in the generated kernel, and the LRGP write positions of
fixture F3 at tile scale.  Every expected value comes from oracle/ or from a
tests/golden fixture."""
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


def test_int64_guard_overflow(ctx):
    """TPC-H Q6 over rows whose exact SUM(l_extendedprice * l_discount) exceeds int64
    (each product fits): the oracle fails with rc -6 and the
    fused kernel's finalize raises HQ_ERR_OVERFLOW (R13: the wrapped sum
    lands beyond the +-2^62 guard)."""
    n = 2
    li = {"l_shipdate": np.full(n, 19940601, np.int32), "l_discount": np.full(n, 6, np.int64),
          "l_quantity": np.full(n, 100, np.int64), "l_extendedprice": np.full(n, 10**18, np.int64)}
    with pytest.raises(oracle.OracleError) as eo:
        oracle.tpch_q6(li)
    assert eo.value.rc == -6
    q = QUERIES["tpch_q6"]
    for em in (hq.EXEC_FUSED, hq.EXEC_FUSED_INTERP):
        E = Engine(ctx, {"lineitem": ctx.load_columns(li)}, exec_mode=em)
        with pytest.raises(hq.HQError) as eg:
            q.execute(E)
        assert eg.value.code == hq.HQ_ERR_OVERFLOW, em
    # below the guard the same plan is exact (the oracle's value)
    li2 = dict(li, l_extendedprice=np.full(n, 10**17, np.int64))
    E = Engine(ctx, {"lineitem": ctx.load_columns(li2)})
    assert q.execute(E).rows(["revenue", "count"]) == oracle.tpch_q6(li2).rows(["revenue", "count"])


@pytest.mark.parametrize("x", [3500, 20000])
def test_shared_hash_spill_to_global(ctx, x):
    """Fig 26's GROUP BY lo_orderkey % x with a hash group-by declared (key domain
    2^31, expected 4096 groups): the generated kernel pre-aggregates in a shared hash
    table of <= 1365 slots (SM_HASH), so with x distinct keys per CTA it fills and
    the remaining keys go to the global table (C2).  x = 20000 also exceeds the
    global table's first capacity (the capacity re-run).  Same rows as the oracle."""
    sf = 1.0
    lo = hqgen.generate("lineorder", sf, columns=["lo_orderkey", "lo_extendedprice"])
    t = ctx.load_columns({c: lo[c] for c in ("lo_orderkey", "lo_extendedprice")})
    pb = PlanBuilder(t)
    pb.compute("k", [("load", "lo_orderkey"), ("mod", x)])
    pb.aggregate(keys=[("k", 0, 1 << 31)], aggs=[("sum", "lo_extendedprice"), ("count", None)],
                 order=[("k", False)], group_capacity=4096, agg_names=["sum", "count"])
    res = ctx.run(pb.plan, keep=pb.keep)
    cols = res.fetch()
    o = oracle.micro_groupby(lo, x, nthreads=8)
    got = list(zip(*[c.tolist() for c in cols]))
    assert got == o.rows(["key", "sum", "count"])
    assert res.qualifying() == len(lo["lo_orderkey"])


def test_f3_lrgp_positions_tile_scale(ctx, golden):
    """Fixture F3 with each fixture row
    standing for a run of T/4 rows, so a fixture CTA is one kernel tile (one grid CTA
    each: 3 tiles -> grid 3): the atomics' order differs between runs, and every run's
    positions must equal the fixture's rule for the order that run took -- CTA totals,
    local exclusive offsets, global offsets = prefix of the totals in atomic order."""
    fx = golden("F3_lrgp_positions.json")
    flags, cs = np.asarray(fx["flags"]), fx["cta_size"]
    ncta = len(flags) // cs
    # discover the tile size of this plan shape
    probe_t = ctx.load_columns({"rowid": np.arange(8, dtype=np.int32), "flag": np.ones(8, np.int32)})
    pb = PlanBuilder(probe_t)
    pb.filter("flag", "=", 1).materialise([("rowid", "i32")])
    T = ctx.run(pb.plan, keep=pb.keep).info().segment_rows
    assert T % cs == 0
    run = T // cs
    rowflag = np.repeat(flags, run).astype(np.int32)  # fixture row i -> rows [i*run, (i+1)*run)
    n = len(rowflag)
    t = ctx.load_columns({"rowid": np.arange(n, dtype=np.int32), "flag": rowflag})
    totals = [int(v) * run for v in fx["expected"]["cta_totals"]]
    local = {int(k): v * run for k, v in fx["expected"]["local_offsets"].items()}
    seen = set()
    for _ in range(40):
        pb = PlanBuilder(t)
        pb.filter("flag", "=", 1).materialise([("rowid", "i32")])
        res = ctx.run(pb.plan, keep=pb.keep)
        out = res.fetch()[0]
        assert res.qualifying() == len(out) == fx["expected"]["count"] * run
        # the order in which the non-empty CTAs took their global offsets
        order = []
        for p in range(0, len(out), 1):
            c = int(out[p]) // T
            if not order or order[-1] != c:
                order.append(c)
        assert sorted(order) == [c for c in range(ncta) if totals[c] > 0], order
        seen.add(tuple(order))
        g_os, acc = {}, 0
        for c in order:
            g_os[c] = acc
            acc += totals[c]
        assert acc == len(out)
        pos = np.full(n, -1, np.int64)
        pos[out] = np.arange(len(out))
        for fr, off in local.items():  # fixture rows that pass: their run of rows
            c = fr // cs
            base = g_os[c] + off
            np.testing.assert_array_equal(pos[fr * run:(fr + 1) * run], np.arange(base, base + run))
        assert np.all(pos[rowflag == 0] == -1)
    assert all(set(o) == {0, 2} for o in seen) and len(seen) >= 1
