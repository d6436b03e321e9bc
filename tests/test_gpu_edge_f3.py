"""Edge cases of the operators added for the TPC-H queries and batch processing
(LEFT OUTER probes, composite keys, predicate instructions, host-streamed fact tables),
each against a result computed by hand or by numpy on the same tiny input."""
import numpy as np
import pytest

from paper_conf_sigmod_funkebnmt18_b200 import hq
from paper_conf_sigmod_funkebnmt18_b200.engine import Engine, fetch

pytestmark = pytest.mark.gpu

ALL_EXEC = [hq.EXEC_FUSED, hq.EXEC_FUSED_INTERP, hq.EXEC_MULTIPASS, hq.EXEC_OAAT]


@pytest.fixture(scope="module")
def ctx():
    import torch
    assert torch.cuda.is_available(), "gpu tests need a CUDA device"
    c = hq.Context(0)
    yield c
    c.close()


def _i32(x):
    return np.asarray(x, dtype=np.int32)


def test_outer_probe_empty_and_partial_build(ctx):
    """LEFT OUTER: every fact row survives; payload = build payload or 0.  An empty
    build (no qualifying rows) gives 0 everywhere."""
    n = 5000  # several tiles and a ragged tail
    fact = ctx.load_columns({"k": _i32(np.arange(n) % 97), "v": _i32(np.arange(n))})
    dim = ctx.load_columns({"dk": _i32(np.arange(0, 97, 3)), "dp": _i32(np.arange(0, 97, 3) * 10 + 1)})
    for preds, expect_hit in ((), True), ([("dk", ">", 1000)], False):
        for em in ALL_EXEC:
            E = Engine(ctx, {"f": fact, "d": dim}, exec_mode=em)
            h = E.hash("d", "dk", payload=["dp"], preds=preds)
            pb = E.plan("f")
            pb.probe(h, "k", "outer", ["p"])
            pb.aggregate(aggs=[("sum", "p"), ("count", None)], agg_names=["s", "c"])
            r = fetch(E.run(pb), pb.result_names)
            k = np.arange(n) % 97
            exp = int(np.where(k % 3 == 0, k * 10 + 1, 0).sum()) if expect_hit else 0
            assert r.rows() == [(exp, n)], (preds, em)


def test_composite_key_long_chains(ctx):
    """A composite table whose first key repeats 64 times (one long probe chain per key):
    only the (k1, k2) pair matches; absent pairs miss."""
    k1 = np.repeat(np.arange(1, 51), 64)
    k2 = np.tile(np.arange(64), 50)
    pay = k1 * 1000 + k2
    dim = ctx.load_columns({"a": _i32(k1), "b": _i32(k2), "p": _i32(pay)})
    rng = np.random.default_rng(7)
    fa = rng.integers(0, 53, 7000)   # 0, 51, 52 absent
    fb = rng.integers(0, 70, 7000)   # 64..69 absent
    fact = ctx.load_columns({"a": _i32(fa), "b": _i32(fb)})
    hit = (fa >= 1) & (fa <= 50) & (fb < 64)
    for em in ALL_EXEC:
        E = Engine(ctx, {"f": fact, "d": dim}, exec_mode=em)
        h = E.hash("d", "a", payload=["p"], key2="b")
        pb = E.plan("f")
        pb.probe(h, "a", "inner", ["p"], key2="b")
        pb.aggregate(aggs=[("sum", "p"), ("count", None)], agg_names=["s", "c"])
        r = fetch(E.run(pb), pb.result_names)
        assert r.rows() == [(int((fa * 1000 + fb)[hit].sum()), int(hit.sum()))], em


def test_predicate_instructions_match_numpy(ctx):
    """acc && reg CMP imm chains, IN over codes < 64, OR of predicate temps."""
    rng = np.random.default_rng(3)
    n = 9000
    a, b, c = rng.integers(0, 60, n), rng.integers(-50, 50, n), rng.integers(0, 10, n)
    fact = ctx.load_columns({"a": _i32(a), "b": _i32(b), "c": _i32(c)})
    codes = [1, 5, 17, 42, 63]
    m0 = np.isin(a, codes) & (b >= -10) & (b < 20) & (c != 3)
    m1 = (a > 50) & (b <= -40) & (c == 9)
    for em in ALL_EXEC:
        E = Engine(ctx, {"f": fact}, exec_mode=em)
        pb = E.plan("f")
        pb.compute("p0", [("load", 1), ("and_in", "a", codes), ("and_ge", "b", -10), ("and_lt", "b", 20), ("and_ne", "c", 3)])
        pb.compute("p1", [("load", 1), ("and_gt", "a", 50), ("and_le", "b", -40), ("and_eq", "c", 9), ("or", "p0")])
        pb.filter("p1", "!=", 0)
        pb.aggregate(aggs=[("sum", "a"), ("count", None)], agg_names=["s", "c"])
        r = fetch(E.run(pb), pb.result_names)
        m = m0 | m1
        assert r.rows() == [(int(a[m].sum()), int(m.sum()))], em
    with pytest.raises(ValueError):  # IN-lists of predicate instructions take codes < 64
        Engine(ctx, {"f": fact}).plan("f").compute("x", [("load", 1), ("and_in", "a", [64])])


@pytest.mark.parametrize("n", [0, 1, 4097])
def test_streamed_tiny_tables(ctx, n):
    """Host-streamed fact tables of 0, 1 and a tile plus one row."""
    v = np.arange(n, dtype=np.int32)
    for block in (1, 4096, None):
        t = ctx.load_columns({"v": v}, stream=True)
        E = Engine(ctx, {"f": t}, stream_block=block)
        pb = E.plan("f")
        pb.filter("v", ">=", 0)
        pb.aggregate(aggs=[("sum", "v"), ("count", None)], agg_names=["s", "c"])
        r = fetch(E.run(pb), pb.result_names)
        assert r.rows() == [(int(v.sum()), n)], (n, block)
