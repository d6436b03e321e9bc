"""Ranked sparse-key join tables (include/hq.h): a build whose unique keys
are sparse over their counted range is stored as [bitmap | rank directory | payload rows
by rank].  Probes of every mode read it in generated kernels; the interpreter and
operator-at-a-time read the linear slot array derived from it; its device view imports
on another handle; a duplicate key is reported.  Expected values: plain numpy joins."""
import numpy as np
import pytest

from paper_conf_sigmod_funkebnmt18_b200 import hq
from paper_conf_sigmod_funkebnmt18_b200.engine import PlanBuilder

pytestmark = pytest.mark.gpu

EXECS = [hq.EXEC_FUSED, hq.EXEC_FUSED_INTERP, hq.EXEC_OAAT]


@pytest.fixture(scope="module")
def ctx():
    import torch
    assert torch.cuda.is_available(), "gpu tests need a CUDA device"
    c = hq.Context(0)
    yield c
    c.close()


def _data(seed=5, nd=40_000, nf=300_000, lo=1_000, span=20_000_000):
    rng = np.random.default_rng(seed)
    keys = (lo + rng.choice(span, nd, replace=False)).astype(np.int32)  # density 0.002: sparse
    pays = [rng.integers(-1_000_000, 1_000_000, nd).astype(np.int32) for _ in range(3)]
    hit = rng.random(nf) < 0.5
    fk = np.where(hit, keys[rng.integers(0, nd, nf)], rng.integers(0, lo + span + 5_000_000, nf)).astype(np.int32)
    return keys, pays, fk


def _lookup(keys, pays, fk):
    order = np.argsort(keys)
    sk = keys[order]
    pos = np.searchsorted(sk, fk)
    pos = np.minimum(pos, len(sk) - 1)
    found = sk[pos] == fk
    return found, [p[order][pos] for p in pays]


def _run(ctx, fact, h, mode, npay, exec_mode):
    pb = PlanBuilder(fact)
    names = [f"p{k}" for k in range(npay)]
    pb.probe(h, "fk", mode, names if mode in ("inner", "outer") else [])
    aggs = [("count", None)] + ([("sum", n) for n in names] if mode in ("inner", "outer") else [])
    pb.aggregate(aggs=aggs, agg_names=["count"] + [f"s{k}" for k in range(len(aggs) - 1)])
    pb.plan.exec = exec_mode
    r = ctx.run(pb.plan, keep=pb.keep + [h])
    return [int(c[0]) for c in r.fetch()]


@pytest.mark.parametrize("npay", [0, 1, 2, 3])
def test_ranked_probes_match_numpy(ctx, npay):
    keys, pays, fk = _data(seed=5 + npay)
    cols = {"k": keys}
    for k in range(npay):
        cols[f"p{k}"] = pays[k]
    dim = ctx.load_columns(cols)
    fact = ctx.load_columns({"fk": fk})
    h = ctx.build_hash(dim, 0, list(range(1, npay + 1)))
    ptr, m = h.device_view()
    assert m.layout == hq.HT_LINEAR and m.compact_kind == 4 and m.nkeys == len(keys)
    found, pv = _lookup(keys, pays, fk)
    modes = ["semi", "anti"] + (["inner", "outer"] if npay else [])
    for mode in modes:
        if mode == "semi":
            want = [int(found.sum())]
        elif mode == "anti":
            want = [int((~found).sum())]
        elif mode == "inner":
            want = [int(found.sum())] + [int(p[found].astype(np.int64).sum()) for p in pv[:npay]]
        else:
            want = [len(fk)] + [int(np.where(found, p, 0).astype(np.int64).sum()) for p in pv[:npay]]
        for ex in EXECS:
            assert _run(ctx, fact, h, mode, npay, ex) == want, (mode, ex)
    # the device view imports on another handle (the multi-GPU path) and probes the same
    h2 = ctx.import_hash(m, ptr, keep=h)
    mode = "inner" if npay else "semi"
    for ex in EXECS:
        assert _run(ctx, fact, h2, mode, npay, ex) == _run(ctx, fact, h, mode, npay, hq.EXEC_FUSED)


def test_ranked_grouped_by_payloads(ctx):
    """An inner probe with two payloads feeding a GROUP BY (TPC-H Q3's shape): the groups
    keyed by (fact key, payload 0) equal numpy's."""
    keys, pays, fk = _data(seed=11, nd=5_000, nf=200_000)
    p0 = (pays[0] % 50).astype(np.int32)
    dim = ctx.load_columns({"k": keys, "a": p0, "b": pays[1]})
    fact = ctx.load_columns({"fk": fk})
    h = ctx.build_hash(dim, 0, [1, 2])
    assert h.device_view()[1].compact_kind == 4
    pb = PlanBuilder(fact)
    pb.probe(h, "fk", "inner", ["a", "b"])
    lo = int(keys.min())
    pb.aggregate(keys=[("fk", lo, int(keys.max()) - lo + 1), ("a", -49, 99)], aggs=[("sum", "b"), ("count", None)],
                 agg_names=["sb", "n"], group_capacity=8192)
    g = ctx.run(pb.plan, keep=pb.keep + [h]).fetch()
    got = sorted(zip(*[c.tolist() for c in g]))
    found, (a, b) = _lookup(keys, [p0, pays[1]], fk)
    ref = {}
    for k, x, y in zip(fk[found].tolist(), a[found].tolist(), b[found].tolist()):
        s, n = ref.get((k, x), (0, 0))
        ref[(k, x)] = (s + y, n + 1)
    assert got == sorted((k, x, s, n) for (k, x), (s, n) in ref.items())


def test_ranked_duplicate_key_is_reported(ctx):
    keys, pays, fk = _data(seed=3, nd=10_000)
    keys[777] = keys[4242]  # one duplicate among sparse keys
    dim = ctx.load_columns({"k": keys, "p": pays[0]})
    fact = ctx.load_columns({"fk": fk})
    h = ctx.build_hash(dim, 0, [1])
    assert h.device_view()[1].compact_kind == 4
    with pytest.raises(hq.HQError) as e:
        _run(ctx, fact, h, "inner", 1, hq.EXEC_FUSED)
    assert e.value.code == hq.HQ_ERR_DUP_KEY


def test_ranked_edges(ctx):
    """One key; keys at the top of the int32 range; a range just under one directory block
    and just over it (the scan's padding)."""
    fact_keys = np.array([2**31 - 1, 2**31 - 2, 5, 6, -7, 0], np.int32)
    fact = ctx.load_columns({"fk": fact_keys})
    for keys in (np.array([2**31 - 1], np.int32),
                 np.array([2**31 - 1, 2**31 - 500_000, 5], np.int32),
                 np.array([5, 5 + 100_000, 5 + 32 * 8192 - 1], np.int32),
                 np.array([6, 6 + 32 * 8192], np.int32)):
        pay = (keys // 3).astype(np.int32)
        dim = ctx.load_columns({"k": keys, "p": pay})
        h = ctx.build_hash(dim, 0, [1])
        found, (pv,) = _lookup(keys, [pay], fact_keys)
        want = [int(found.sum()), int(pv[found].astype(np.int64).sum())]
        for ex in EXECS:
            assert _run(ctx, fact, h, "inner", 1, ex) == want, (keys, ex)


@pytest.mark.parametrize("hit_rate", [1.0, 0.37, 0.0])
def test_materialise_behind_a_global_probe(ctx, hit_rate):
    """A3 with warp workgroups: a materialising pipeline behind a global
    probe buffers each warp's rows and flushes them with one atomic; every selected row
    lands exactly once (dense positions), including full selectivity (a flush per tile),
    none, and the capacity re-run; segment_rows is 0 (no tile segments)."""
    rng = np.random.default_rng(21)
    nd, nf = 30_000, 700_001  # a ragged last tile
    keys = (10 + rng.choice(5_000_000, nd, replace=False)).astype(np.int32)
    pay = rng.integers(0, 1 << 30, nd).astype(np.int32)
    hit = rng.random(nf) < hit_rate
    fk = np.where(hit, keys[rng.integers(0, nd, nf)], -5).astype(np.int32)
    rowid = np.arange(nf, dtype=np.int32)
    dim = ctx.load_columns({"k": keys, "p": pay})
    fact = ctx.load_columns({"fk": fk, "rowid": rowid})
    h = ctx.build_hash(dim, 0, [1])
    found, (pv,) = _lookup(keys, [pay], fk)
    want = sorted(zip(rowid[found].tolist(), pv[found].tolist()))
    for cap in (0, 1000):  # 1000: undersized -> F_CAPACITY -> one exact re-run
        pb = PlanBuilder(fact)
        pb.probe(h, "fk", "inner", ["p"])
        pb.materialise([("rowid", "i32"), ("p", "i32")], capacity=cap)
        r = ctx.run(pb.plan, keep=pb.keep + [h])
        a, b = r.fetch()
        assert r.qualifying() == len(a) == len(want)
        assert sorted(zip(a.tolist(), b.tolist())) == want
        assert r.info().segment_rows == 0
