#!/usr/bin/env python
"""TPC-H Q3 lineitem pipeline, operator prefixes: filter only, + orders probe (count sink),
+ group-by (the query's pipeline).  Fused-kernel CUDA-event times; diagnostic.

    python scripts/ablate_tpch_q3.py [sf]
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_sigmod_funkebnmt18_b200 import hq  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200.engine import Engine  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200.queries import BUILDING, QUERIES, load_tables  # noqa: E402

sf = float(sys.argv[1]) if len(sys.argv) > 1 else 30
torch.cuda.set_device(0)
ctx = hq.Context(0)
q = QUERIES["tpch_q3"]
E = Engine(ctx, load_tables(ctx, q, sf))
hc = E.hash("tpch_customer", "c_custkey", preds=[("c_mktsegment", "=", BUILDING)])
po = E.plan("orders")
po.filter("o_orderdate", "<", 19950315)
po.probe(hc, "o_custkey", "semi")
po.materialise([("o_orderkey", "i32"), ("o_orderdate", "i32"), ("o_shippriority", "i32")])
ro = E.run(po, partitioned=False)
ho = E.hash_from(ro, ["o_orderkey", "o_orderdate", "o_shippriority"], "o_orderkey", ["o_orderdate", "o_shippriority"])
nk = max(int(ho.meta().nkeys), 0)
rows = E.tables["lineitem"].nrows


def plan(k):
    pl = E.plan("lineitem")
    pl.filter("l_shipdate", ">", 19950315)
    if k >= 1:
        pl.probe(ho, "l_orderkey", "inner", ["o_orderdate", "o_shippriority"])
    pl.compute("rev", [("load", "l_discount"), ("rsub", 100), ("mul", "l_extendedprice")])
    if k >= 2:
        pl.aggregate(keys=[("l_orderkey", 0, 1 << 31), ("o_orderdate", 19920101, 70000), ("o_shippriority", 0, 8)],
                     aggs=[("sum", "rev"), ("count", None)], agg_names=["revenue", "count"],
                     group_capacity=max(1024, nk // 12))
    elif k == 1:
        pl.compute("t", [("load", "o_orderdate"), ("add", "o_shippriority"), ("add", "l_orderkey")])
        pl.aggregate(aggs=[("count", None), ("sum", "rev"), ("sum", "t")], agg_names=["c", "s", "t"])
    else:
        pl.compute("t", [("load", "l_orderkey")])
        pl.aggregate(aggs=[("count", None), ("sum", "rev"), ("sum", "t")], agg_names=["c", "s", "t"])
    return pl


for k, name in [(0, "filter"), (1, "filter+probe"), (2, "filter+probe+groupby")]:
    ctx.enable_timing(True)
    for _ in range(5):
        r = E.run(plan(k))
    kt = ctx.kernel_times()[1:]
    ms = sorted(kt)[len(kt) // 2]
    print(f"{name:22s} kernel {ms:.3f} ms  {rows * 24 / ms / 1e6:.0f} GB/s", flush=True)
