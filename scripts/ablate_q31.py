#!/usr/bin/env python
"""Per-operator cost of the SSB Q3.1 pipeline (generated kernel): probes only
(count), + group-by sink (C3 smem hash), + C2 ablation."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_sigmod_funkebnmt18_b200 import hq  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200.engine import Engine  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200.queries import ASIA, QUERIES, load_tables  # noqa: E402

sf = float(sys.argv[1]) if len(sys.argv) > 1 else 10
torch.cuda.set_device(0)
ctx = hq.Context(0)
q = QUERIES["ssb_q31"]
E = Engine(ctx, load_tables(ctx, q, sf))
hc = E.hash("customer", "c_custkey", payload=["c_nation"], preds=[("c_region", "=", ASIA)])
hs = E.hash("supplier", "s_suppkey", payload=["s_nation"], preds=[("s_region", "=", ASIA)])
hd = E.hash("date", "d_datekey", payload=["d_year"], preds=[("d_year", "between", 1992, 1997)])
rows = E.tables["lineorder"].nrows


def plan(k, sink):
    pb = E.plan("lineorder")
    if k >= 1:
        pb.probe(hs, "lo_suppkey", "inner", ["s_nation"])
    if k >= 2:
        pb.probe(hc, "lo_custkey", "inner", ["c_nation"])
    if k >= 3:
        pb.probe(hd, "lo_orderdate", "inner", ["d_year"])
    if sink == "count":
        pb.compute("t", [("load", "lo_custkey"), ("add", "lo_suppkey"), ("add", "lo_orderdate"), ("add", "lo_revenue")])
        pb.aggregate(aggs=[("count", None), ("sum", "t")], agg_names=["c", "s"])
    else:
        pb.aggregate(keys=[("c_nation", 0, 25), ("s_nation", 0, 25), ("d_year", 1992, 7)],
                     aggs=[("sum", "lo_revenue"), ("count", None)], agg_names=["revenue", "count"])
    return pb


for k, sink, res in [(0, "count", hq.RES_LRGP), (1, "count", hq.RES_LRGP), (2, "count", hq.RES_LRGP),
                     (3, "count", hq.RES_LRGP), (3, "group", hq.RES_LRGP), (3, "group", hq.RES_ATOMIC)]:
    E.resolution = res
    ctx.enable_timing(True)
    for _ in range(4):
        E.run(plan(k, sink)).fetch()
    kt = ctx.kernel_times()[1:]
    ms = sum(kt) / len(kt)
    print(f"q31 probes={k} sink={sink:5s} res={'C2' if res else 'C3'} kernel {ms:.3f} ms  {rows * 16 / ms / 1e6:.0f} GB/s")
