#!/usr/bin/env python
"""Per-operator cost of the Q4.1 pipeline: time the fused kernel for growing
prefixes of the plan (scan only, +probe supplier, +customer, +part, +date,
+compute/group).  Diagnostic for the ncu-guided tuning loop."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_sigmod_funkebnmt18_b200 import hq  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200.engine import Engine  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200.queries import AMERICA, MFGR1, MFGR2, QUERIES, load_tables  # noqa: E402

sf = float(sys.argv[1]) if len(sys.argv) > 1 else 10
torch.cuda.set_device(0)
ctx = hq.Context(0)
q = QUERIES["ssb_q41"]
E = Engine(ctx, load_tables(ctx, q, sf))
hs = E.hash("supplier", "s_suppkey", preds=[("s_region", "=", AMERICA)])
hc = E.hash("customer", "c_custkey", payload=["c_nation"], preds=[("c_region", "=", AMERICA)])
hp = E.hash("part", "p_partkey", preds=[("p_mfgr", "in", [MFGR1, MFGR2])])
hd = E.hash("date", "d_datekey", payload=["d_year"])
for h, n in ((hs, "supp"), (hc, "cust"), (hp, "part"), (hd, "date")):
    m = h.info()
    print(n, "layout", m.layout, "cap", m.capacity, "keys", m.nkeys, "bytes", m.bytes)


def plan(k, sink="count"):
    pb = E.plan("lineorder")
    cols = ["lo_suppkey", "lo_custkey", "lo_partkey", "lo_orderdate", "lo_revenue", "lo_supplycost"]
    if k >= 1:
        pb.probe(hs, "lo_suppkey", "semi")
    if k >= 2:
        pb.probe(hc, "lo_custkey", "inner", ["c_nation"])
    if k >= 3:
        pb.probe(hp, "lo_partkey", "semi")
    if k >= 4:
        pb.probe(hd, "lo_orderdate", "inner", ["d_year"])
    if sink == "count":
        # touch every column so the stage layout is the same as Q4.1
        pb.compute("t", [("load", cols[0])] + [("add", c) for c in cols[1:]])
        pb.aggregate(aggs=[("count", None), ("sum", "t")], agg_names=["c", "s"])
    else:
        pb.compute("profit", [("load", "lo_revenue"), ("sub", "lo_supplycost")])
        pb.aggregate(keys=[("d_year", 1992, 7), ("c_nation", 0, 25)], aggs=[("sum", "profit"), ("count", None)],
                     agg_names=["profit", "count"])
    return pb


rows = len(E.tables["lineorder"].names) and E.tables["lineorder"].nrows
for k, sink in [(0, "count"), (1, "count"), (2, "count"), (3, "count"), (4, "count"), (4, "group")]:
    ctx.enable_timing(True)
    for _ in range(4):
        pb = plan(k, sink)
        r = E.run(pb)
        r.fetch()
    kt = ctx.kernel_times()[1:]
    ms = sum(kt) / len(kt)
    print(f"probes={k} sink={sink:5s} kernel {ms:.3f} ms  {rows * 24 / ms / 1e6:.0f} GB/s  rows/clk/SM "
          f"{rows / (ms * 1e-3) / 148 / 1.965e9:.3f}")
E.resolution = hq.RES_ATOMIC
ctx.enable_timing(True)
for _ in range(4):
    E.run(plan(4, "group")).fetch()
kt = ctx.kernel_times()[1:]
print(f"probes=4 sink=group C2 (per-row global atomics) kernel {sum(kt) / len(kt):.3f} ms")
