"""Re-run one query's final pipeline N times on the same hash tables (timing study)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_sigmod_funkebnmt18_b200 import hq
from paper_conf_sigmod_funkebnmt18_b200.engine import Engine
from paper_conf_sigmod_funkebnmt18_b200.queries import QUERIES, load_tables
q = QUERIES[sys.argv[1]]; sf = float(sys.argv[2]); n = int(sys.argv[3]); builds = int(sys.argv[4])
ctx = hq.Context(0)
tables = load_tables(ctx, q, sf)
E = Engine(ctx, tables)
ctx.enable_timing(True)
for b in range(builds):
    res, pb = q.run(E)
    ctx.kernel_times()
    for i in range(n):
        r = ctx.run(pb.plan, keep=pb.keep)
    print("build", b, [round(x, 3) for x in ctx.kernel_times()], flush=True)
