"""Host-side phase timing of one query step (builds / fused pipeline / finalize+fetch)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_sigmod_funkebnmt18_b200 import hq
from paper_conf_sigmod_funkebnmt18_b200.engine import Engine
from paper_conf_sigmod_funkebnmt18_b200 import queries as Q

qn, sf, reps = sys.argv[1], float(sys.argv[2]), int(sys.argv[3])
q = Q.QUERIES[qn]
ctx = hq.Context(0)
tables = Q.load_tables(ctx, q, sf)
ctx.sync()
E = Engine(ctx, tables)
orig_run = E.run
marks = {}
def run(pb, partitioned=True):
    ctx.sync(); marks["built"] = time.perf_counter()
    r = orig_run(pb, partitioned)
    ctx.sync(); marks["ran"] = time.perf_counter()
    return r
E.run = run
for i in range(reps):
    ctx.sync(); t0 = time.perf_counter()
    res, pb = q.run(E)
    out = E.finish(res, pb)
    t3 = time.perf_counter()
    if i >= 2:
        print(f"builds {1e3*(marks['built']-t0):.3f} ms  pipeline {1e3*(marks['ran']-marks['built']):.3f} ms  finish {1e3*(t3-marks['ran']):.3f} ms  total {1e3*(t3-t0):.3f}")
