"""Stress: repeat the HBM-resident run of a query under environment knobs of the
query compiler and count results differing from the oracle (diagnoses rare races).
usage: stress_resident.py QUERY SF REPS [ENV=VAL,ENV=VAL ...] (one variant per arg)"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import hqgen  # noqa: E402
import oracle  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200 import hq  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200.engine import Engine  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200.queries import QUERIES, load_tables  # noqa: E402

qname, sf, reps = sys.argv[1], float(sys.argv[2]), int(sys.argv[3])
variants = sys.argv[4:] or [""]
torch.cuda.set_device(0)
ctx = hq.Context(0)
q = QUERIES[qname]
tabs = hqgen.SSB_TABLES if q.bench == "ssb" else hqgen.TPCH_TABLES
host = {t: hqgen.generate(t, sf) for t in q.columns if t in tabs}
o = oracle.ssb_q41(host["lineorder"], host["date"], host["customer"], host["supplier"], host["part"], nthreads=os.cpu_count())
exp = o.rows()
E = Engine(ctx, load_tables(ctx, q, sf, host=host))
for v in variants:
    env = dict(x.split("=") for x in v.split(",") if x)
    os.environ.update(env)
    bad = 0
    for i in range(reps):
        g = q.execute(E)
        if g.rows(["d_year", "c_nation", "profit", "count"]) != exp:
            bad += 1
            if bad <= 2:
                print("  DIFF", v, [(a, b) for a, b in zip(g.rows(["d_year", "c_nation", "profit", "count"]), exp) if a != b][:2])
    print(f"{qname} sf {sf} [{v or 'default'}]: {bad}/{reps} differ from the oracle", flush=True)
