"""Stress: repeat each query REPS times on one device at SF and compare every run with
the first run's rows (rare races show as differing runs).  Queries with a LIMIT run
without it (limit=0: the full pre-LIMIT set under the total order) when listed as name:full.
usage: stress_queries.py SF REPS q1,q2:full,..."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import hqgen  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200 import hq  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200.engine import Engine  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200.queries import QUERIES, load_tables  # noqa: E402

sf, reps, names = float(sys.argv[1]), int(sys.argv[2]), sys.argv[3].split(",")
torch.cuda.set_device(0)
ctx = hq.Context(0)
for qspec in names:
    qn, _, mode = qspec.partition(":")
    kw = {"limit": 0} if mode == "full" else {}
    q = QUERIES[qn]
    tabs = hqgen.SSB_TABLES if q.bench == "ssb" else hqgen.TPCH_TABLES
    host = {t: hqgen.generate(t, sf) for t in q.columns if t in tabs}
    E = Engine(ctx, load_tables(ctx, q, sf, host=host))
    first = q.execute(E, **kw)
    key = lambda r: sorted(r.rows()) if qn.endswith("_mat") else r.rows()
    ref = key(first)
    bad = 0
    for i in range(reps):
        g = q.execute(E, **kw)
        if key(g) != ref or g.qualifying != first.qualifying:
            bad += 1
    print(f"{qspec} sf {sf:g}: {bad}/{reps} runs differ from the first run ({first.nrows} rows)", flush=True)
