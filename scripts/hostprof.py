"""cProfile of the host side of repeated query steps (where the Python / C++ host time
between kernel launches goes).  python scripts/hostprof.py --query ssb_q11 --sf 1 --steps 200"""
import argparse
import cProfile
import os
import pstats
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_sigmod_funkebnmt18_b200 import hq  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200.engine import Engine  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200.queries import QUERIES, load_tables  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--query", default="ssb_q11")
ap.add_argument("--sf", type=float, default=1)
ap.add_argument("--steps", type=int, default=200)
a = ap.parse_args()
torch.cuda.set_device(0)
q = QUERIES[a.query]
ctx = hq.Context(0)
E = Engine(ctx, load_tables(ctx, q, a.sf))
for _ in range(5):
    q.execute(E)
pr = cProfile.Profile()
pr.enable()
for _ in range(a.steps):
    q.execute(E)
pr.disable()
st = pstats.Stats(pr)
st.sort_stats("tottime").print_stats(25)
