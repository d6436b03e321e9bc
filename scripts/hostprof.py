"""cProfile of the host side of repeated query steps (where the Python / C++ host time
between kernel launches goes).  python scripts/hostprof.py --query ssb_q11 --sf 1 --steps 200
[--dist: the distributed engine over NCCL at world size 1]"""
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
ap.add_argument("--dist", action="store_true")
ap.add_argument("--broadcast", action="store_true", help="--dist with the root-broadcast design")
a = ap.parse_args()
torch.cuda.set_device(0)
q = QUERIES[a.query]
ctx = hq.Context(0)
tables = load_tables(ctx, q, a.sf)
if a.dist:
    import torch.distributed as dist
    from paper_conf_sigmod_funkebnmt18_b200.dist import DistributedEngine, run_query
    os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
    os.environ.setdefault("MASTER_PORT", "29572")
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    E = DistributedEngine(ctx, tables, replicated=not a.broadcast)

    def step():
        return run_query(E, q)
else:
    E = Engine(ctx, tables)

    def step():
        return q.execute(E)
for _ in range(5):
    step()
pr = cProfile.Profile()
pr.enable()
for _ in range(a.steps):
    step()
pr.disable()
st = pstats.Stats(pr)
st.sort_stats("tottime").print_stats(30)
st.sort_stats("cumtime").print_stats(40)
