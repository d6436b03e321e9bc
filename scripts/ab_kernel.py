"""A/B of the fused kernel time of one query (median of REPS live CUDA-event timings of
the query's last pipeline), for environment knobs set by the caller."""
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

from paper_conf_sigmod_funkebnmt18_b200 import hq  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200.engine import Engine  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200.queries import QUERIES, load_tables  # noqa: E402

qname, sf, reps = sys.argv[1], float(sys.argv[2]), int(sys.argv[3])
kw = dict(x.split("=") for x in sys.argv[4].split(",")) if len(sys.argv) > 4 else {}
torch.cuda.set_device(0)
ctx = hq.Context(0)
q = QUERIES[qname]
E = Engine(ctx, load_tables(ctx, q, sf))
for _ in range(3):
    q.execute(E, **kw)
ctx.enable_timing(True)
ctx.kernel_times()
ts = []
for _ in range(reps):
    q.execute(E, **kw)
    ts.append(ctx.kernel_times()[-1])
env = ",".join(f"{k}={v}" for k, v in os.environ.items() if k.startswith("HQ_JIT"))
print(f"{qname} sf {sf:g} {kw} [{env or 'default'}]: median {statistics.median(ts):.4f} ms, min {min(ts):.4f} ms", flush=True)
