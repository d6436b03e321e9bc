"""Stress: repeat streamed and resident runs of a query, count results that differ
from the first resident run (diagnoses intermittent mismatches)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import hqgen  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200 import hq  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200.engine import Engine  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200.queries import QUERIES  # noqa: E402

qname, sf, block, reps_s, reps_r = sys.argv[1], float(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4]), int(sys.argv[5])
torch.cuda.set_device(0)
ctx = hq.Context(0)
q = QUERIES[qname]
tabs = hqgen.SSB_TABLES if q.bench == "ssb" else hqgen.TPCH_TABLES
host = {t: hqgen.generate(t, sf, columns=q.columns[t]) for t in q.columns if t in tabs}
fact = {}
for c in q.columns[q.fact]:
    arr = host[q.fact][c]
    t = torch.empty(arr.shape[0], dtype={1: torch.int8, 4: torch.int32, 8: torch.int64}[arr.itemsize], pin_memory=True)
    t.numpy()[:] = arr
    fact[c] = t
dims = {t: ctx.load_columns({c: host[t][c] for c in cols}) for t, cols in q.columns.items() if t != q.fact}
Er = Engine(ctx, {**dims, q.fact: ctx.load_columns({c: host[q.fact][c] for c in fact})})
ref = q.execute(Er)
bad_r = 0
for i in range(reps_r):
    g = q.execute(Er)
    if g.rows() != ref.rows() or g.qualifying != ref.qualifying:
        bad_r += 1
        print("resident DIFF", i, g.qualifying, ref.qualifying, [(x, y) for x, y in zip(g.rows(), ref.rows()) if x != y][:3])
st = ctx.load_columns(fact, stream=True)
Es = Engine(ctx, {**dims, q.fact: st}, stream_block=block)
bad_s = 0
for i in range(reps_s):
    g = q.execute(Es)
    if g.rows() != ref.rows() or g.qualifying != ref.qualifying:
        bad_s += 1
        print("streamed DIFF", i, g.qualifying, ref.qualifying, [(x, y) for x, y in zip(g.rows(), ref.rows()) if x != y][:3])
print(f"{qname} sf {sf}: resident {bad_r}/{reps_r} differ, streamed (block {block}) {bad_s}/{reps_s} differ", flush=True)
