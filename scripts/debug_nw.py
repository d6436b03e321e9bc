import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_sigmod_funkebnmt18_b200 import hq
from paper_conf_sigmod_funkebnmt18_b200.engine import PlanBuilder
ctx = hq.Context(0)
n = int(sys.argv[1]); a, b = int(sys.argv[2]), int(sys.argv[3]); kind = sys.argv[4]
rowid = np.arange(n, dtype=np.int32); c8 = (rowid % 3).astype(np.int8); c64 = rowid.astype(np.int64) * 3
t = ctx.load_columns({"rowid": rowid, "c8": c8, "c64": c64})
pb = PlanBuilder(t); pb.plan.row_begin, pb.plan.row_end = a, b
if kind == "scalar":
    pb.aggregate(aggs=[("count", None), ("sum", "rowid"), ("sum", "c8"), ("sum", "c64")], agg_names=["c", "s", "s8", "s64"])
elif kind == "group":
    pb.aggregate(keys=[("c8", 0, 3)], aggs=[("count", None), ("sum", "rowid")], agg_names=["c", "s"])
else:
    pb.materialise([("rowid", "i32")])
r = ctx.run(pb.plan, keep=pb.keep)
out = r.fetch()
sl = slice(a, b)
if kind == "scalar":
    exp = [b - a, int(rowid[sl].astype(np.int64).sum()), int(c8[sl].astype(np.int64).sum()), int(c64[sl].sum())]
    got = [int(x[0]) for x in out]
elif kind == "group":
    exp = [(g, int((c8[sl] == g).sum()), int(rowid[sl][c8[sl] == g].astype(np.int64).sum())) for g in range(3)]
    got = list(zip(*[x.tolist() for x in out]))
else:
    exp = b - a; got = len(out[0]); assert np.array_equal(np.sort(out[0]), rowid[sl])
print(kind, os.environ.get("HQ_DEBUG_NW"), "OK" if got == exp else f"MISMATCH got={got} exp={exp}", flush=True)
