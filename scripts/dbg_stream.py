"""Debug: streamed vs resident results of a query for several block sizes."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import hqgen  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200 import hq  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200.engine import Engine  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200.queries import QUERIES  # noqa: E402

qname, sf = sys.argv[1], float(sys.argv[2])
blocks = [int(x) for x in sys.argv[3].split(",")]
pin = len(sys.argv) <= 4 or sys.argv[4] != "nopin"
torch.cuda.set_device(0)
ctx = hq.Context(0)
q = QUERIES[qname]
tabs = hqgen.SSB_TABLES if q.bench == "ssb" else hqgen.TPCH_TABLES
host = {t: hqgen.generate(t, sf, columns=q.columns[t]) for t in q.columns if t in tabs}
fact = {}
for c in q.columns[q.fact]:
    arr = host[q.fact][c]
    t = torch.empty(arr.shape[0], dtype={1: torch.int8, 4: torch.int32, 8: torch.int64}[arr.itemsize], pin_memory=pin)
    t.numpy()[:] = arr
    fact[c] = t
dims = {t: ctx.load_columns({c: host[t][c] for c in cols}) for t, cols in q.columns.items() if t != q.fact}
ref = q.execute(Engine(ctx, {**dims, q.fact: ctx.load_columns({c: host[q.fact][c] for c in fact})}))
st = ctx.load_columns(fact, stream=True)
for b in blocks:
    for em in (hq.EXEC_FUSED, hq.EXEC_FUSED_INTERP):
        for rep in range(2):
            got = q.execute(Engine(ctx, {**dims, q.fact: st}, stream_block=b, exec_mode=em))
            ok = got.rows() == ref.rows() and got.qualifying == ref.qualifying
            print(qname, sf, "block", b, "exec", em, "rep", rep, "OK" if ok else "DIFF", got.qualifying, ref.qualifying, flush=True)
            if not ok:
                gr, rr = got.rows(), ref.rows()
                print("  nrows", len(gr), len(rr), [(a, b2) for a, b2 in zip(gr, rr) if a != b2][:3])
