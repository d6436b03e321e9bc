#!/usr/bin/env python
"""Run one query a few times on cuda:0 (for ncu captures).

    python scripts/profile_query.py --query ssb_q41 --sf 10 --reps 3 [--exec oaat] [--resolution atomic]
"""
import argparse
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import hqgen  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200 import hq  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200.engine import Engine  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200.queries import QUERIES, load_tables  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--query", default="ssb_q41")
    ap.add_argument("--sf", type=float, default=10)
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--exec", default="fused", choices=["fused", "oaat", "multipass"])
    ap.add_argument("--resolution", default="lrgp", choices=["lrgp", "atomic"])
    ap.add_argument("--kw", default="", help="query kwargs k=v,...")
    a = ap.parse_args()
    kw = {k: int(v) for k, v in (x.split("=") for x in a.kw.split(",") if x)}
    torch.cuda.set_device(0)
    q = QUERIES[a.query]
    ctx = hq.Context(0)
    t0 = time.time()
    tables = load_tables(ctx, q, a.sf)
    ctx.sync()
    print(f"loaded in {time.time() - t0:.1f}s", flush=True)
    E = Engine(ctx, tables, exec_mode={"fused": hq.EXEC_FUSED, "oaat": hq.EXEC_OAAT, "multipass": hq.EXEC_MULTIPASS}[a.exec],
               resolution=hq.RES_LRGP if a.resolution == "lrgp" else hq.RES_ATOMIC)
    ctx.enable_timing(True)
    for i in range(a.reps):
        r = q.execute(E, **kw)
    kt = ctx.kernel_times()
    print(a.query, a.sf, "rows", r.nrows, "qualifying", r.qualifying, "fused kernel ms", [round(x, 3) for x in kt])


if __name__ == "__main__":
    main()
