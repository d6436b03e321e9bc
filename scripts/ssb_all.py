#!/usr/bin/env python
"""All 13 SSB queries (and the TPC-H ones) on one B200: fused-kernel time,
rows/s and achieved GB/s over the referenced fact columns, like the paper's
per-query SSB evaluation (Fig 20-22), at --sf.  Also the
multi-pass and operator-at-a-time pipeline times of the same plans.
Writes gpurun_out/ssb_all_sf<sf>.{json,md}.

    python scripts/ssb_all.py --sf 30
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import hqgen  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200 import hq  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200.engine import Engine  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200.queries import QUERIES, load_tables  # noqa: E402

SSB = ["ssb_q11", "ssb_q12", "ssb_q13", "ssb_q21", "ssb_q22", "ssb_q23", "ssb_q31", "ssb_q32", "ssb_q33",
       "ssb_q34", "ssb_q41", "ssb_q42", "ssb_q43"]


def pipeline_ms(ctx, E, q, reps, wall=False):
    q.execute(E)
    ts = []
    ctx.enable_timing(True)
    ctx.kernel_times()
    for _ in range(reps):
        if wall:
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            q.run(E)
            torch.cuda.synchronize()
            ts.append((time.perf_counter() - t0) * 1e3)
        else:
            q.run(E)
            t = ctx.kernel_times()
            ts.append(t[-1])  # the fact pipeline is the query's last pipeline
    ctx.enable_timing(False)
    return float(np.median(ts))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--sf", type=float, default=30)
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--queries", default=",".join(SSB))
    a = ap.parse_args()
    torch.cuda.set_device(0)
    ctx = hq.Context(0)
    host = {t: hqgen.generate(t, a.sf) for t in hqgen.SSB_TABLES}
    rows = []
    for name in a.queries.split(","):
        q = QUERIES[name]
        tables = load_tables(ctx, q, a.sf, host=host)
        n = int(tables[q.fact].nrows)
        E = Engine(ctx, tables)
        r = q.execute(E)
        ms = pipeline_ms(ctx, E, q, a.reps)
        mp = pipeline_ms(ctx, Engine(ctx, tables, exec_mode=hq.EXEC_MULTIPASS), q, a.reps)
        oa = pipeline_ms(ctx, Engine(ctx, tables, exec_mode=hq.EXEC_OAAT), q, max(2, a.reps // 2), wall=True)
        b = n * q.fact_bytes_per_row()
        row = {"query": name, "rows": n, "groups": r.nrows, "qualifying": r.qualifying, "fused_ms": ms,
               "rows_per_s": n / ms * 1e3, "gbs": b / ms / 1e6, "multipass_ms": mp, "oaat_wall_ms": oa}
        rows.append(row)
        print(json.dumps(row), flush=True)
        del tables, E
    d = os.path.join(ROOT, "gpurun_out")
    os.makedirs(d, exist_ok=True)
    with open(os.path.join(d, f"ssb_all_sf{a.sf:g}.json"), "w") as f:
        json.dump({"sf": a.sf, "queries": rows}, f, indent=1)
    L = [f"All SSB queries on one B200, SF {a.sf:g} (lineorder resident in HBM): fused pipeline kernel time "
         f"(CUDA events, median of {a.reps}), rows/s and GB/s over the referenced fact columns; multi-pass = its "
         "pipeline (count kernel .. library reduction, events); op-at-a-time = wall clock around the plan.", "",
         "| query | qualifying | groups | fused ms | G rows/s | GB/s | multi-pass ms | op-at-a-time ms |",
         "|---|---|---|---|---|---|---|---|"]
    for r in rows:
        L.append(f"| {r['query']} | {r['qualifying']} | {r['groups']} | {r['fused_ms']:.3f} | {r['rows_per_s'] / 1e9:.0f} | "
                 f"{r['gbs']:.0f} | {r['multipass_ms']:.3f} | {r['oaat_wall_ms']:.3f} |")
    with open(os.path.join(d, f"ssb_all_sf{a.sf:g}.md"), "w") as f:
        f.write("\n".join(L) + "\n")
    print("\n".join(L))


if __name__ == "__main__":
    main()
