#!/usr/bin/env python
"""Every TPC-H query of the build on one B200 at --sf (tables resident in HBM):
per query the fused-pipeline kernel times (one per pipeline, CUDA events on the
context stream), the whole query on the device (hash builds, every pipeline,
finalize and the result fetch; CUDA events around q.execute), lineitem (fact)
rows per second of the whole query, and the multi-pass / operator-at-a-time
times of the same plans (paper Exp 4, Fig 22-24).  Writes
gpurun_out/tpch_all_sf<sf>.{json,md}.

    python scripts/tpch_all.py --sf 10
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import hqgen  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200 import hq  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200.engine import Engine  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200.queries import QUERIES, load_tables  # noqa: E402

TPCH = ["tpch_q1", "tpch_q3", "tpch_q4", "tpch_q5", "tpch_q6", "tpch_q7", "tpch_q9", "tpch_q10", "tpch_q13", "tpch_q17",
        "tpch_q18", "tpch_q19", "tpch_q21"]


def measure(ctx, E, q, reps):
    """(median query ms on the device, median summed pipeline-kernel ms, kernel ms list of the median rep)."""
    q.execute(E)  # warm: NVRTC compile of each pipeline shape
    stream = torch.cuda.current_stream()
    walls, sums, lists = [], [], []
    ctx.enable_timing(True)
    ctx.kernel_times()
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record(stream)
        q.execute(E)
        e1.record(stream)
        torch.cuda.synchronize()
        walls.append(e0.elapsed_time(e1))
        ks = ctx.kernel_times()
        sums.append(sum(ks))
        lists.append(ks)
    ctx.enable_timing(False)
    i = int(np.argsort(walls)[len(walls) // 2])
    return float(walls[i]), float(np.median(sums)), [round(k, 4) for k in lists[i]]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--sf", type=float, default=10)
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--queries", default=",".join(TPCH))
    a = ap.parse_args()
    torch.cuda.set_device(0)
    ctx = hq.Context(0)  # on torch's current stream: the events below see its kernels
    host = {t: hqgen.generate(t, a.sf) for t in hqgen.TPCH_TABLES}
    rows = []
    for name in a.queries.split(","):
        q = QUERIES[name]
        tables = load_tables(ctx, q, a.sf, host=host)
        n = int(tables["lineitem"].nrows) if "lineitem" in tables else int(tables[q.fact].nrows)
        E = Engine(ctx, tables)
        r = q.execute(E)
        wall, kern, klist = measure(ctx, E, q, a.reps)
        mp, _, _ = measure(ctx, Engine(ctx, tables, exec_mode=hq.EXEC_MULTIPASS), q, max(2, a.reps // 2))
        oa, _, _ = measure(ctx, Engine(ctx, tables, exec_mode=hq.EXEC_OAAT), q, 2)
        row = {"query": name, "lineitem_rows": n, "result_rows": r.nrows, "qualifying": r.qualifying,
               "pipelines": len(klist), "kernel_ms": klist, "kernels_ms": kern, "query_ms": wall,
               "rows_per_s": n / wall * 1e3, "multipass_query_ms": mp, "oaat_query_ms": oa}
        rows.append(row)
        print(json.dumps(row), flush=True)
        del tables, E
    d = os.path.join(ROOT, "gpurun_out")
    os.makedirs(d, exist_ok=True)
    with open(os.path.join(d, f"tpch_all_sf{a.sf:g}.json"), "w") as f:
        json.dump({"sf": a.sf, "queries": rows}, f, indent=1)
    L = [f"TPC-H queries on one B200, SF {a.sf:g} (tables resident in HBM). query ms = the whole query on the "
         "device (builds, every pipeline, finalize, result fetch; CUDA events, median of "
         f"{a.reps}); kernels = the fused pipeline kernels in plan order (CUDA events); rows/s = lineitem "
         "rows / query ms. Multi-pass and operator-at-a-time: the same plans' whole-query times.", "",
         "| query | pipelines | fused kernels ms | query ms | G lineitem rows/s | multi-pass ms | op-at-a-time ms |",
         "|---|---|---|---|---|---|---|"]
    for r in rows:
        L.append(f"| {r['query']} | {r['pipelines']} | {' + '.join(f'{k:.3f}' for k in r['kernel_ms'])} | "
                 f"{r['query_ms']:.3f} | {r['rows_per_s'] / 1e9:.1f} | {r['multipass_query_ms']:.3f} | "
                 f"{r['oaat_query_ms']:.3f} |")
    with open(os.path.join(d, f"tpch_all_sf{a.sf:g}.md"), "w") as f:
        f.write("\n".join(L) + "\n")
    print("\n".join(L))


if __name__ == "__main__":
    main()
