#!/usr/bin/env python
"""Reduction micro-benchmarks of the paper on B200:

* Exp 1 (Fig 16-17): Query 1 selection + projection, materialised,
  selectivity swept 0..1 -- A1 (multi-pass), A2 (per-row atomics), A3 with SIMD-style
  local resolution (warp ballots/shuffles, the default) and A3-WE (work-efficient
  Blelloch scan over the workgroup, App C Fig 24);
* App G.1: the same query as a single-tuple aggregation -- B1, B2, B3, B3-WE;
* Exp 2 (Fig 26): SUM(lo_extendedprice) GROUP BY lo_orderkey % x,
  x = 2 .. 16384 groups -- C1, C2, C3, C3-WE (sort + segmented scan);

each also as the operator-at-a-time plan.  Times are the pipeline's device time
(CUDA events around the fused kernel, or around the whole multi-pass sequence),
median of --reps after one warm-up, at SSB SF --sf (lineorder rows resident).
Writes gpurun_out/micro_sweeps.{json,md}.

    python scripts/micro_sweeps.py --sf 10
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

from paper_conf_sigmod_funkebnmt18_b200 import hq  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200.engine import Engine  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200.queries import QUERIES, load_tables  # noqa: E402

MODES = {  # technique letter -> (exec mode, resolution)
    "1": (hq.EXEC_MULTIPASS, hq.RES_LRGP),
    "2": (hq.EXEC_FUSED, hq.RES_ATOMIC),
    "3": (hq.EXEC_FUSED, hq.RES_LRGP),
    "3WE": (hq.EXEC_FUSED, hq.RES_WE),
}


def timed(ctx, tables, q, exec_mode, res, reps, **kw):
    """Median pipeline time (ms) of `reps` runs (results stay on the device)."""
    E = Engine(ctx, tables, exec_mode=exec_mode, resolution=res)
    q.execute(E, **kw)  # warm-up (compiles the plan's kernels)
    ctx.enable_timing(True)
    ctx.kernel_times()
    out = None
    ts = []
    for _ in range(reps):
        if exec_mode == hq.EXEC_OAAT:  # many kernels + host syncs: wall clock around the plan
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            out, _pb = q.run(E, **kw)
            torch.cuda.synchronize()
            ts.append((time.perf_counter() - t0) * 1e3)
        else:
            out, _pb = q.run(E, **kw)
            ts += ctx.kernel_times()
    ctx.enable_timing(False)
    return float(np.median(ts)), out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--sf", type=float, default=10)
    ap.add_argument("--reps", type=int, default=5)
    a = ap.parse_args()
    torch.cuda.set_device(0)
    ctx = hq.Context(0)
    res = {"sf": a.sf, "exp1": [], "g1": [], "exp2": []}
    tables = load_tables(ctx, QUERIES["micro_select"], a.sf)
    n = int(next(iter(tables.values())).nrows)
    res["rows"] = n
    for x in (-1, 0, 2, 5, 12, 24):
        sel = max(0, 2 * x + 1) / 50.0
        row = {"x": x, "selectivity": sel}
        for tech, (em, rr) in MODES.items():
            row["A" + tech], r = timed(ctx, tables, QUERIES["micro_select"], em, rr, a.reps, x=x)
            row["qualifying"] = int(r.qualifying())
            row["B" + tech], _ = timed(ctx, tables, QUERIES["micro_sum"], em, rr, a.reps, x=x)
        row["A_oaat"], _ = timed(ctx, tables, QUERIES["micro_select"], hq.EXEC_OAAT, hq.RES_LRGP, a.reps, x=x)
        res["exp1"].append(row)
        print("exp1/g1", json.dumps(row), flush=True)
    del tables
    tables = load_tables(ctx, QUERIES["micro_groupby"], a.sf)
    for x in (2, 8, 32, 128, 512, 2048, 8192, 16384):
        row = {"groups": x}
        for tech, (em, rr) in MODES.items():
            row["C" + tech], r = timed(ctx, tables, QUERIES["micro_groupby"], em, rr, a.reps, x=x)
        row["C_oaat"], _ = timed(ctx, tables, QUERIES["micro_groupby"], hq.EXEC_OAAT, hq.RES_LRGP, a.reps, x=x)
        res["exp2"].append(row)
        print("exp2", json.dumps(row), flush=True)
    d = os.path.join(ROOT, "gpurun_out")
    os.makedirs(d, exist_ok=True)
    with open(os.path.join(d, "micro_sweeps.json"), "w") as f:
        json.dump(res, f, indent=1)
    L = [f"Reduction micro-benchmarks on one B200, SSB lineorder SF {a.sf:g} ({n} rows, resident in HBM); "
         "pipeline device time in ms (median of "
         f"{a.reps}); 1 = multi-pass (count kernel, prefix sum, write kernel, library reduce/sort), 2 = per-row global "
         "atomics, 3 = local resolution + global propagation (LRGP with SIMD-style warp resolution, the default), 3WE = "
         "the same with work-efficient (Blelloch) resolution over the workgroup (App C, Fig 24); op-at-a-time = wall "
         "clock around the plan (its kernels plus host synchronisations).", "",
         "Exp 1 / App G.1: `lo_quantity BETWEEN 25-x AND 25+x`, revenue = extendedprice*discount+tax; A = materialised, "
         "B = single-tuple SUM", "",
         "| x | selectivity | A1 | A2 | A3 (SIMD) | A3-WE | A op-at-a-time | B1 | B2 | B3 (SIMD) | B3-WE |",
         "|---|---|---|---|---|---|---|---|---|---|---|"]
    for r in res["exp1"]:
        L.append(f"| {r['x']} | {r['selectivity']:.2f} | {r['A1']:.3f} | {r['A2']:.3f} | {r['A3']:.3f} | {r['A3WE']:.3f} | "
                 f"{r['A_oaat']:.3f} | {r['B1']:.3f} | {r['B2']:.3f} | {r['B3']:.3f} | {r['B3WE']:.3f} |")
    L += ["", "Exp 2: `SUM(lo_extendedprice) GROUP BY lo_orderkey % x`", "",
          "| groups | C1 | C2 | C3 (SIMD) | C3-WE | C op-at-a-time |", "|---|---|---|---|---|---|"]
    for r in res["exp2"]:
        L.append(f"| {r['groups']} | {r['C1']:.3f} | {r['C2']:.3f} | {r['C3']:.3f} | {r['C3WE']:.3f} | {r['C_oaat']:.3f} |")
    with open(os.path.join(d, "micro_sweeps.md"), "w") as f:
        f.write("\n".join(L) + "\n")
    print("\n".join(L))


if __name__ == "__main__":
    main()
