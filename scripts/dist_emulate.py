#!/usr/bin/env python
"""N-way multi-GPU emulation on one B200 (the driver has no 8-GPU node): for N in
1, 2, 4, 8 the work of ONE rank -- the full dimension builds and the fused pipeline over
its 1/N range partition of the fact table, finalize -- is timed on the device (eager
steps with the fused kernel timed, and the prepared CUDA-graph step).  The ranks of a
range partition are symmetric (uniform synthetic data), so the emulated N-GPU job time
is one rank's time plus the collectives; reported as whole-job rows/s:
pipeline-only = N_rows / fused kernel time, step = N_rows / rank step time.
Co-partitioned queries (Query.copart, TPC-H Q3): the rank's orders AND lineitem
co-partition (hqgen.copartition), every build local -- the rank's whole step.

    python scripts/dist_emulate.py --query ssb_q41 --sf 100 [--steps 10]
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import hqgen  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200 import hq  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200.dist import partition  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200.engine import Engine  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200.queries import QUERIES, load_tables  # noqa: E402


def timed(fn, k):
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(k + 1)]
    torch.cuda.synchronize()
    ev[0].record()
    for i in range(k):
        fn()
        ev[i + 1].record()
    torch.cuda.synchronize()
    return [ev[i].elapsed_time(ev[i + 1]) for i in range(k)]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--query", default="ssb_q41")
    ap.add_argument("--sf", type=float, default=100)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--out", default="")
    a = ap.parse_args()
    torch.cuda.set_device(0)
    q = QUERIES[a.query]
    n = hqgen.table_rows(q.fact, a.sf)
    ctx = hq.Context(0)
    dims = {t: cols for t, cols in q.columns.items() if t != q.fact and t != q.copart}
    host_dims = {t: hqgen.generate(t, a.sf, columns=cols) for t, cols in dims.items()}
    out = {"query": a.query, "sf": a.sf, "fact_rows": n, "copartitioned": q.copart is not None, "per_n": []}
    for N in (1, 2, 4, 8):
        crange = None
        if q.copart is not None:
            crange, (lo, hi) = hqgen.copartition(q.fact, q.copart, a.sf, 0, N)
        else:
            lo, hi = partition(n, 0, N)
        tables = load_tables(ctx, q, a.sf, fact_range=(lo, hi), host=host_dims, copart_range=crange)
        E = Engine(ctx, tables)
        for _ in range(3):
            q.execute(E)
        ctx.kernel_times()
        ctx.enable_timing(True)
        eager = timed(lambda: q.execute(E), a.steps)
        kt = ctx.kernel_times()
        ctx.enable_timing(False)
        per = max(1, len(kt) // a.steps)
        kern = statistics.median([max(kt[i:i + per]) for i in range(0, per * a.steps, per)])
        try:
            pq = E.prepare(q)
            for _ in range(3):
                pq.execute()
            step = statistics.median(timed(pq.execute, a.steps))
            pq.close()
            mode = "prepared"
        except hq.HQError:  # not capturable (TPC-H Q3): the eager step
            step, mode = statistics.median(eager), "eager"
        rec = {"n_gpus": N, "rank_rows": hi - lo, "kernel_ms": kern, "eager_step_ms": statistics.median(eager),
               "step_ms": step, "step_mode": mode,
               "pipeline_rows_per_s": n / (kern / 1e3), "step_rows_per_s": n / (step / 1e3),
               "step_over_kernel": step / kern}
        out["per_n"].append(rec)
        print(json.dumps(rec), flush=True)
        del E, tables
        torch.cuda.empty_cache()
    if a.out:
        with open(a.out, "w") as f:
            json.dump(out, f, indent=1)


if __name__ == "__main__":
    main()
