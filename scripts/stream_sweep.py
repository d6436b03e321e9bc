#!/usr/bin/env python
"""Batch processing (SURVEY.md §8(f) f4 i; PAPER.md Exp 5): the fact
table stays in pinned host memory and streams through the fused kernel in blocks
(double-buffered device ring, copies on their own stream).  For each block size:
the streamed pipeline time (CUDA events from before the first copy to after the
last kernel), the fact bytes / time (host-link GB/s), against (a) the measured
pinned host->device copy bandwidth of the same bytes (the roofline of this mode)
and (b) copy-then-run: one HQ_HOST_COPY load of the whole fact table followed by
the HBM-resident pipeline.  Writes gpurun_out/stream_sweep_<query>_sf<sf>.{json,md}.

    python scripts/stream_sweep.py --query ssb_q41 --sf 30
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
from paper_conf_sigmod_funkebnmt18_b200.queries import QUERIES  # noqa: E402


def events_ms(fn, reps):
    s = torch.cuda.current_stream()
    ts = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record(s)
        fn()
        e1.record(s)
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    return float(np.median(ts))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--query", default="ssb_q41")
    ap.add_argument("--sf", type=float, default=30)
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--blocks", default="65536,262144,1048576,4194304,16777216")
    ap.add_argument("--no-copy-then-run", action="store_true")
    a = ap.parse_args()
    torch.cuda.set_device(0)
    ctx = hq.Context(0)
    q = QUERIES[a.query]
    tabs = hqgen.SSB_TABLES if q.bench == "ssb" else hqgen.TPCH_TABLES
    host = {t: hqgen.generate(t, a.sf, columns=q.columns[t]) for t in q.columns if t in tabs and t != q.fact}
    # the fact columns are generated straight into pinned host buffers (SF300: 43 GB)
    nf = hqgen.table_rows(q.fact, a.sf)
    schema = dict(hqgen.SCHEMAS[hqgen.TABLE_NAMES[q.fact]])
    tdt = {"i1": torch.int8, "i4": torch.int32, "i8": torch.int64}
    fact = {c: torch.empty(nf, dtype=tdt[schema[c]], pin_memory=True) for c in q.columns[q.fact]}
    hqgen.generate(q.fact, a.sf, columns=q.columns[q.fact], out={c: t.numpy() for c, t in fact.items()})
    n = int(next(iter(fact.values())).numel())
    nbytes = sum(int(t.numel() * t.element_size()) for t in fact.values())
    dims = {t: ctx.load_columns({c: host[t][c] for c in cols}) for t, cols in q.columns.items() if t != q.fact}
    # (a) the host-link roofline: one pinned H2D copy of the same bytes
    dev = {c: torch.empty_like(t, device="cuda") for c, t in fact.items()}
    h2d = events_ms(lambda: [dev[c].copy_(fact[c], non_blocking=True) for c in fact], a.reps)
    # HBM-resident reference: the fused pipeline over device columns
    Er = Engine(ctx, {**dims, q.fact: ctx.load_columns(dev)})
    ref = q.execute(Er)
    resident = events_ms(lambda: q.run(Er), a.reps)
    # (b) copy-then-run: HQ_HOST_COPY load + pipeline
    def copy_then_run():
        E = Engine(ctx, {**dims, q.fact: ctx.load_columns(fact)})
        q.run(E)
    seq = float("nan") if a.no_copy_then_run else events_ms(copy_then_run, a.reps)
    st = ctx.load_columns(fact, stream=True)
    rows = []
    for b in [int(x) for x in a.blocks.split(",")]:
        E = Engine(ctx, {**dims, q.fact: st}, stream_block=b)
        got = q.execute(E)
        same = got.rows() == ref.rows() and got.qualifying == ref.qualifying
        if not same:
            print("DIFF", b, got.qualifying, ref.qualifying, [(x, y) for x, y in zip(got.rows(), ref.rows()) if x != y][:3],
                  flush=True)
        ms = events_ms(lambda: q.run(E), a.reps)
        again = q.execute(E)
        same = same and again.rows() == ref.rows()
        row = {"block_rows": b, "block_mb": b * nbytes / n / 1e6, "device_ring_mb": 2 * b * nbytes / n / 1e6,
               "ms": ms, "gbs": nbytes / ms / 1e6,
               "frac_of_h2d": h2d / ms, "identical_to_resident": same}
        rows.append(row)
        print(json.dumps(row), flush=True)
    out = {"query": a.query, "sf": a.sf, "fact_rows": n, "fact_bytes": nbytes, "h2d_ms": h2d,
           "h2d_gbs": nbytes / h2d / 1e6, "resident_query_ms": resident, "copy_then_run_ms": seq, "streamed": rows}
    d = os.path.join(ROOT, "gpurun_out")
    os.makedirs(d, exist_ok=True)
    tag = f"{a.query}_sf{a.sf:g}"
    with open(os.path.join(d, f"stream_sweep_{tag}.json"), "w") as f:
        json.dump(out, f, indent=1)
    assert all(r["identical_to_resident"] for r in rows), "a streamed result differs from the resident one"
    L = [f"Batch processing of {a.query} SF {a.sf:g}: {n} fact rows, {nbytes / 1e9:.2f} GB of referenced fact columns "
         f"in pinned host memory. Pinned H2D copy of the same bytes: {h2d:.1f} ms ({nbytes / h2d / 1e6:.1f} GB/s, the "
         f"roofline of this mode). HBM-resident query: {resident:.2f} ms. Copy-then-run (HQ_HOST_COPY load + query): "
         f"{seq:.1f} ms. Streamed (CUDA events, median of {a.reps}; results identical to the resident run):", "",
         "| block rows | block MB | device ring MB | streamed ms | host-link GB/s | of pinned H2D |",
         "|---|---|---|---|---|---|"]
    for r in rows:
        L.append(f"| {r['block_rows']} | {r['block_mb']:.1f} | {r['device_ring_mb']:.1f} | {r['ms']:.1f} | {r['gbs']:.1f} | "
                 f"{r['frac_of_h2d']:.2f} |")
    with open(os.path.join(d, f"stream_sweep_{tag}.md"), "w") as f:
        f.write("\n".join(L) + "\n")
    print("\n".join(L))


if __name__ == "__main__":
    main()
