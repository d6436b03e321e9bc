#!/usr/bin/env python
"""Fact-column placement experiment: the same query with its fact columns loaded
separately (HQ_HOST_COPY, one allocation per column) and borrowed from ONE device
buffer at chosen offsets (HQ_DEVICE_BORROW): back to back, 4 GiB apart (congruent
addresses), and skewed.  Reports the fused kernel's CUDA-event time per layout.

    python scripts/exp_col_layout.py --query ssb_q41 --sf 100 [--reps 7]
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
from paper_conf_sigmod_funkebnmt18_b200.engine import Engine  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200.queries import QUERIES, load_tables  # noqa: E402


def align(x, a):
    return (x + a - 1) // a * a


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--query", default="ssb_q41")
    ap.add_argument("--sf", type=float, default=100)
    ap.add_argument("--reps", type=int, default=7)
    ap.add_argument("--layouts", default="sep,packed,pow2,skew,skew2")
    a = ap.parse_args()
    torch.cuda.set_device(0)
    q = QUERIES[a.query]
    ctx = hq.Context(0)
    tables = load_tables(ctx, q, a.sf)
    host_fact = hqgen.generate(q.fact, a.sf, columns=q.columns[q.fact])
    names = list(host_fact)
    nb = [host_fact[c].nbytes for c in names]
    out = {"query": a.query, "sf": a.sf, "layouts": {}}
    for lay in a.layouts.split(","):
        if lay == "sep":
            t = tables
        else:
            if lay == "packed":
                offs = [sum(align(b, 256) for b in nb[:k]) for k in range(len(nb))]
            elif lay == "pow2":
                offs = [k * (1 << 32) for k in range(len(nb))]
            elif lay == "skew":  # 2 MiB-aligned slots plus k x 41 x 256 B
                slot = align(max(nb), 1 << 21)
                offs = [k * slot + k * 41 * 256 for k in range(len(nb))]
            else:  # skew2: k x (slot + 1 MiB + 4 KiB)
                slot = align(max(nb), 1 << 21)
                offs = [k * (slot + (1 << 20) + 4096) for k in range(len(nb))]
            total = offs[-1] + nb[-1] + 4096
            buf = torch.empty(total, dtype=torch.uint8, device="cuda")
            cols = {}
            for c, o, b in zip(names, offs, nb):
                h = torch.from_numpy(host_fact[c].view("uint8"))
                buf[o:o + b].copy_(h)
                cols[c] = buf[o:o + b].view({1: torch.int8, 4: torch.int32, 8: torch.int64}[host_fact[c].itemsize])
            t = dict(tables)
            t[q.fact] = ctx.load_columns(cols)
        E = Engine(ctx, t)
        for _ in range(2):
            q.execute(E)
        ctx.kernel_times()
        ctx.enable_timing(True)
        for _ in range(a.reps):
            q.execute(E)
        kt = ctx.kernel_times()
        ctx.enable_timing(False)
        med = statistics.median(kt[-a.reps:])
        gbs = sum(nb) / med / 1e6
        out["layouts"][lay] = {"kernel_ms": round(med, 4), "GB/s": round(gbs, 1)}
        print(lay, round(med, 4), "ms", round(gbs, 1), "GB/s", flush=True)
        del E, t
        if lay != "sep":
            del buf, cols
        torch.cuda.synchronize()
    print(json.dumps(out))


if __name__ == "__main__":
    main()
