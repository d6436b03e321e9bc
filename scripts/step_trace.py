#!/usr/bin/env python
"""GPU timeline of one query step (CUPTI through torch.profiler): every kernel and
memcpy of the step with its start offset and duration, the idle gaps between them,
and the CUDA runtime calls that block the host (stream syncs) -- where the time
outside the fused kernel goes.

    python scripts/step_trace.py --query ssb_q41 --sf 100 [--steps 3] [--json out.json] [--dist]

--dist: the distributed engine (dist.DistributedEngine over NCCL) at world size 1 -- the
fixed cost of its collectives and fault exchange over the single-device step.
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_sigmod_funkebnmt18_b200 import hq  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200.engine import Engine  # noqa: E402
from paper_conf_sigmod_funkebnmt18_b200.queries import QUERIES, load_tables  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--query", default="ssb_q41")
    ap.add_argument("--sf", type=float, default=10)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--json", default="")
    ap.add_argument("--dist", action="store_true")
    ap.add_argument("--broadcast", action="store_true", help="--dist with the root-broadcast design")
    a = ap.parse_args()
    torch.cuda.set_device(0)
    q = QUERIES[a.query]
    ctx = hq.Context(0)
    tables = load_tables(ctx, q, a.sf)
    ctx.sync()
    if a.dist:
        import torch.distributed as dist
        from paper_conf_sigmod_funkebnmt18_b200.dist import DistributedEngine, run_query
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ.setdefault("MASTER_PORT", "29571")
        dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
        E = DistributedEngine(ctx, tables, replicated=not a.broadcast)

        def execute():
            return run_query(E, q)
    else:
        E = Engine(ctx, tables)

        def execute():
            return q.execute(E)
    for _ in range(3):
        execute()
    torch.cuda.synchronize()
    from torch.profiler import ProfilerActivity, profile
    marker = torch.zeros(1024, device="cuda")
    with profile(activities=[ProfilerActivity.CPU, ProfilerActivity.CUDA]) as prof:
        for _ in range(a.steps):
            torch.cuda.synchronize()
            with torch.profiler.record_function("hq_step"):
                marker.mul_(1.5)  # a step-start marker kernel on the GPU timeline
                execute()
            torch.cuda.synchronize()
    evs = prof.events()
    hsteps = sorted([e for e in evs if e.name == "hq_step" and e.device_type == torch.autograd.DeviceType.CPU],
                    key=lambda e: e.time_range.start)
    gpu = sorted([e for e in evs if e.device_type == torch.autograd.DeviceType.CUDA and e.name != "hq_step"],
                 key=lambda e: e.time_range.start)
    syncs = [e for e in evs if e.device_type == torch.autograd.DeviceType.CPU and "Synchronize" in e.name]
    # GPU ops of step k: from its marker kernel to the next marker (CPU and GPU clocks may differ)
    mk = [i for i, e in enumerate(gpu) if "MulFunctor" in e.name]
    out = []
    for si, st in enumerate(hsteps):
        if si >= len(mk):
            break
        lo, hi = mk[si], (mk[si + 1] if si + 1 < len(mk) else len(gpu))
        ks = gpu[lo + 1:hi]
        t0, t1 = st.time_range.start, st.time_range.end
        ss = [e for e in syncs if t0 <= e.time_range.start <= t1]
        g0 = gpu[lo].time_range.end
        rows = []
        prev = None
        busy = 0.0
        for e in ks:
            s, d = e.time_range.start - g0, e.time_range.end - e.time_range.start
            gap = (e.time_range.start - prev) if prev is not None else s
            prev = max(prev or 0, e.time_range.end)
            busy += d
            rows.append({"name": e.name[:70], "start_us": s, "dur_us": d, "gap_before_us": gap})
        span = (ks[-1].time_range.end - g0) if ks else 0.0
        rec = {"step": si, "host_us": t1 - t0, "gpu_span_us": span, "gpu_busy_us": busy, "n_gpu_ops": len(ks),
               "syncs": [{"name": x.name, "start_us": x.time_range.start - t0,
                          "dur_us": x.time_range.end - x.time_range.start} for x in ss], "ops": rows}
        out.append(rec)
        print(f"step {si}: host {rec['host_us']:.1f} us, GPU span {span:.1f} us, busy {busy:.1f} us over {len(ks)} ops, "
              f"{len(ss)} host syncs ({sum(x['dur_us'] for x in rec['syncs']):.1f} us blocked)")
        if si == len(hsteps) - 1:
            for r in rows:
                print(f"  +{r['start_us']:9.1f} us  gap {r['gap_before_us']:8.1f}  dur {r['dur_us']:9.1f}  {r['name']}")
            for x in rec["syncs"]:
                print(f"  host sync at +{x['start_us']:.1f} us (host clock) for {x['dur_us']:.1f} us ({x['name']})")
    if a.json:
        with open(a.json, "w") as f:
            json.dump({"query": a.query, "sf": a.sf, "steps": out}, f, indent=1)


if __name__ == "__main__":
    main()
