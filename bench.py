#!/usr/bin/env python
"""bench.py -- fact rows/s of the fused query pipeline on B200 (driver contract).

Default workload: SSB Q4.1 at SF 100 (600 M lineorder rows, 24 B/row = 14.4 GB of
referenced fact columns), the BASELINE.json config quoted "partitioned across
1/2/4/8 B200" (configs[4]).  One *step* = one full query: the four dimension
hash builds (root builds + NCCL broadcast when N>1), the fused probe/aggregate
pipeline over the (local) fact range, the partial-aggregate reduce (N>1) and
finalisation + result fetch on rank 0.  Columns are HBM-resident when the timed
region starts (14.4 GB >> 126 MB L2, so no flush is needed between steps).

Also reported: the dominant kernel's roofline (algorithmic bytes / measured
kernel time vs MEASURED_PEAKS.json's HBM copy bandwidth), e2e through the C ABI
from pinned host buffers, the CPU oracle on a bounded sample (cpu_baseline),
SM clocks during the timed region and the number of libhq kernel launches.
At N=1 the other BASELINE.json configs are measured too ("per_query").

    python bench.py [--gpus N] [--steps K] [--warmup W] [--query Q --sf S] [--impl reference]
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import hqgen  # noqa: E402

DEFAULT_QUERY, DEFAULT_SF = "ssb_q41", 100.0
# other BASELINE.json configs, measured at N=1 into "per_query"
EXTRA = [("tpch_q6", 10.0), ("tpch_q1", 10.0), ("ssb_q11", 10.0), ("ssb_q12", 10.0), ("ssb_q13", 10.0),
         ("ssb_q31", 30.0), ("tpch_q3", 30.0)]
METRIC = "fact rows/s per query"


# ----------------------------------------------------------------- helpers
def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy read+write)"
    return 6650.0, "fallback (B200_PROFILING.md: 6.65 TB/s)"


class ClockSampler:
    """Samples SM clocks and clock-event reasons with NVML during the timed region."""

    REASONS = {0x4: "sw_power_cap", 0x8: "hw_slowdown", 0x20: "sw_thermal_slowdown",
               0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown", 0x2: "applications_clocks_setting"}

    def __init__(self, device_index: int):
        self.samples, self.reasons, self.ok = [], set(), False
        try:
            import pynvml
            import torch
            pynvml.nvmlInit()
            pr = torch.cuda.get_device_properties(device_index)
            bus = f"{pr.pci_domain_id:08x}:{pr.pci_bus_id:02x}:{pr.pci_device_id:02x}.0"
            self.h = pynvml.nvmlDeviceGetHandleByPciBusId(bus)
            self.max = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.nv = pynvml
            self.ok = True
        except Exception as e:  # noqa: BLE001
            self.err = str(e)

    def _run(self):
        while not self.stop:
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                r = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for bit, name in self.REASONS.items():
                    if r & bit:
                        self.reasons.add(name)
            except Exception:  # noqa: BLE001
                pass
            time.sleep(0.005)  # ~5 samples over a 10-step timed region of the headline query

    def __enter__(self):
        self.stop = False
        if self.ok:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        self.stop = True
        if self.ok:
            self.t.join()

    def summary(self):
        if not self.ok:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "error": getattr(self, "err", "")}
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None, "sm_max_mhz": self.max,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


def gen_host(q, sf, seed, fact_range, with_dims, pinned=True, copart_range=None):
    """Referenced columns as numpy arrays (pinned host memory for the fact table).
    copart_range: this rank's rows of the co-partitioned order table (q.copart)."""
    import torch
    host = {}
    for t, cols in q.columns.items():
        if t != q.fact and not with_dims:
            continue
        rr = fact_range if t == q.fact else (copart_range if t == q.copart else None)
        n = (rr[1] - rr[0]) if rr else hqgen.table_rows(t, sf, seed)
        out = None
        if pinned and t == q.fact:
            schema = dict(hqgen.SCHEMAS[hqgen.TABLE_NAMES[t]])
            tdt = {"i1": torch.int8, "i4": torch.int32, "i8": torch.int64}
            out = {c: torch.empty(n, dtype=tdt[schema[c]], pin_memory=True).numpy() for c in cols}
        host[t] = hqgen.generate(t, sf, seed, columns=cols, row_range=rr, out=out)
    return host


def oracle_call(qname, host, nthreads, fact_rows=None):
    """The CPU oracle on the first `fact_rows` fact rows (bounded sample)."""
    import oracle
    from paper_conf_sigmod_funkebnmt18_b200.queries import QUERIES
    q = QUERIES[qname]
    t = {k: dict(v) for k, v in host.items()}
    if fact_rows is not None:
        t[q.fact] = {c: a[:fact_rows] for c, a in t[q.fact].items()}
    f = {
        "tpch_q6": lambda: oracle.tpch_q6(t["lineitem"], nthreads),
        "tpch_q1": lambda: oracle.tpch_q1(t["lineitem"], nthreads),
        "ssb_q11": lambda: oracle.ssb_q1(1, t["lineorder"], t["date"], nthreads=nthreads),
        "ssb_q12": lambda: oracle.ssb_q1(2, t["lineorder"], t["date"], nthreads=nthreads),
        "ssb_q13": lambda: oracle.ssb_q1(3, t["lineorder"], t["date"], nthreads=nthreads),
        "ssb_q31": lambda: oracle.ssb_q31(t["lineorder"], t["customer"], t["supplier"], t["date"], nthreads=nthreads),
        "ssb_q41": lambda: oracle.ssb_q41(t["lineorder"], t["date"], t["customer"], t["supplier"], t["part"],
                                          nthreads=nthreads),
        "tpch_q3": lambda: oracle.tpch_q3(t["tpch_customer"], t["orders"], t["lineitem"], nthreads=nthreads),
    }[qname]
    t0 = time.perf_counter()
    f()
    return time.perf_counter() - t0


def cpu_baseline(qname, host, n_fact, budget_s=30.0):
    """Time the oracle (as it stands, all host cores) on the whole workload, or on
    a prefix sample when the whole would take longer than ~budget_s."""
    cores = os.cpu_count() or 1
    s0 = min(n_fact, 2_000_000)
    dt0 = oracle_call(qname, host, cores, s0)  # includes the dimension hash-map builds
    est = dt0 * n_fact / max(s0, 1)
    s = n_fact if est <= budget_s else max(s0, int(n_fact * budget_s / est))
    dt = oracle_call(qname, host, cores, s)
    # the oracle single-threaded too (a bounded prefix)
    s1 = min(n_fact, 4_000_000)
    dt1 = oracle_call(qname, host, 1, s1)
    return {"value": s / dt, "unit": "rows/s", "cores": cores, "kind": "oracle",
            "sample": f"first {s} of {n_fact} fact rows (full dimension tables), tuple-at-a-time C++ oracle, "
                      f"{cores} threads, {dt:.2f} s",
            "single_thread": {"value": s1 / dt1, "unit": "rows/s", "cores": 1,
                              "sample": f"first {s1} fact rows, 1 thread, {dt1:.2f} s"}}


def exec_timing(qname, host, local, fused_ms, mode="oaat", steps=2):
    """The same query executed operator-at-a-time (Fig 6 baseline, HQ_EXEC_OAAT)
    or by multi-pass query compilation (Fig 7-9, HQ_EXEC_MULTIPASS): device time
    per step with CUDA events, vs the fused step."""
    import torch
    from paper_conf_sigmod_funkebnmt18_b200 import hq
    from paper_conf_sigmod_funkebnmt18_b200.engine import Engine
    from paper_conf_sigmod_funkebnmt18_b200.queries import QUERIES
    q = QUERIES[qname]
    dev = torch.device("cuda", local)
    ctx = hq.Context(local)
    dtab = {t: {c: torch.from_numpy(np.asarray(a)).to(dev) for c, a in cols.items()} for t, cols in host.items()}
    tables = {t: ctx.load_columns(cols) for t, cols in dtab.items()}
    em = {"oaat": hq.EXEC_OAAT, "multipass": hq.EXEC_MULTIPASS}[mode]
    E = Engine(ctx, tables, exec_mode=em)
    q.execute(E)
    stream = torch.cuda.current_stream(dev)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record(stream)
    for _ in range(steps):
        q.execute(E)
    e1.record(stream)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / steps
    del tables, dtab, E
    ctx.close()
    torch.cuda.empty_cache()
    return {"ms_per_step": ms, "fused_speedup": ms / fused_ms, "steps": steps,
            "exec": {"oaat": "HQ_EXEC_OAAT", "multipass": "HQ_EXEC_MULTIPASS"}[mode]}


# --------------------------------------------------------- device measurement
def measure(qname, sf, steps, warmup, seed, rank, world, local, with_e2e=True, host=None):
    import torch
    import torch.distributed as dist
    from paper_conf_sigmod_funkebnmt18_b200 import hq
    from paper_conf_sigmod_funkebnmt18_b200.dist import DistributedEngine, partition, run_query
    from paper_conf_sigmod_funkebnmt18_b200.engine import Engine
    from paper_conf_sigmod_funkebnmt18_b200.queries import QUERIES

    q = QUERIES[qname]
    dev = torch.device("cuda", local)
    n = hqgen.table_rows(q.fact, sf, seed)
    a, b = partition(n, rank, world)
    root = rank == 0
    dist_mode = world > 1 or os.environ.get("HQ_FORCE_DIST") == "1"
    # co-partitioned queries (TPC-H Q3): orders and lineitem partitioned together by order,
    # every rank builds locally (dist.DistributedEngine copartitioned)
    copart = dist_mode and q.copart is not None and os.environ.get("HQ_DIST_COPART", "1") == "1"
    # dimension tables replicated on every rank and built there (no table broadcast);
    # HQ_DIST_BROADCAST=1: the root builds and broadcasts them
    replicated = dist_mode and not copart and os.environ.get("HQ_DIST_BROADCAST") != "1"
    crange = None
    if copart:
        crange, (a, b) = hqgen.copartition(q.fact, q.copart, sf, rank, world, seed)
    if host is None:
        host = gen_host(q, sf, seed, (a, b), with_dims=root or world == 1 or copart or replicated,
                        copart_range=crange)
    ctx = hq.Context(local)
    # HBM-resident copies (torch memory, borrowed by libhq)
    dtab = {t: {c: torch.from_numpy(np.asarray(arr)).to(dev) for c, arr in cols.items()} for t, cols in host.items()}
    torch.cuda.synchronize()
    tables = {t: ctx.load_columns(cols) for t, cols in dtab.items()}

    def make_engine(tbls):
        # HQ_FORCE_DIST=1 runs the distributed engine (broadcast + reduce) even at N=1
        if dist_mode:
            return DistributedEngine(ctx, tbls, copartitioned=copart, replicated=replicated)
        return Engine(ctx, tbls)

    E = make_engine(tables)

    def step(Eng):
        return run_query(Eng, q)

    def barrier():
        if world > 1:
            dist.barrier()

    stream = torch.cuda.current_stream(dev)

    def timed(run_step, k):
        """k steps between a barrier + sync on both sides; CUDA events on the stream
        between the steps (per-step times for the median / min)."""
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(k + 1)]
        barrier()
        torch.cuda.synchronize()
        ev[0].record(stream)
        o = None
        for i in range(k):
            o = run_step()
            ev[i + 1].record(stream)
        torch.cuda.synchronize()
        barrier()
        per = [ev[i].elapsed_time(ev[i + 1]) for i in range(k)]
        return ev[0].elapsed_time(ev[k]) / k, per, o

    for _ in range(warmup):
        out = step(E)
    # eager steps (the plan built by the host every step), with the fused kernels timed
    ctx.kernel_times()
    ctx.enable_timing(True)
    l0 = ctx.launches()
    with ClockSampler(local) as clk:
        ms_eager, per_eager, out = timed(lambda: step(E), steps)
    launches_eager = ctx.launches() - l0
    kt = ctx.kernel_times()
    ctx.enable_timing(False)
    per_step = max(1, len(kt) // steps)
    # the dominant kernel: the longest fused launch of each step (the fact-table pipeline)
    fact_kt = [max(kt[i:i + per_step]) for i in range(0, per_step * steps, per_step)] if kt else []
    kms = statistics.mean(fact_kt) if fact_kt else float("nan")
    # prepared query (CUDA graph of the whole step: builds + fused pipeline + finalize
    # re-executed every launch; include/hq.h "prepared queries") where the plan is static
    prep = None
    # (distributed: the two-graph prepared step of dist.PreparedDistQuery, replicated dimensions)
    if os.environ.get("HQ_BENCH_EAGER") != "1" and ((not dist_mode) or replicated):
        try:
            pq = E.prepare(q)
            for _ in range(warmup):
                pq.execute()
            l1 = ctx.launches()
            with ClockSampler(local) as clk2:
                ms_prep, per_prep, out_p = timed(pq.execute, steps)
            if (out_p is None) != (out is None) or (out_p is not None and out_p.rows() != out.rows()):
                raise RuntimeError("prepared result differs from the eager one")
            prep = {"ms": ms_prep, "per": per_prep, "launches": ctx.launches() - l1, "clocks": clk2.summary()}
            pq.close()
        except Exception as e:  # noqa: BLE001 -- a query the graph cannot hold runs eagerly
            prep = {"error": str(e)[:200]}
    ms, per, launches, clocks = ms_eager, per_eager, launches_eager, clk.summary()
    mode = "eager"
    if prep and "ms" in prep:
        ms, per, launches, clocks, mode = prep["ms"], prep["per"], prep["launches"], prep["clocks"], "prepared"
    if world > 1:
        t = torch.tensor([ms], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())

    res = {"ms": ms, "kernel_ms": kms, "launches": launches, "clocks": clocks, "rows": n,
           "local_rows": b - a, "result": out, "mode": mode, "step_ms_median": statistics.median(per),
           "step_ms_min": min(per), "eager": {"ms_per_step": ms_eager, "median": statistics.median(per_eager),
                                               "min": min(per_eager), "launches": launches_eager},
           "prepared": prep, "copart": copart, "replicated": replicated}
    # ---- e2e: host (pinned) buffers through the public API, H2D inside the timed region.
    # Dimension tables are copied (HQ_HOST_COPY); the fact table streams from its pinned
    # host buffers through the fused kernel in blocks (HQ_HOST_STREAM, batch processing:
    # block b+1 crosses the host link while block b is processed, SURVEY.md §8(f) f4 i).
    if with_e2e:
        e2e_steps = max(1, min(steps, 3))
        h2d = sum(arr.nbytes for cols in host.values() for arr in cols.values())

        def e2e_step():
            tb = {t: ctx.load_columns(cols, stream=(t == q.fact)) for t, cols in host.items()}
            Eng = make_engine(tb)
            o = run_query(Eng, q)
            d2h = sum(c.nbytes for c in o.columns.values()) if o is not None else 0
            del Eng, tb
            return d2h

        e2e_step()
        barrier()
        torch.cuda.synchronize()
        f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        f0.record(stream)
        d2h = 0
        for _ in range(e2e_steps):
            d2h = e2e_step()
        f1.record(stream)
        torch.cuda.synchronize()
        barrier()
        ems = f0.elapsed_time(f1) / e2e_steps
        if world > 1:
            t = torch.tensor([ems], device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ems = float(t.item())
        res["e2e"] = {"value": n / (ems / 1e3), "unit": "rows/s", "h2d_bytes_per_step": int(h2d),
                      "d2h_bytes_per_step": int(d2h), "ms_per_step": ems, "steps": e2e_steps,
                      "mode": f"fact table streamed from pinned host memory (HQ_HOST_STREAM, {hq.STREAM_BLOCK_ROWS}-row "
                              "blocks, copies overlapped with the fused kernel); dimensions HQ_HOST_COPY"}
    res["host"] = host
    del tables, dtab, E
    ctx.close()
    torch.cuda.empty_cache()
    return res


def bytes_ratio(qname, sf):
    """Fused vs multi-pass vs operator-at-a-time DRAM bytes of this query, as measured by
    scripts/bytes_ratio.py under ncu at the bench's scale factor (profiles/r02), with the
    paper's GTX 970 figures beside it."""
    for rel in ("profiles/r02/bytes_ratio_bench_sfs.json", "profiles/r01/bytes_ratio_sf10.json"):
        p = os.path.join(ROOT, rel)
        if not os.path.exists(p):
            continue
        br = json.load(open(p))["queries"].get(qname)
        if not br:
            continue
        f, o = br["fused"]["pipeline"]["dram_bytes"], br["oaat"]["pipeline"]["dram_bytes"]
        ft, ot = br["fused"]["pipeline"]["time_s"], br["oaat"]["pipeline"]["time_s"]
        out = {"ratio": o / f, "fused_bytes": f, "oaat_bytes": o, "kernel_time_ratio": ot / max(ft, 1e-12),
               "sf": br.get("sf", 10), "bench_sf": sf, "source": rel + " (scripts/bytes_ratio.py: ncu, --cache-control all)",
               "paper": "up to 7.5x memory volume and 9.5x kernel time, fused vs operator-at-a-time, GTX 970 "
                        "(PAPER.md P:40-42)"}
        if "multipass" in br:
            m = br["multipass"]["pipeline"]["dram_bytes"]
            out.update({"multipass_bytes": m, "multipass_ratio": m / f})
        return out
    return None


def roofline(q, local_rows, kernel_ms, peak, peak_src):
    bpr = q.fact_bytes_per_row()
    traffic = None
    tp = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tp):
        with open(tp) as f:
            tr = json.load(f)
        e = tr.get(q.name)
        if e and e.get("rows") == local_rows:
            traffic = e.get("dram_bytes_per_launch")
    achieved = local_rows * bpr / (kernel_ms / 1e3) / 1e9
    return {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
            "traffic": traffic, "algorithmic_bytes": local_rows * bpr, "bytes_per_row": bpr,
            "kernel": "hq_jit_kernel (NVRTC-generated fused pipeline)", "kernel_ms": kernel_ms, "peak_source": peak_src}


# ----------------------------------------------------------------- arms
def run_reference(args):
    """--impl reference: the CPU oracle (the only reference this paper-only tier has),
    on the bench config, each step a bounded prefix sample of the fact table."""
    if int(os.environ.get("RANK", "0")) != 0:
        return
    from paper_conf_sigmod_funkebnmt18_b200.queries import QUERIES
    q = QUERIES[args.query]
    n = hqgen.table_rows(q.fact, args.sf, args.seed)
    cores = os.cpu_count() or 1
    probe = min(n, 2_000_000)
    host = gen_host(q, args.sf, args.seed, (0, probe), with_dims=True, pinned=False)
    est = oracle_call(args.query, host, cores) * n / probe  # upper bound: includes the map builds
    sample = n if est <= 10.0 else max(probe, int(n * 10.0 / est))  # whole workload, or ~10 s per step
    host = gen_host(q, args.sf, args.seed, (0, sample), with_dims=True, pinned=False)
    for _ in range(args.warmup):
        oracle_call(args.query, host, cores)
    ts = [oracle_call(args.query, host, cores) for _ in range(args.steps)]
    dt = sum(ts) / len(ts)
    v = sample / dt
    line = {"metric": METRIC, "value": v, "unit": "rows/s", "n_gpus": args.gpus, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": dt * 1e3, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "int64", "data": "synthetic (hqgen)",
            "impl": "reference",
            "config": {"workload": f"{args.query}_sf{args.sf:g}", "query": args.query, "sf": args.sf,
                       "fact_rows": n, "sample_rows_per_step": sample},
            "cpu_baseline": {"value": v, "unit": "rows/s", "cores": cores, "kind": "oracle",
                             "sample": f"first {sample} of {n} fact rows per step (full dimension tables)"},
            "e2e": {"value": v, "unit": "rows/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def run_hq(args):
    import torch
    import torch.distributed as dist
    from paper_conf_sigmod_funkebnmt18_b200.queries import QUERIES

    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    if world > 1 or os.environ.get("HQ_FORCE_DIST") == "1":
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    peak, peak_src = peaks()
    q = QUERIES[args.query]
    r = measure(args.query, args.sf, args.steps, args.warmup, args.seed, rank, world, local)
    value = r["rows"] / (r["ms"] / 1e3)
    line = None
    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": "rows/s", "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": r["ms"], "higher_is_better": True,
                "scaling": "strong", "vs_baseline": None, "dtype": "int64",
                "data": "synthetic (hqgen TPC-H/SSB-shaped generator, seed %d)" % args.seed,
                "config": {"workload": f"{args.query}_sf{args.sf:g}", "query": args.query, "sf": args.sf,
                           "fact_rows": r["rows"], "fact_bytes": r["rows"] * q.fact_bytes_per_row(),
                           "l2": "inputs larger than L2 (no flush needed)",
                           "parallelism": (f"orders/lineitem co-partitioned by order dp{world}, local builds, "
                                           "top-k rows gathered" if r["copart"] else
                                           f"fact range partition dp{world}, dimensions replicated and built on every "
                                           "rank, 1 reduce" if r["replicated"] else
                                           f"fact range partition dp{world}, dimension HTs broadcast, 1 reduce"),
                           "step": "hash builds + fused pipeline + reduce + finalize/fetch",
                           "step_mode": r["mode"] + ((" (two CUDA graphs around the partials all-reduce; every kernel "
                                                      "re-executed per step)" if (world > 1 or os.environ.get("HQ_FORCE_DIST") == "1")
                                                      else " (CUDA graph of the whole step; every kernel re-executed per step)")
                                                     if r["mode"] == "prepared" else "")},
                "step_ms_median": r["step_ms_median"], "step_ms_min": r["step_ms_min"], "eager": r["eager"],
                "roofline": roofline(q, r["local_rows"], r["kernel_ms"], peak, peak_src),
                "e2e": r.get("e2e"), "gpu_launches": r["launches"], "clocks": r["clocks"]}
        line["roofline"]["kernel_share_of_step"] = r["kernel_ms"] / r["ms"]
        if world == 1:
            line["cpu_baseline"] = cpu_baseline(args.query, r["host"], r["rows"])
            line["oaat"] = exec_timing(args.query, r["host"], local, r["ms"], "oaat")
            line["multipass"] = exec_timing(args.query, r["host"], local, r["ms"], "multipass")
        line["dram_bytes_fused_vs_oaat"] = bytes_ratio(args.query, args.sf)
    del r
    if world == 1 and not args.no_extra and args.query == DEFAULT_QUERY:
        per = []
        for qn, sf in EXTRA:
            try:
                x = measure(qn, sf, args.steps, args.warmup, args.seed, 0, 1, local, with_e2e=False)
                qq = QUERIES[qn]
                per.append({"query": qn, "sf": sf, "fact_rows": x["rows"], "value": x["rows"] / (x["ms"] / 1e3),
                            "unit": "rows/s", "ms_per_step": x["ms"], "step_mode": x["mode"],
                            "step_ms_median": x["step_ms_median"], "step_ms_min": x["step_ms_min"],
                            "eager_ms_per_step": x["eager"]["ms_per_step"],
                            "step_over_kernel": x["ms"] / x["kernel_ms"],
                            "roofline": roofline(qq, x["local_rows"], x["kernel_ms"], peak, peak_src),
                            "dram_bytes_fused_vs_oaat": bytes_ratio(qn, sf)})
                del x
            except Exception as e:  # noqa: BLE001
                per.append({"query": qn, "sf": sf, "error": str(e)[:200]})
        line["per_query"] = per
    if rank == 0:
        print(json.dumps(line), flush=True)
    if dist.is_initialized():
        dist.barrier()
        dist.destroy_process_group()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="hq", choices=["hq", "reference"])
    ap.add_argument("--query", default=DEFAULT_QUERY)
    ap.add_argument("--sf", type=float, default=DEFAULT_SF)
    ap.add_argument("--seed", type=int, default=hqgen.DEFAULT_SEED)
    ap.add_argument("--no-extra", action="store_true", help="skip the per_query configs at N=1")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    if args.impl == "reference":
        run_reference(args)
    else:
        run_hq(args)


if __name__ == "__main__":
    main()
