#!/usr/bin/env python
"""DRAM bytes of the fused plan vs the multi-pass and the operator-at-a-time
plans of the same query (the BASELINE.json metric's second half; SURVEY.md
§8(d.3); the paper's three execution models, e.g. 8.4 -> 4.4 -> 1.8 GB for SSB
Q3.1).

Runs every query once per mode under
  ncu --cache-control all --clock-control none --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum
and sums the metrics over all kernels of the execution (as the paper summed
per-kernel nvprof metrics), split into the fact pipeline and the
rest (hash builds, finalize).  Writes profiles/<round>/bytes_ratio.{json,md}.

    python scripts/bytes_ratio.py --sf 10                         # every query at SF 10
    python scripts/bytes_ratio.py --queries ssb_q41:100,ssb_q31:30  # per-query scale factors

At SF >= 30 every intermediate of the operator-at-a-time and multi-pass plans is many
times the 126 MB L2, so the per-kernel counts charge (nearly) all of their write-backs;
at SF 10 part of them stays in L2 between kernels and the ratios are lower bounds.
"""
import argparse
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
QUERIES = ["tpch_q6", "tpch_q1", "ssb_q11", "ssb_q12", "ssb_q13", "ssb_q31", "ssb_q31_mat", "ssb_q41", "tpch_q3"]
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-9, "us": 1e-6, "ms": 1e-3, "s": 1,
         "nsecond": 1e-9, "usecond": 1e-6, "msecond": 1e-3}
PIPELINE = ("hq_jit_kernel", "hq_fused_pipeline_kernel", "hq_oaat", "cub::", "DeviceScan", "mp_")
MODES = ("fused", "multipass", "oaat")


def run(q, sf, mode):
    log = os.path.join(ROOT, "gpurun_out", f"ncu_{q}_{mode}.csv")
    cmd = ["ncu", "--cache-control", "all", "--clock-control", "none", "--metrics",
           "dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum", "--csv", "--log-file", log,
           sys.executable, os.path.join(ROOT, "scripts", "profile_query.py"), "--query", q, "--sf", str(sf),
           "--reps", "1", "--exec", mode]
    subprocess.run(cmd, capture_output=True, text=True, timeout=1800)
    rows = list(csv.reader(io.StringIO(open(log).read())))
    hi = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
    h = rows[hi]
    ik, im, iu, iv = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Unit"), h.index("Metric Value")
    tot = {"pipeline": {}, "other": {}}
    kernels = set()
    for r in rows[hi + 1:]:
        part = "pipeline" if any(p in r[ik] for p in PIPELINE) else "other"
        v = float(r[iv].replace(",", "")) * SCALE.get(r[iu], 1.0)
        tot[part][r[im]] = tot[part].get(r[im], 0.0) + v
        kernels.add((part, r[ik].split("(")[0][:50]))
    return tot, sorted(kernels)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--sf", type=float, default=10)
    ap.add_argument("--round", default="r01")
    ap.add_argument("--queries", default=",".join(QUERIES))
    a = ap.parse_args()
    out = {}
    sfs = {}
    for qs in a.queries.split(","):
        q, _, qsf = qs.partition(":")
        sf = float(qsf) if qsf else a.sf
        sfs[q] = sf
        out[q] = {"sf": sf}
        for mode in MODES:
            tot, kernels = run(q, sf, mode)
            out[q][mode] = {part: {"dram_bytes": d.get("dram__bytes_read.sum", 0) + d.get("dram__bytes_write.sum", 0),
                                   "time_s": d.get("gpu__time_duration.sum", 0)} for part, d in tot.items()}
            out[q][mode]["kernels"] = kernels
        print(q, sf, json.dumps({m: {p: out[q][m][p] for p in ("pipeline", "other")} for m in MODES}), flush=True)
    d = os.path.join(ROOT, "gpurun_out")  # copied to profiles/<round>/ after the run
    os.makedirs(d, exist_ok=True)
    tag = f"sf{a.sf:g}" if len(set(sfs.values())) <= 1 and a.sf in sfs.values() else "bench_sfs"
    with open(os.path.join(d, f"bytes_ratio_{tag}.json"), "w") as f:
        json.dump({"sf": a.sf, "sfs": sfs, "cache_control": "all", "queries": out,
                   "paper": {"volume_reduction_up_to": 7.5, "kernel_time_reduction_up_to": 9.5, "gpu": "GTX 970",
                             "cite": "PAPER.md P:40-42 (abstract), GTX970 setup P:1369-1379"}}, f, indent=1)
    lines = [f"DRAM bytes (ncu dram__bytes_read.sum + dram__bytes_write.sum, --cache-control all) summed over all kernels "
             f"of one query execution at the SF of each row; 'pipeline' = the fact-table pipeline kernels (fused: one generated "
             "kernel; multi-pass: generated count + write kernels, CUB scan / reduce / sort, reduce-by-key scatter; "
             "op-at-a-time: filter/probe/compute/scan/compact/gather/agg kernels), 'all' adds hash builds and finalize. "
             "Times are ncu kernel durations (cold caches, serialised), summed.",
             "The paper's reductions for context: up to 7.5x memory volume and 9.5x kernel time, fused vs "
             "operator-at-a-time, on a GTX 970 (PAPER.md P:40-42).",
             "", "| query | SF | fused GB | multi-pass GB | OAAT GB | MP/fused bytes | OAAT/fused bytes | OAAT/fused bytes (all) "
             "| fused ms | multi-pass ms | OAAT ms | MP/fused time | OAAT/fused time |",
             "|---|---|---|---|---|---|---|---|---|---|---|---|---|"]
    for q, m in out.items():
        fp, mp, op = m["fused"]["pipeline"], m["multipass"]["pipeline"], m["oaat"]["pipeline"]
        fa = fp["dram_bytes"] + m["fused"]["other"]["dram_bytes"]
        oa = op["dram_bytes"] + m["oaat"]["other"]["dram_bytes"]
        fb = max(fp["dram_bytes"], 1)
        ft = max(fp["time_s"], 1e-12)
        lines.append(f"| {q} | {m['sf']:g} | {fp['dram_bytes'] / 1e9:.3f} | {mp['dram_bytes'] / 1e9:.3f} | {op['dram_bytes'] / 1e9:.3f} | "
                     f"{mp['dram_bytes'] / fb:.2f}x | {op['dram_bytes'] / fb:.2f}x | {oa / max(fa, 1):.2f}x | "
                     f"{fp['time_s'] * 1e3:.3f} | {mp['time_s'] * 1e3:.3f} | {op['time_s'] * 1e3:.3f} | "
                     f"{mp['time_s'] / ft:.2f}x | {op['time_s'] / ft:.2f}x |")
    with open(os.path.join(d, f"bytes_ratio_{tag}.md"), "w") as f:
        f.write("\n".join(lines) + "\n")
    print("\n".join(lines))


if __name__ == "__main__":
    main()
