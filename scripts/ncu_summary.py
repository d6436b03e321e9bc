#!/usr/bin/env python
"""Summarise ncu --set full captures (one kernel each) into profiles/<round>/:
a markdown table and traffic.json (DRAM bytes per launch, consumed by bench.py's
roofline.traffic).

    python scripts/ncu_summary.py --round r01 gpurun_out/q41_sf100_jit.ncu-rep:ssb_q41:100 ...
"""
import argparse
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

METRICS = {
    "gpu__time_duration.sum": "time",
    "dram__bytes_read.sum": "dram_read",
    "dram__bytes_write.sum": "dram_write",
    "dram__bytes_read.sum.pct_of_peak_sustained_elapsed": "dram_pct",
    "dram__bytes_read.sum.per_second": "dram_read_bw",
    "lts__t_sectors_srcunit_tex_op_read.sum": "l2_sectors_read",
    "lts__throughput.avg.pct_of_peak_sustained_elapsed": "l2_pct",
    "sm__warps_active.avg.pct_of_peak_sustained_active": "warps_active_pct",
    "smsp__issue_active.avg.pct_of_peak_sustained_active": "issue_active_pct",
    "smsp__inst_executed.sum": "warp_inst",
    "launch__registers_per_thread": "regs",
    "launch__shared_mem_per_block_dynamic": "dyn_smem",
    "launch__grid_size": "grid",
    "launch__block_size": "block",
}
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12, "nsecond": 1e-9, "usecond": 1e-6,
         "msecond": 1e-3, "second": 1, "ns": 1e-9, "us": 1e-6, "ms": 1e-3, "s": 1,
         "byte/s": 1, "Kbyte/s": 1e3, "Mbyte/s": 1e6, "Gbyte/s": 1e9, "Tbyte/s": 1e12, "Kbyte/block": 1e3, "byte/block": 1}


def read(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, units, vals = rows[0], rows[1], rows[2]
    res = {"kernel": vals[h.index("Kernel Name")] if "Kernel Name" in h else ""}
    for m, k in METRICS.items():
        if m not in h:
            continue
        i = h.index(m)
        try:
            v = float(vals[i].replace(",", ""))
        except ValueError:
            continue
        res[k] = v * SCALE.get(units[i], 1.0)
    return res


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--round", default="r01")
    ap.add_argument("reps", nargs="+", help="report.ncu-rep:query:sf")
    a = ap.parse_args()
    import hqgen
    from paper_conf_sigmod_funkebnmt18_b200.queries import QUERIES
    outdir = os.path.join(ROOT, "profiles", a.round)
    os.makedirs(outdir, exist_ok=True)
    tpath = os.path.join(ROOT, "profiles", "traffic.json")
    traffic = json.load(open(tpath)) if os.path.exists(tpath) else {}
    lines = ["| query | SF | rows | kernel ms | algorithmic GB | DRAM read GB | DRAM write MB | traffic/alg | "
             "achieved GB/s | DRAM read GB/s (ncu) | DRAM % of peak | L2 % | warps active % | issue active % | regs | dyn smem KB |",
             "|---|---|---|---|---|---|---|---|---|---|---|---|---|---|---|---|"]
    for spec in a.reps:
        rep, q, sf = spec.split(":")
        sf = float(sf)
        r = read(rep)
        qq = QUERIES[q]
        rows = hqgen.table_rows(qq.fact, sf)
        alg = rows * qq.fact_bytes_per_row()
        dram = r.get("dram_read", 0) + r.get("dram_write", 0)
        t = r.get("time", float("nan"))
        traffic[q] = {"sf": sf, "rows": rows, "dram_bytes_per_launch": dram, "algorithmic_bytes": alg,
                      "kernel_s_ncu": t, "report": os.path.basename(rep), "round": a.round}
        lines.append(f"| {q} | {sf:g} | {rows} | {t * 1e3:.3f} | {alg / 1e9:.3f} | {r.get('dram_read', 0) / 1e9:.3f} | "
                     f"{r.get('dram_write', 0) / 1e6:.2f} | {dram / alg:.3f} | {alg / t / 1e9:.0f} | "
                     f"{r.get('dram_read_bw', 0) / 1e9:.0f} | {r.get('dram_pct', 0):.1f} | {r.get('l2_pct', 0):.1f} | {r.get('warps_active_pct', 0):.1f} | "
                     f"{r.get('issue_active_pct', 0):.1f} | {r.get('regs', 0):.0f} | {r.get('dyn_smem', 0) / 1e3:.0f} |")
    rev = subprocess.run(["git", "-C", ROOT, "rev-parse", "--short", "HEAD"], capture_output=True, text=True).stdout.strip()
    head = (f"ncu --set full --clock-control none captures of the generated fused kernel (one launch each, "
            f"cold L2 per replay), code at {rev}. achieved = algorithmic bytes / ncu kernel time.\n\n")
    with open(os.path.join(outdir, "ncu_summary.md"), "w") as f:
        f.write(head + "\n".join(lines) + "\n")
    with open(tpath, "w") as f:
        json.dump(traffic, f, indent=1)
    print("\n".join(lines))


if __name__ == "__main__":
    main()
