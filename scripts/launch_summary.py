#!/usr/bin/env python
"""Summarise an `ncu --metrics gpu__time_duration.sum --csv` launch list by kernel:
launches, total time, share of all launches (cold-cache, serialised times: the
kernel's SHARE of the step is what to compare with the live bench).

    python scripts/launch_summary.py gpurun_out/launches_q41.csv "title" > profiles/r01/launches_ssb_q41_sf100.md
"""
import csv
import io
import sys

SCALE = {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3}


def main():
    rows = list(csv.reader(io.StringIO(open(sys.argv[1]).read())))
    hi = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
    h = rows[hi]
    ik, iu, iv = h.index("Kernel Name"), h.index("Metric Unit"), h.index("Metric Value")
    agg = {}
    for r in rows[hi + 1:]:
        name = r[ik].replace("(anonymous namespace)::", "").replace("<unnamed>::", "").split("(")[0].replace("void ", "").strip()
        name = name.split("<")[0] if "cub::" not in name else name[:60]
        us = float(r[iv].replace(",", "")) * SCALE.get(r[iu], 1.0)
        n, t = agg.get(name, (0, 0.0))
        agg[name] = (n + 1, t + us)
    tot = sum(t for _, t in agg.values()) or 1.0
    print(sys.argv[2] if len(sys.argv) > 2 else "")
    print()
    print("| kernel | launches | total us | share |")
    print("|---|---|---|---|")
    for k, (n, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
        print(f"| {k} | {n} | {t:.1f} | {100 * t / tot:.1f}% |")


if __name__ == "__main__":
    main()
