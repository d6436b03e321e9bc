#!/usr/bin/env python
"""Aggregate an ncu `--page source --print-source=cuda,sass --csv` export by CUDA
source line: warp-stall samples and executed instructions per line.

    ncu -i rep.ncu-rep --page source --csv --print-source=cuda,sass > x.csv
    python scripts/ncu_lines.py x.csv [top]
"""
import csv
import sys


def main():
    rows = list(csv.reader(open(sys.argv[1])))
    top = int(sys.argv[2]) if len(sys.argv) > 2 else 30
    hdr = next(r for r in rows if "Warp Stall Sampling (All Samples)" in r)
    iw = hdr.index("Warp Stall Sampling (All Samples)")
    ie = hdr.index("Instructions Executed")
    fname = "?"
    out = []
    for r in rows:
        if r and r[0] == "File Path":
            fname = r[1].split("/")[-1]
            continue
        if len(r) <= ie or not r[0].isdigit() or r[2] != "-":
            continue
        f = lambda x: float(x) if x not in ("", "-") else 0.0  # noqa: E731
        out.append((f(r[iw]), f(r[ie]), f"{fname}:{r[0]}", r[1].strip()[:80]))
    tw = sum(o[0] for o in out) or 1
    te = sum(o[1] for o in out) or 1
    print(f"total stall samples {tw:.0f}, instructions {te:.4g}")
    for w, e, loc, src in sorted(out, key=lambda o: -o[0])[:top]:
        print(f"{100 * w / tw:5.1f}% stalls {100 * e / te:5.1f}% inst  {loc:22s} {src}")


if __name__ == "__main__":
    main()
