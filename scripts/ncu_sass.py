#!/usr/bin/env python
"""Print an ncu `--page source --print-source=sass --csv` export as an annotated
SASS listing: stall samples and executed warp instructions per instruction.

    ncu -i rep.ncu-rep --page source --csv --print-source=sass > x.csv
    python scripts/ncu_sass.py x.csv [min_inst_fraction]
"""
import csv
import sys


def main():
    rows = list(csv.reader(open(sys.argv[1], errors="replace")))
    thr = float(sys.argv[2]) if len(sys.argv) > 2 else 0.0
    hdr = next(r for r in rows if "Address" in r and "Source" in r)
    ia, isrc = hdr.index("Address"), hdr.index("Source")
    iw = hdr.index("Warp Stall Sampling (All Samples)")
    ie = hdr.index("Instructions Executed")
    it = hdr.index("Thread Instructions Executed")
    body = [r for r in rows if len(r) > ie and r[ia].startswith("0x")]
    f = lambda x: float(x) if x not in ("", "-") else 0.0  # noqa: E731
    tw = sum(f(r[iw]) for r in body) or 1
    te = sum(f(r[ie]) for r in body) or 1
    print(f"total samples {tw:.0f}  warp inst {te:.4g}")
    for r in body:
        e = f(r[ie])
        if e / te < thr and f(r[iw]) / tw < thr:
            continue
        th = f(r[it]) / e if e else 0
        print(f"{r[ia][-5:]} {100 * f(r[iw]) / tw:5.1f}% {100 * e / te:5.2f}% {th:4.1f}  {r[isrc].strip()}")


if __name__ == "__main__":
    main()
