#!/usr/bin/env python
"""Per-SASS-instruction executed counts of an ncu capture, normalised per row
(thread-instructions / fact rows), for reading where a generated kernel's
issue slots go.

    python scripts/ncu_sass_rows.py rep.ncu-rep ROWS [min_per_row]
"""
import csv
import io
import subprocess
import sys


def main():
    rep, rows = sys.argv[1], float(sys.argv[2])
    lo = float(sys.argv[3]) if len(sys.argv) > 3 else 0.2
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=sass"],
                         capture_output=True, text=True, errors="replace").stdout
    r = list(csv.reader(io.StringIO(out)))
    hdr = r[1]
    ie, iw = hdr.index("Instructions Executed"), hdr.index("Warp Stall Sampling (All Samples)")
    it = hdr.index("Thread Instructions Executed")
    tot = tt = 0.0
    for x in r[2:]:
        if len(x) <= ie:
            continue
        n, t = float(x[ie] or 0), float(x[it] or 0)
        tot += n
        tt += t
        if n * 32 / rows > lo:
            print(f"{n * 32 / rows:6.2f} {x[iw]:>6} {x[1].strip()[:100]}")
    print(f"warp-inst x32 per row {tot * 32 / rows:.1f}; thread-inst per row {tt / rows:.1f}")


if __name__ == "__main__":
    main()
