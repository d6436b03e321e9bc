#!/usr/bin/env python
"""SASS evidence from ncu reports: the Blackwell data-movement / synchronisation
instructions of each captured fused kernel (1-D TMA bulk copies `UBLKCP`, mbarrier
`SYNCS.*`, warp votes, shared / global loads) with their executed warp-instruction
counts, plus the per-row instruction count -- markdown for profiles/<round>/.

    python scripts/sass_excerpt.py gpurun_out/r02ev/ssb_q41_sf100_jit.ncu-rep:600011291 ... > profiles/r02/sass_excerpt.md
"""
import csv
import io
import subprocess
import sys

KEYS = ("UBLKCP", "SYNCS", "UTMA", "LDGSTS", "ATOMS", "REDG", "RED.", "VOTE", "MATCH", "LDS", "LDG", "BAR")


def sass(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr = next(r for r in rows if "Address" in r and "Source" in r)
    ia, isrc, ie = hdr.index("Address"), hdr.index("Source"), hdr.index("Instructions Executed")
    return [(r[ia], r[isrc].strip(), float(r[ie] or 0)) for r in rows if len(r) > ie and r[ia].startswith("0x")]


def main():
    print("# SASS excerpt of the generated fused kernels (ncu --set full captures, `--page source --print-source sass`)\n")
    print("Executed warp instructions per opcode family; `UBLKCP` = `cp.async.bulk` (1-D TMA) issued by the producer "
          "lane, `SYNCS.*` = mbarrier arrive / try-wait (hardware transaction barriers), `ATOMS` = shared-memory atomics "
          "(pre-aggregation), `REDG`/`RED` = fire-and-forget global reductions (global propagation).\n")
    for arg in sys.argv[1:]:
        rep, _, rows = arg.partition(":")
        ins = sass(rep)
        tot = sum(e for _, _, e in ins)
        print(f"## {rep.split('/')[-1]}\n")
        print(f"{len(ins)} SASS instructions, {tot:.4g} warp instructions executed"
              + (f", {tot / float(rows):.2f} per fact row" if rows else "") + "\n")
        fam = {}
        for _, src, e in ins:
            op = src.split()[0] if not src.startswith("@") else src.split()[1]
            for k in KEYS:
                if op.startswith(k):
                    fam[op] = fam.get(op, 0) + e
        print("| opcode | warp instructions executed |\n|---|---|")
        for op, e in sorted(fam.items(), key=lambda x: -x[1]):
            print(f"| `{op}` | {e:.4g} |")
        print("\nTMA / mbarrier instructions as compiled:\n\n```")
        for a, src, e in ins:
            if "UBLKCP" in src or "SYNCS" in src:
                print(f"{a[-5:]}  {e:>12.0f}  {src}")
        print("```\n")


if __name__ == "__main__":
    main()
