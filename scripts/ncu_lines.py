#!/usr/bin/env python
"""Aggregate an ncu source capture (--import-source on) by CUDA source line:
executed warp-instructions and stall samples per (file, line), top N.

    python scripts/ncu_lines.py report.ncu-rep [N]
"""
import csv
import io
import subprocess
import sys


def main():
    rep = sys.argv[1]
    top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
    txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    agg = {}
    src = {}
    cur_file = None
    header = None
    for row in csv.reader(io.StringIO(txt)):
        if not row:
            continue
        if row[0] == "File Path":
            cur_file = row[1].split("/")[-1]
            header = None
            continue
        if row[0] == "Line No":
            header = row
            continue
        if header is None or len(row) < len(header):
            continue
        try:
            line = int(row[0])
        except ValueError:
            continue
        iE = header.index("Instructions Executed")
        iW = header.index("Warp Stall Sampling (All Samples)")
        try:
            e = int(row[iE] or 0)
            w = int(row[iW] or 0)
        except ValueError:
            continue
        k = (cur_file, line)
        a = agg.setdefault(k, [0, 0])
        a[0] += e
        a[1] += w
        src[k] = row[1][:70]
    tot = sum(v[0] for v in agg.values()) or 1
    st = sum(v[1] for v in agg.values()) or 1
    print(f"total warp-instructions {tot}, stall samples {st}")
    for k, v in sorted(agg.items(), key=lambda kv: -kv[1][0])[:top]:
        print(f"{k[0]:>16s}:{k[1]:<5d} exec {100 * v[0] / tot:5.1f}%  stall {100 * v[1] / st:5.1f}%  {src[k]}")


if __name__ == "__main__":
    main()
