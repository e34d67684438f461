#!/usr/bin/env python
"""Warp-stall samples per CUDA source line of an ncu --set full report (needs -lineinfo).

    python tools/ncu_lines.py gpurun_out/<name>.ncu-rep [n_lines]
"""
import csv
import io
import subprocess
import sys


def main(rep, nlines=30):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass,cuda"],
                         capture_output=True, text=True).stdout
    cur, hdr, ci, rows = None, None, None, []
    for r in csv.reader(io.StringIO(out)):
        if not r:
            continue
        if r[0] == "File Path":
            cur = r[1]
            continue
        if r[0] == "Line No":
            hdr = r
            ci = hdr.index("Warp Stall Sampling (All Samples)")
            continue
        if hdr and cur and r[0].isdigit() and len(r) == len(hdr):
            try:
                v = float(r[ci])
            except ValueError:
                v = 0.0
            rows.append((v, cur.split("/")[-1], int(r[0]), r[1].strip()[:100]))
    rows.sort(reverse=True)
    tot = sum(r[0] for r in rows) or 1.0
    for v, f, ln, src in rows[:nlines]:
        print(f"{100 * v / tot:5.1f}%  {f}:{ln}  {src}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 30)
