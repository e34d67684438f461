#!/usr/bin/env python
"""Segment-length sweep (BASELINE configs[3]): seg_reduce / seg_scan f32 add over
2^28 elements for seglen in workloads.C4_SEGLENS, every regime forced and auto,
both layouts.  Device time with CUDA events (median of reps, inputs 1 GiB > L2).
Writes JSON to stdout: the regime-threshold evidence table in DESIGN.md.

    python tools/seg_sweep.py [--reps 5] [--quick] > profiles/r01_seg_sweep.json
"""
import argparse
import json
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import workloads  # noqa: E402
import paper_conf_pldi_henriksenseho17_b200 as fs  # noqa: E402


def timeit(fn, reps):
    ts = []
    for _ in range(reps + 2):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        b.synchronize()
        ts.append(a.elapsed_time(b))
    return statistics.median(ts[2:])


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--quick", action="store_true")
    ap.add_argument("--auto-only", action="store_true", help="skip the forced-regime rows")
    ap.add_argument("--seglens", default="", help="comma-separated subset of C4 seglens")
    ap.add_argument("--what", default="reduce,scan", help="reduce and/or scan")
    args = ap.parse_args()
    n = 1 << (24 if args.quick else 28)
    x = workloads.device_uniform(n, 5, "cuda")
    rows = []
    seglens = [L for L in workloads.C4_SEGLENS if L <= n]
    if args.seglens:
        keep = {int(v) for v in args.seglens.split(",")}
        seglens = [L for L in seglens if L in keep]
    what = set(args.what.split(","))
    for L in seglens:
        nseg = n // L
        m = nseg * L
        xv = x[:m]
        red_bytes = 4 * m + 4 * nseg
        rec = {"seglen": L, "nseg": nseg, "auto_regime": fs.seg_regime(nseg, L)}
        for reg in ((-1,) if args.auto_only else (-1, 0, 1, 2, 3)) if "reduce" in what else ():
            if reg == 0 and L > 8192:
                continue
            if reg in (1,) and L > (1 << 22):
                continue
            fs.force_seg_regime(reg)
            try:
                out = torch.empty(nseg, device="cuda")
                ms = timeit(lambda: fs.seg_reduce(xv, nseg, L, "add", out=out), args.reps)
            finally:
                fs.force_seg_regime(-1)
            rec[f"reduce_row_r{reg}_GBs"] = round(red_bytes / ms / 1e6, 1)
        if "reduce" in what:
            out = torch.empty(nseg, device="cuda")
            ms = timeit(lambda: fs.seg_reduce(xv, nseg, L, "add", layout="col", out=out), args.reps)
            rec["reduce_col_GBs"] = round(red_bytes / ms / 1e6, 1)
        if "scan" not in what:
            rows.append(rec)
            print(json.dumps(rec), file=sys.stderr, flush=True)
            continue
        sout = torch.empty(m, device="cuda")
        ms = timeit(lambda: fs.seg_scan(xv, nseg, L, "add", out=sout), args.reps)
        rec["scan_row_GBs"] = round(8 * m / ms / 1e6, 1)
        ms = timeit(lambda: fs.seg_scan(xv, nseg, L, "add", layout="col", out=sout), args.reps)
        rec["scan_col_GBs"] = round(8 * m / ms / 1e6, 1)
        rows.append(rec)
        print(json.dumps(rec), file=sys.stderr, flush=True)
    print(json.dumps({"n": n, "dtype": "f32", "op": "add", "unit": "GB/s (algorithmic bytes / median device time)",
                      "rows": rows}))


if __name__ == "__main__":
    main()
