#!/usr/bin/env python
"""A/B timing of the flat scanomap and long-row seg_scan (run once per FUTSEG_SCAN_KERNEL
setting: unset = ring scan, "ws" = slab scan).  Device time, CUDA events, median of reps,
L2 flushed by reading 1 GB before each rep.  Also checks the result against torch.cumsum in
f64 on a sample (sanity only; the parity tests are tests/test_gpu_parity.py)."""
import json
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_pldi_henriksenseho17_b200 as fs  # noqa: E402

PEAK = 6546.9


def main():
    reps = 7
    n = 1 << 28
    x = torch.rand(n, device="cuda")
    y = torch.empty_like(x)
    flush = torch.empty(1 << 28, device="cuda")
    res = {"kernel": os.environ.get("FUTSEG_SCAN_KERNEL", "ring")}
    cases = [("scanomap_f32_add_2^28", lambda: fs.scanomap(x, "add", out=y))]
    for lg in (21, 23, 25, 27):
        L = 1 << lg
        cases.append((f"seg_scan_f32_add_L2^{lg}", lambda L=L: fs.seg_scan(x, n // L, L, "add", out=y)))
    xi = torch.randint(-1000, 1000, (n,), device="cuda", dtype=torch.int32)
    yi = torch.empty_like(xi)
    cases.append(("scanomap_i32_max_2^28", lambda: fs.scanomap(xi, "max", out=yi)))
    for name, fn in cases:
        fn()
        ts = []
        for _ in range(reps):
            flush.sum()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            fn()
            b.record()
            b.synchronize()
            ts.append(a.elapsed_time(b))
        ms = statistics.median(ts)
        res[name] = {"ms": round(ms, 4), "GB_s": round(8 * n / ms / 1e6, 1),
                     "frac": round(8 * n / ms / 1e6 / PEAK, 4)}
    fs.scanomap(x, "add", out=y)
    ref = torch.cumsum(x.double(), 0)
    err = ((y.double() - ref).abs() / ref.abs().clamp_min(1)).max().item()
    res["max_rel_err_vs_f64"] = err
    fs.scanomap(xi, "max", out=yi)
    res["i32_max_exact"] = bool(torch.equal(yi, torch.cummax(xi, 0).values))
    print(json.dumps(res))


if __name__ == "__main__":
    main()
