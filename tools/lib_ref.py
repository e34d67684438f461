#!/usr/bin/env python
"""Library reference points on the same B200 (context for DESIGN.md, not a bench value):
torch.cumsum (CUB DeviceScan), torch.sum (CUB reduce), x.clone() (copy) and
x.t().contiguous() on the C4/C5 shapes, device-timed with CUDA events (median)."""
import json
import statistics

import torch


def t(fn, reps=10):
    ts = []
    for _ in range(reps + 3):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        b.synchronize()
        ts.append(a.elapsed_time(b))
    return statistics.median(ts[3:])


def main():
    n = 1 << 28
    x = torch.rand(n, device="cuda")
    y = torch.empty_like(x)
    res = {}
    for name, fn, by in [("copy_f32_2^28", lambda: y.copy_(x), 8 * n),
                         ("torch.cumsum_f32_2^28", lambda: torch.cumsum(x, 0, out=y), 8 * n),
                         ("torch.sum_f32_2^28", lambda: x.sum(), 4 * n),
                         ("torch.sum_rows_L1024", lambda: x.view(-1, 1024).sum(1), 4 * n),
                         ("torch.cumsum_rows_L1024", lambda: torch.cumsum(x.view(-1, 1024), 1, out=y.view(-1, 1024)), 8 * n),
                         ("transpose_2^14_f32", lambda: y.view(1 << 14, 1 << 14).copy_(x.view(1 << 14, 1 << 14).t()), 8 * n)]:
        ms = t(fn)
        res[name] = {"ms": round(ms, 4), "GB_s": round(by / ms / 1e6, 1)}
    print(json.dumps(res, indent=1))


if __name__ == "__main__":
    main()
