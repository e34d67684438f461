#!/usr/bin/env python
"""Fraction of the HBM peak of the flat and segmented primitives for every dtype and op (2^27
elements, 1 GB L2 flush read before each rep, median of 5): spots a dtype / op falling off a cliff."""
import json, os, statistics, sys, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_pldi_henriksenseho17_b200 as fs
PEAK = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "MEASURED_PEAKS.json")))["hbm_gbs"]
n = 1 << 27
flush = torch.empty(1 << 28, device="cuda")


def t(fn):
    fn()
    ts = []
    for _ in range(5):
        flush.sum()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); fn(); b.record(); b.synchronize(); ts.append(a.elapsed_time(b))
    return statistics.median(ts)


res = {}
for dt in (torch.int32, torch.int64, torch.float32):
    x = (torch.rand(n, device="cuda") * 1000).to(dt)
    es = x.element_size()
    for op in ("add", "min", "argmin"):
        ib = 8 if op == "argmin" else 0
        cases = {
            "redomap": (lambda: fs.redomap(x, op), es * n),
            "scanomap": (lambda: fs.scanomap(x, op), (2 * es + ib) * n),
            "seg_reduce_L1024": (lambda: fs.seg_reduce(x, n // 1024, 1024, op), es * n),
            "seg_scan_L1024": (lambda: fs.seg_scan(x, n // 1024, 1024, op), (2 * es + ib) * n),
            "seg_scan_L65537": (lambda: fs.seg_scan(x[: (n // 65537) * 65537], n // 65537, 65537, op),
                                (2 * es + ib) * (n // 65537) * 65537),
            "seg_reduce_col_L1024": (lambda: fs.seg_reduce(x, n // 1024, 1024, op, layout="col"), es * n),
        }
        for name, (fn, by) in cases.items():
            ms = t(fn)
            res[f"{name}/{str(dt).split('.')[-1]}/{op}"] = round(by / ms / 1e6 / PEAK, 3)
print(json.dumps(res, indent=1))
