#!/usr/bin/env python
"""Per-tile pipeline trace of scan_ring_kernel (build with -DFS_RING_TRACE, load via FUTSEG_LIB):
for the f32 add scanomap over 2^28, the distribution of load latency (issue -> landed),
queueing (landed -> scanned), look-back (scanned -> prefix), write-back and store times."""
import ctypes
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_pldi_henriksenseho17_b200 as fs  # noqa: E402

n = 1 << 28
x = torch.rand(n, device="cuda")
y = torch.empty_like(x)
flush = torch.empty(1 << 28, device="cuda")
for _ in range(3):
    flush.sum()
    fs.scanomap(x, "add", out=y)
torch.cuda.synchronize()
buf = np.zeros(65536 * 6, np.uint64)
lib = ctypes.CDLL(fs.library_path())
assert lib.fs_debug_ring_trace(buf.ctypes.data_as(ctypes.c_void_p), ctypes.c_size_t(buf.nbytes)) == 0
nt = (n + 9215) // 9216
tr = buf.reshape(-1, 6)[:nt].astype(np.int64)
t0 = tr[:, 0].min()
tr = tr - t0
res = {"tiles": int(nt), "span_us": float(tr[:, 5].max() / 1e3)}
for name, a, b in (("load", 0, 1), ("agg", 1, 2), ("lookback", 2, 3), ("writeback", 3, 4), ("store", 4, 5),
                   ("hold", 0, 5)):
    d = (tr[:, b] - tr[:, a]) / 1e3
    res[name + "_us"] = {"p10": round(float(np.percentile(d, 10)), 3), "p50": round(float(np.median(d)), 3),
                         "p90": round(float(np.percentile(d, 90)), 3), "max": round(float(d.max()), 3)}
# steady-state throughput: tiles finished per us in the middle half
fin = np.sort(tr[:, 5])
q1, q3 = fin[nt // 4], fin[3 * nt // 4]
res["mid_GBs"] = round((nt // 2) * 9216 * 8 / ((q3 - q1) / 1e9) / 1e9, 1)
res["first_landed_us"] = float(np.sort(tr[:, 1])[0] / 1e3)
print(json.dumps(res, indent=1))
