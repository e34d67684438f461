"""C2 NN argmin redomap latency: cold (1 GB read between reps evicts the 6.8 MB) and warm,
device time with CUDA events, median of 20 (dev aid for the NN kernel's launch shape)."""
import os, statistics, sys, torch
sys.path.insert(0, ".")
import numpy as np
import paper_conf_pldi_henriksenseho17_b200 as fs, workloads
lat, lng, q = workloads.c2_nn()
lat, lng = torch.from_numpy(lat).cuda(), torch.from_numpy(lng).cuda()
flush = torch.empty(1 << 28, device="cuda")
for cold in (True, False):
    ts = []
    for _ in range(23):
        if cold:
            flush.sum()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); fs.redomap(lat, "argmin", map="nn_dist", lng=lng, query=q); b.record(); b.synchronize()
        ts.append(a.elapsed_time(b) * 1e3)
    print(os.environ.get("TAG", ""), "cold" if cold else "warm", round(statistics.median(ts[3:]), 2), "us")
