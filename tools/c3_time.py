"""Time stream_red and kmeans_step at the kdd_cup shape (BASELINE configs[2]: n=494,019,
d=34, k=5) with CUDA events: warm (inputs in L2) and cold (L2 flushed)."""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import workloads  # noqa: E402
import paper_conf_pldi_henriksenseho17_b200 as fs  # noqa: E402

pts, mem = workloads.c3_kmeans(keys="clustered")
P, M = torch.from_numpy(pts).cuda(), torch.from_numpy(mem).cuda()
cen = P[:5].clone()
flush = torch.ones(1 << 28, dtype=torch.float32, device="cuda")
b_sr = pts.shape[0] * (34 * 4 + 4)


def t(fn, cold, reps=20):
    fn()
    ms = []
    for _ in range(reps):
        if cold:
            torch.amax(flush)  # evict by READING 1 GB: no dirty lines left to write back
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        b.synchronize()
        ms.append(a.elapsed_time(b))
    return statistics.median(ms)


for name, fn, b in (("stream_red_c3", lambda: fs.stream_red(P, M, 5), b_sr),
                    ("kmeans_step_c3", lambda: fs.kmeans_step(P, cen, prev=M), b_sr + 4 * pts.shape[0])):
    for cold in (False, True):
        ms = t(fn, cold)
        print(f"{name} {'cold' if cold else 'warm'}: {ms * 1e3:.1f} us  {b / ms / 1e6:.0f} GB/s")
