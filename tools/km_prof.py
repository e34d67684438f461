"""Profiling driver: fused K-means step at C5 (n = 2^26, d = 34, k = 32) on cuda:0."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import workloads  # noqa: E402
import paper_conf_pldi_henriksenseho17_b200 as fs  # noqa: E402

dev = torch.device("cuda:0")
pts, mem = workloads.c5_kmeans_shard(0, dev, n=1 << int(os.environ.get("KM_LOGN", "26")))
g = torch.Generator(device=dev).manual_seed(77)
cen = pts[torch.randint(0, pts.shape[0], (32,), device=dev, generator=g)].clone()
for _ in range(3):
    out = fs.kmeans_step(pts, cen, prev=mem)
torch.cuda.synchronize()
print("delta", int(out[4].item()), "counts", out[2].tolist()[:8])
