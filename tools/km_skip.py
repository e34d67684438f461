"""K-means step timing at C5 with FUTSEG_KM_SKIP (debug switches: 1 no MMA2, 2 no MMA1, 4 no A
stores to TMEM, 8 no X stores to smem) -- where the time goes (dev aid)."""
import os, sys, torch
sys.path.insert(0, ".")
import paper_conf_pldi_henriksenseho17_b200 as fs, workloads
pts, mem = workloads.c5_kmeans_shard(0, "cuda", n=1 << 26)
g = torch.Generator(device="cuda").manual_seed(77)
cen = pts[torch.randint(0, pts.shape[0], (32,), device="cuda", generator=g)].clone()
for _ in range(2): fs.kmeans_step(pts, cen, prev=mem)
ts = []
for _ in range(5):
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(); fs.kmeans_step(pts, cen, prev=mem); b.record(); b.synchronize(); ts.append(a.elapsed_time(b))
print("skip", os.environ.get("FUTSEG_KM_SKIP", "0"), "ms", sorted(ts)[2])
