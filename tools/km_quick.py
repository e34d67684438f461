"""Quick check of fs_kmeans_step: parity on small shapes, then C5 timing (dev aid)."""
import sys, time
import numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_pldi_henriksenseho17_b200 as fs, oracle, workloads

def check(n, d, k, seed=0):
    r = np.random.default_rng(seed)
    pts = r.random((n, d)).astype(np.float32)
    cen = pts[r.choice(n, k, replace=False)].copy() if n >= k else r.random((k, d)).astype(np.float32)
    prev = r.integers(0, k, n).astype(np.int32)
    m, s, c, nc, dl = fs.kmeans_step(torch.from_numpy(pts).cuda(), torch.from_numpy(cen).cuda(), prev=torch.from_numpy(prev).cuda())
    torch.cuda.synchronize()
    wm, ws, wc, wn, wd = oracle.kmeans_step(pts, cen, prev)
    gm = m.cpu().numpy()
    bad = int((gm != wm).sum())
    cerr = int(np.abs(c.cpu().numpy() - wc).max()) if k else 0
    serr = float(np.max(np.abs(s.cpu().numpy() - ws) / np.maximum(ws, 1e-30)))
    print(f"n={n} d={d} k={k}: membership mismatches {bad}, counts maxerr {cerr}, sums max rel err {serr:.2e}, delta {int(dl.cpu()[0])} vs {wd}", flush=True)
    return bad == 0 and cerr == 0 and serr < 1e-4

ok = True
for (n, d, k) in [(128, 34, 32), (1000, 34, 5), (50_021, 34, 32), (50_021, 8, 8), (50_021, 33, 17), (4097, 40, 32), (777, 1, 3), (100_003, 2, 32)]:
    ok &= check(n, d, k)
pts, mem = workloads.c5_kmeans_shard(0, "cuda")
g = torch.Generator(device="cuda").manual_seed(77)
cen = pts[torch.randint(0, pts.shape[0], (32,), device="cuda", generator=g)].clone()
out = [torch.empty(pts.shape[0], dtype=torch.int32, device="cuda"), torch.empty((32, 34), device="cuda"),
       torch.empty(32, dtype=torch.int32, device="cuda"), torch.empty((32, 34), device="cuda"), torch.empty(1, dtype=torch.int64, device="cuda")]
f = lambda: fs.kmeans_step(pts, cen, prev=mem, membership=out[0], sums=out[1], counts=out[2], new_centres=out[3], delta=out[4])
for _ in range(3): f()
torch.cuda.synchronize()
ts = []
for _ in range(10):
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(); f(); b.record(); b.synchronize(); ts.append(a.elapsed_time(b))
ms = float(np.median(ts))
byt = pts.shape[0] * (34 * 4 + 8)
print(f"C5 kmeans_step: {ms:.3f} ms  {byt / ms / 1e6:.1f} GB/s  frac {byt / ms / 1e6 / 6546.9:.3f}", flush=True)
print("ALL OK" if ok else "FAILURES")
