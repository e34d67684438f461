"""Repeat the C5 k-means step (and a kdd-shaped one) many times and check every result against
the first (membership bit-exact, counts exact): a race in the pipeline shows up as a launch
failure or a changed result (dev aid; compute-sanitizer is closed on this pool)."""
import sys, torch
sys.path.insert(0, ".")
import paper_conf_pldi_henriksenseho17_b200 as fs, workloads
for n, k in ((1 << 26, 32), (494_019, 5), (3_000_017, 32)):
    pts, mem = workloads.c5_kmeans_shard(0, "cuda", n=n)
    g = torch.Generator(device="cuda").manual_seed(77)
    cen = pts[torch.randint(0, pts.shape[0], (k,), device="cuda", generator=g)].clone()
    m0, s0, c0, _, d0 = fs.kmeans_step(pts, cen, prev=mem)
    m0, c0 = m0.clone(), c0.clone()
    bad = 0
    for it in range(40):
        m, s, c, _, d = fs.kmeans_step(pts, cen, prev=mem)
        bad += int(not torch.equal(m, m0)) + int(not torch.equal(c, c0))
    torch.cuda.synchronize()
    print("n", n, "k", k, "mismatches", bad)
