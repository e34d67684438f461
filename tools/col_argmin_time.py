import os, statistics, sys, torch
sys.path.insert(0, ".")
import paper_conf_pldi_henriksenseho17_b200 as fs
n = 1 << 27
x = torch.rand(n, device="cuda")
flush = torch.empty(1 << 28, device="cuda")
out = []
for L in (64, 1024, 16384, 1 << 20):
    nseg = n // L
    fn = lambda: fs.seg_reduce(x, nseg, L, "argmin", layout="col")
    fn()
    ts = []
    for _ in range(5):
        flush.sum()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); fn(); b.record(); b.synchronize(); ts.append(a.elapsed_time(b))
    out.append((L, round(4 * n / statistics.median(ts) / 1e6 / 6533.5, 3)))
print(os.environ.get("TAG", ""), out)
