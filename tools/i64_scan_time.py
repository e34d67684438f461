import statistics, sys, torch
sys.path.insert(0, ".")
import paper_conf_pldi_henriksenseho17_b200 as fs
n = 1 << 27
x = torch.randint(-1000, 1000, (n,), device="cuda", dtype=torch.int64)
y = torch.empty_like(x)
flush = torch.empty(1 << 28, device="cuda")
fs.scanomap(x, "add", out=y)
ts = []
for _ in range(7):
    flush.sum()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(); fs.scanomap(x, "add", out=y); b.record(); b.synchronize(); ts.append(a.elapsed_time(b))
ms = statistics.median(ts)
print("i64 scanomap 2^27:", round(ms, 4), "ms", round(16 * n / ms / 1e6 / 6533.5, 4))
