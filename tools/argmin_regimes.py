import json, statistics, sys, torch
sys.path.insert(0, ".")
import paper_conf_pldi_henriksenseho17_b200 as fs
n = 1 << 27
x = torch.rand(n, device="cuda")
flush = torch.empty(1 << 28, device="cuda")
for L in (4097, 16384, 65536, 65537, 1 << 20, 1 << 22):
    nseg = n // L
    rec = {"L": L}
    for reg in (-1, 5, 9):
        fs.force_seg_regime(reg)
        try:
            fn = lambda: fs.seg_scan(x[: nseg * L], nseg, L, "argmin")
            fn(); launched = fs.last_seg_regime()
            ts = []
            for _ in range(5):
                flush.sum()
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(); fn(); b.record(); b.synchronize(); ts.append(a.elapsed_time(b))
            rec[reg] = (launched, round(16 * nseg * L / statistics.median(ts) / 1e6 / 6533.5, 3))
        finally:
            fs.force_seg_regime(-1)
    print(json.dumps(rec))
