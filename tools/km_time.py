import sys, os
import numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_pldi_henriksenseho17_b200 as fs, workloads
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
print(f"mode={os.environ.get('FUTSEG_KM_DEBUG','0')} C5 kmeans_step: {ms:.3f} ms  {byt / ms / 1e6:.1f} GB/s  frac {byt / ms / 1e6 / 6546.9:.3f}", flush=True)
# SM clock / power while the step runs back to back (NVML), to see whether the tensor-core-heavy
# kernel runs under the power cap
import threading, pynvml
pynvml.nvmlInit()
h = pynvml.nvmlDeviceGetHandleByIndex(0)
samples, stop = [], threading.Event()
def samp():
    while not stop.is_set():
        samples.append((pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM), pynvml.nvmlDeviceGetPowerUsage(h) / 1000,
                        pynvml.nvmlDeviceGetCurrentClocksEventReasons(h)))
        stop.wait(0.02)
th = threading.Thread(target=samp); th.start()
for _ in range(300): f()
torch.cuda.synchronize(); stop.set(); th.join()
cl = sorted(s[0] for s in samples); pw = sorted(s[1] for s in samples)
print(f"clocks during 300 steps: median {cl[len(cl)//2]} MHz (min {cl[0]}), power median {pw[len(pw)//2]:.0f} W max {pw[-1]:.0f} W, reasons {sorted(set(s[2] for s in samples))}")
