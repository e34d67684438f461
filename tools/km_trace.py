"""Pipeline trace of fs_kmeans_step (CTA 0): per-stage clock64 stamps of the convert, decide and MMA
roles (FUTSEG_KM_TRACE=1, debug build only), summarised as steady-state intervals (dev aid)."""
import ctypes, os, sys
os.environ.setdefault("FUTSEG_KM_TRACE", "0")  # the traced CTA
import numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_pldi_henriksenseho17_b200 as fs, workloads
pts, mem = workloads.c5_kmeans_shard(0, "cuda", n=1 << int(os.environ.get("KM_LOGN", "24")))
g = torch.Generator(device="cuda").manual_seed(77)
cen = pts[torch.randint(0, pts.shape[0], (32,), device="cuda", generator=g)].clone()
for _ in range(2):
    fs.kmeans_step(pts, cen, prev=mem)
torch.cuda.synchronize()
a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
a.record(); fs.kmeans_step(pts, cen, prev=mem); b.record(); b.synchronize()
print("kernel ms", a.elapsed_time(b))
ns = (pts.shape[0] + 147) // 148 // 128 + 1
buf = np.zeros((ns, 16), np.int64)
assert fs.C.fs_debug_km_trace(buf.ctypes.data_as(ctypes.c_void_p), ns) == 0
t = buf - buf[0, 0]
names = ["cv_begin", "cv_ready", "cv_end", "dc_begin", "dc_ready", "dc_end", "mma1", "mma2"]
ok = np.all(buf[:, [0, 1, 2, 3, 4, 5, 6, 7]] != 0, axis=1)
t = t[ok][5:-5]
print("stages traced", len(t))
print("per-stage period (cycles): conv end", np.median(np.diff(t[:, 2])), " mma1", np.median(np.diff(t[:, 6])),
      " dec end", np.median(np.diff(t[:, 5])), " mma2", np.median(np.diff(t[:, 7])))
print("median durations: convert wait (ready-begin)", np.median(t[:, 1] - t[:, 0]), " convert work (end-ready)",
      np.median(t[:, 2] - t[:, 1]))
print("  conv end -> mma1 issue", np.median(t[:, 6] - t[:, 2]), "  mma1 issue -> decide ready", np.median(t[:, 4] - t[:, 6]),
      "  decide wait (ready-begin)", np.median(t[:, 4] - t[:, 3]), "  decide work (end-ready)", np.median(t[:, 5] - t[:, 4]))
print("  decide end -> mma2 issue", np.median(t[:, 7] - t[:, 5]), "  mma2(s) issue -> conv ready(s+NX)",
      [np.median(t[k:, 1] - t[:-k, 7]) for k in (2, 4)])
print("  MMA1: a1full seen -> issued", np.median(t[:, 9] - t[:, 8]), " commit+stamp", np.median(t[:, 6] - t[:, 9]),
      " conv end -> seen", np.median(t[:, 8] - t[:, 2]))
print("  MMA2: start -> issued", np.median(t[:, 11] - t[:, 10]), " decide end -> start", np.median(t[:, 10] - t[:, 5]))
for i in range(0, min(len(t), 6)):
    print(i, list(t[i] - t[i, 0]))
d = np.diff(t[:, 2])
print("convert-end period: mean %.0f median %.0f p90 %.0f p99 %.0f max %.0f" % (d.mean(), np.median(d), np.percentile(d, 90), np.percentile(d, 99), d.max()))
big = np.argsort(-d)[:12]
print("largest gaps at stage (mod 16):", [(int(i + 5), int((i + 5) % 16), int(d[i])) for i in sorted(big)])
for col, nm in ((7, "mma2"), (5, "dec end"), (6, "mma1")):
    dd = np.diff(t[:, col])
    print(f"{nm} period mean {dd.mean():.0f} median {np.median(dd):.0f}")
g0 = int(sorted(big)[len(big) // 2]) + 5
print("events per stage around a gap (cols: cv_begin cv_ready cv_end dc_begin dc_ready dc_end mma1 mma2), relative to cv_begin of the first row:")
base = t[g0 - 8, 0]
for i in range(g0 - 8, g0 + 4):
    print(i + 5, (i + 5) % 16, [int(v - base) for v in t[i, :8]])
# convert waits: raw slot (begin -> 12), TMEM slot (12 -> 13), X slot (13 -> ready)
print("convert waits (median cycles): raw", np.median(t[:, 12] - t[:, 0]), " tmem slot", np.median(t[:, 13] - t[:, 12]),
      " x slot", np.median(t[:, 1] - t[:, 13]))
