"""Run one primitive on the C4/C1 size a few times (for ncu / quick timing on the GPU box).

    python tools/prof_case.py scanomap            # f32 add scan over 2^28
    python tools/prof_case.py seg_scan 1000 [col]  # f32 add seg_scan, seglen 1000, 2^28 elements
    python tools/prof_case.py seg_reduce 33 [col]
Prints the median device time and GB/s (algorithmic bytes) of 10 runs."""
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import workloads  # noqa: E402
import paper_conf_pldi_henriksenseho17_b200 as fs  # noqa: E402

what = sys.argv[1]
n = 1 << 28
x = workloads.device_uniform(n, 5, "cuda")
if what == "scanomap":
    out = torch.empty_like(x)
    fn, by = (lambda: fs.scanomap(x, "add", out=out)), 8 * n
elif what == "scanomap_mis":  # misaligned views: the look-back scan_kernel without TMA
    out = torch.empty_like(x)
    fn, by = (lambda: fs.scanomap(x[1:], "add", out=out[1:])), 8 * (n - 1)
else:
    L = int(sys.argv[2])
    layout = sys.argv[3] if len(sys.argv) > 3 else "row"
    nseg = n // L
    xv = x[: nseg * L]
    if what == "seg_scan":
        out = torch.empty_like(xv)
        fn, by = (lambda: fs.seg_scan(xv, nseg, L, "add", layout=layout, out=out)), 8 * nseg * L
    else:
        out = torch.empty(nseg, device="cuda")
        fn, by = (lambda: fs.seg_reduce(xv, nseg, L, "add", layout=layout, out=out)), 4 * nseg * (L + 1)
ts = []
for _ in range(12):
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    fn()
    b.record()
    b.synchronize()
    ts.append(a.elapsed_time(b))
ms = statistics.median(ts[2:])
print(f"{' '.join(sys.argv[1:])}: {ms * 1e3:.1f} us  {by / ms / 1e6:.1f} GB/s  frac {by / ms / 1e6 / 6546.9:.3f}  "
      f"regime {fs.last_seg_regime() if what != 'scanomap' else '-'}")
