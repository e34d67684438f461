"""transpose_2d 2^14 x 2^14 f32 (C5) device time, 1 GB L2 flush read before each rep, median of 9."""
import os, statistics, sys, torch
sys.path.insert(0, ".")
import paper_conf_pldi_henriksenseho17_b200 as fs
x = torch.rand(1 << 14, 1 << 14, device="cuda")
y = torch.empty_like(x)
flush = torch.empty(1 << 28, device="cuda")
for shape in ((1 << 14, 1 << 14), (4096, 65536), (65536, 4096)):
    xs = x.view(-1)[: shape[0] * shape[1]].view(*shape)
    ys = y.view(-1)[: shape[0] * shape[1]].view(shape[1], shape[0])
    fs.transpose_2d(xs, out=ys)
    ts = []
    for _ in range(9):
        flush.sum()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); fs.transpose_2d(xs, out=ys); b.record(); b.synchronize(); ts.append(a.elapsed_time(b))
    ms = statistics.median(ts)
    print(os.environ.get("TAG", ""), shape, round(ms, 4), "ms", round(8 * xs.numel() / ms / 1e6 / 6546.9, 4))
assert torch.equal(ys, xs.t())
