"""Small invocations of every libfutseg primitive for compute-sanitizer (tools/sanitize.sh)."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import workloads  # noqa: E402
import paper_conf_pldi_henriksenseho17_b200 as fs  # noqa: E402


def cu(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


x = cu(workloads.mixed(300_001, 1, np.float32))
xi = cu(workloads.mixed(300_001, 2, np.int64))
for op in ("add", "min", "argmin"):
    fs.redomap(x, op)
    fs.redomap(xi, op)
    fs.scanomap(x, op)
    fs.scanomap(xi[1:], op)
lat, lng, q = workloads.c2_nn(base=20_000, reps=2)
fs.redomap(cu(lat), "argmin", map="nn_dist", lng=cu(lng), query=q)
fs.scanomap(cu(lat), "min", map="nn_dist", lng=cu(lng), query=q)
fs.redomap(cu(workloads.mixed((5000, 34), 3, np.float32)), "vadd")
for nseg, L in ((10_000, 1), (7_001, 3), (4096, 32), (1000, 33), (300, 1000), (20, 10_000), (2, 150_000)):
    m = x[: nseg * L]
    for reg in (-1, 0, 1, 2, 3):
        fs.force_seg_regime(reg)
        fs.seg_reduce(m, nseg, L, "add")
        fs.seg_reduce(m, nseg, L, "argmin")
    fs.force_seg_regime(-1)
    fs.seg_reduce(m, nseg, L, "max", layout="col")
    fs.seg_scan(m, nseg, L, "add")
    fs.seg_scan(m, nseg, L, "argmin", layout="col")
pts, mem = workloads.c3_kmeans(n=30_000, d=34, k=5)
fs.stream_red(cu(pts), cu(mem), 5)
pts, mem = workloads.c3_kmeans(n=30_000, d=34, k=32)
fs.stream_red(cu(pts), cu(mem), 32)
fs.stream_red(cu(workloads.mixed((3000, 100), 4, np.float32)), cu(workloads.ints(3000, 5, 0, 70)), 70)
fs.transpose_2d(cu(workloads.mixed((333, 517), 6, np.float32)))
fs.transpose_2d(cu(workloads.mixed((256, 128), 7, np.int64)))
# seg_scan KS0 (power-of-two rows: one warp, several warps, ragged tail)
for nseg, L in ((1001, 2), (999, 16), (300, 128), (101, 512), (37, 1024)):
    fs.seg_scan(x[: nseg * L], nseg, L, "add")
    fs.seg_scan(x[: nseg * L], nseg, L, "argmin")
    fs.seg_scan(xi[: nseg * L], nseg, L, "min")
# NEXT-2 nn_knn (cooperative launch, grid barrier) and NEXT-1 kmeans_step
lat2, lng2, q2 = workloads.c2_nn(base=30_000, reps=3)
fs.nn_knn(cu(lat2), cu(lng2), q2, 100)
fs.nn_knn(cu(lat2[:777]), cu(lng2[:777]), q2, 1000)
pts, _ = workloads.c3_kmeans(n=20_011, d=34, k=32)
fs.kmeans_step(cu(pts), cu(pts[:32].copy()), prev=cu(workloads.ints(20_011, 3, 0, 32)))
pts, _ = workloads.c3_kmeans(n=5_003, d=7, k=5)
fs.kmeans_step(cu(pts), cu(pts[:5].copy()))
# seg_scan KS1 (short non-power-of-two rows), scan_reduce, seg_map_reduce (all regimes)
for nseg, L in ((1001, 3), (257, 7), (300, 31)):
    fs.seg_scan(x[: nseg * L], nseg, L, "add")
    fs.seg_scan(xi[: nseg * L], nseg, L, "max")
for red in ("add", "max", "min"):
    fs.scan_reduce(x[:200_001], red)
    fs.scan_reduce(xi[:77_777], red)
for nseg, L in ((1000, 8), (300, 33), (5, 20_000)):
    fs.seg_map_reduce(x[: nseg * L], nseg, L, 1.0, "add")
    fs.seg_map_reduce(xi[: nseg * L], nseg, L, 2, "argmin")
xb = cu(workloads.mixed(600 * 8192, 8, np.float32))  # CTA-per-row regime (>= 4 rows per SM)
fs.seg_map_reduce(xb, 600, 8192, 1.0, "max")
# seg_scan KS2 (CTA per row, running carry): whole + partial chunks, argmin, misaligned view
xk = cu(workloads.mixed(600 * 12_289 + 1, 9, np.float32))
fs.seg_scan(xk[: 600 * 12_289], 600, 12_289, "add")
fs.seg_scan(xk[1:], 600, 12_289, "argmin")
# round 2: every seg_scan regime of the plan (fs::seg_scan_plan), forced where applicable --
# KS0-BIG (power-of-two rows of 2-8 CTA steps), KS3 (several rows per CTA, one row per CTA,
# 8-byte, misaligned views), KS2, the flat slab scan per row, the look-back scan
xr = cu(workloads.mixed(150 * 12_288 + 8, 10, np.float32))
xri = cu(workloads.mixed(150 * 12_288 + 8, 10, np.int64))
for reg in (5, 7, 8, 9, 10, 11, 12):
    fs.force_seg_regime(reg)
    for nseg, L in ((64, 2048), (17, 8192), (300, 33), (7, 1000), (3, 16_384), (150, 12_288), (777, 3)):
        fs.seg_scan(xr[: nseg * L], nseg, L, "add")
        fs.seg_scan(xri[: nseg * L], nseg, L, "min")
    fs.force_seg_regime(-1)
for nseg, L, off in ((64, 1000, 1), (7, 4097, 1), (300, 33, 3)):
    fs.seg_scan(xr[off: off + nseg * L], nseg, L, "max")   # KS3 on misaligned views
    fs.seg_scan(xri[off: off + nseg * L], nseg, L, "add")
xl = cu(workloads.mixed(2 * (1 << 20), 11, np.float32))
fs.force_seg_regime(12)
fs.seg_scan(xl, 2, 1 << 20, "add")  # the flat per-row slab scan
fs.force_seg_regime(-1)
# the tcgen05 k-means step (TMA ring, TMEM A, both MMAs, d = 34 specialisation and run-time d,
# a partial last stage) and the multi-GPU exchange kernels
pts, _ = workloads.c3_kmeans(n=40_011, d=34, k=32)
fs.kmeans_step(cu(pts), cu(pts[:32].copy()), prev=cu(workloads.ints(40_011, 3, 0, 32)))
pts, _ = workloads.c3_kmeans(n=9_999, d=40, k=17)
fs.kmeans_step(cu(pts), cu(pts[:17].copy()))
v = cu(workloads.mixed(9, 12, np.float32))
i = cu(np.arange(9, dtype=np.int64))
k = fs.argmin_pack(v, i)
fs.argmin_unpack(k[:1], torch.float32)
k8 = fs.argmin_pack(cu(workloads.mixed(9, 13, np.int64)), i)
fs.argmin_unpack(k8, torch.int64, P=9)
pk = fs.partials_pack(cu(workloads.mixed((5, 7), 14, np.float32)), cu(np.arange(5, dtype=np.int32)))
fs.partials_unpack(pk, torch.empty((5, 7), device="cuda"), torch.empty(5, dtype=torch.int32, device="cuda"))
fs.copy_2d(x[1:], 33, 17, 41, torch.empty(33 * 19 + 1, device="cuda")[1:], 19)
# seg_reduce: odd short rows staged by TMA (several tiles + ragged tail), column layout short
# rows (m <= 8, >= 148*8*256 columns), the flat period stream (w <= 1024) and two-level split combine
xs = cu(workloads.mixed(2_200_000, 15, np.float32))
xs8 = cu(workloads.mixed(2_200_000, 16, np.int64))
for nseg, L in ((7697, 3), (1001, 33), (777, 63), (2049, 31)):
    fs.seg_reduce(xs[: nseg * L], nseg, L, "add")
    fs.seg_reduce(xs8[: nseg * L], nseg, L, "argmin")
fs.seg_reduce(xs[: 310_001 * 7], 310_001, 7, "argmin", layout="col")
fs.seg_reduce(xs[1: 1 + 310_001 * 3], 310_001, 3, "add", layout="col")
for nseg, L in ((268, 5_003), (3, 9_001), (512, 4_099), (5, 200_003), (64, 30_001)):
    fs.seg_reduce(xs[: nseg * L], nseg, L, "add", layout="col")
    fs.seg_reduce(xs8[: nseg * L], nseg, L, "argmin", layout="col")
    fs.seg_reduce(xs[1: 1 + nseg * L], nseg, L, "max", layout="col")
# seg_scan column layout: the one-pass look-back kernel (vector / scalar columns, 8-byte, argmin)
# and the short-rows kernel
for nseg, L in ((512, 2_049), (5, 30_001), (2, 100_003), (4096, 65)):
    fs.seg_scan(xs[: nseg * L], nseg, L, "add", layout="col")
    fs.seg_scan(xs8[: nseg * L], nseg, L, "argmin", layout="col")
    fs.seg_scan(xs[1: 1 + nseg * L], nseg, L, "max", layout="col")
fs.seg_scan(xs[1: 1 + 303_105 * 3], 303_105, 3, "add", layout="col")
fs.seg_scan(xs[: 303_105 * 7], 303_105, 7, "argmin", layout="col")
# seg_scan KS3 through the TMA ring (short and long rows, 8-byte, leftover rows)
for nseg, L in ((30_001, 3), (9_001, 7), (1_001, 33), (77, 1000), (50, 4097)):
    fs.seg_scan(xs[: nseg * L], nseg, L, "add")
    fs.seg_scan(xs8[: nseg * L], nseg, L, "max")
# seg_scan KS2 through the TMA ring (rows of several tiles, partial last tile)
fs.seg_scan(xs[: 149 * 12_292], 149, 12_292, "add")
fs.seg_scan(xs8[: 150 * 12_292], 150, 12_292, "min")
torch.cuda.synchronize()
print("sanitize cases done")
# round 2: the ring scan (scanomap and the aligned segmented look-back): more tiles than CTAs
# (every ring slot reused, both consumer groups, end markers), a ragged sub-vector tail, 8-byte
# tiles, a carry-in, segment starts inside tiles (masked aggregate vectors)
xg = cu(workloads.mixed(2_000_003, 17, np.float32))
xg8 = cu(workloads.mixed(1_000_001, 18, np.int64))
fs.scanomap(xg, "add")
fs.scanomap(xg8, "max")
fs.scanomap(xg[:777_777], "add", carry=xg[:1].clone())
fs.force_seg_regime(5)
fs.seg_scan(xg[: 100 * 10_001], 100, 10_001, "add")
fs.seg_scan(xg8[: 300 * 3001], 300, 3001, "min")
fs.force_seg_regime(-1)
fs.seg_scan(xg[: 50 * 40_001], 50, 40_001, "max")  # the plan's ring choice (L > 4096, L % 4 != 0)
torch.cuda.synchronize()
print("ring cases ok")
