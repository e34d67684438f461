"""GPU parity, edge cases of the method (round 2): integer wrap-around on every primitive
that adds integers, every segmented regime forced and the regime the dispatcher reports
checked against the one it launched, reading R18's fma rounding on the tensor-core K-means
path, and the full-size C5 legs (k-means step, transpose) against the oracle.

Bar (BASELINE.json north_star): integers, indices, argmin, min/max bit-exact; f32 add within
1e-4 of the f64 oracle relative to the same sum over |x| (R2).  Reading R1
(DESIGN.md): integer ADD wraps modulo 2^32 / 2^64 (PAPER.md L121-133 define reduce and scan
with an associative operator and its neutral element; two's-complement wrap is the only
reading under which integer results do not depend on the reduction order).
"""
import concurrent.futures as cf
import json
import os

import numpy as np
import pytest
import torch

import oracle
import workloads

pytestmark = pytest.mark.gpu

INTS = [np.int32, np.int64]


@pytest.fixture(scope="module")
def fs():
    import paper_conf_pldi_henriksenseho17_b200 as m
    return m


def cu(a, offset=0):
    a = np.ascontiguousarray(a)
    if offset:
        t = torch.from_numpy(np.concatenate([np.zeros(offset, a.dtype), a.reshape(-1)])).cuda()
        return t[offset:].view(a.shape) if a.ndim > 1 else t[offset:]
    return torch.from_numpy(a).cuda()


def host(t):
    return t.detach().cpu().numpy()


def eq(got, want, what):
    if isinstance(want, tuple):
        np.testing.assert_array_equal(host(got[1]), want[1], err_msg=f"{what} index")
        np.testing.assert_array_equal(host(got[0]), want[0], err_msg=f"{what} value")
    else:
        np.testing.assert_array_equal(host(got), want, err_msg=what)


def wrap_input(n, seed, dt, op):
    """Full-range integers for ADD (sums wrap many times); full range too for MIN/MAX/ARGMIN
    (extremes INT_MIN/INT_MAX appear), with planted argmin ties."""
    x = workloads.full_range(n, seed, dt)
    if op == "argmin" and n > 10:
        x[n // 5] = x[n - 2] = x.min()
    return x


# ------------------------------------------------------------------ R1: wrap-around everywhere
@pytest.mark.parametrize("dt", INTS)
@pytest.mark.parametrize("op", ["add", "min", "max", "argmin"])
@pytest.mark.parametrize("n,off", [(1, 0), (1000, 1), (65_537, 0), ((1 << 22) + 3, 0), (3_000_017, 1)])
def test_redomap_wrap(fs, dt, op, n, off):
    x = wrap_input(n, n % 101, dt, op)
    eq(fs.redomap(cu(x, off), op), oracle.reduce(x, op), f"redomap {op} n={n}")


@pytest.mark.parametrize("dt", INTS)
@pytest.mark.parametrize("op", ["add", "max", "argmin"])
@pytest.mark.parametrize("n,off", [(7, 0), (4096, 1), (1_000_003, 0), (5_000_011, 2)])
def test_scanomap_wrap(fs, dt, op, n, off):
    x = wrap_input(n, n % 97, dt, op)
    eq(fs.scanomap(cu(x, off), op), oracle.scan(x, op), f"scanomap {op} n={n}")


@pytest.mark.parametrize("dt", INTS)
def test_scanomap_wrap_carry(fs, dt):
    """F5 (L1071-1074): scan of the second half continued from the first half's total."""
    x = workloads.full_range(2_000_001, 3, dt)
    h = 777_777
    a = fs.scanomap(cu(x[:h]), "add")
    b = fs.scanomap(cu(x[h:]), "add", carry=a[-1:].clone())
    np.testing.assert_array_equal(np.concatenate([host(a), host(b)]), oracle.scan(x, "add"))


SEG_SHAPES = [(1000, 1), (777, 3), (300, 16), (200, 33), (64, 64), (50, 1000), (9, 4097), (3, 65_537),
              (2, 300_001)]


@pytest.mark.parametrize("dt", INTS)
@pytest.mark.parametrize("regime", [-1, 0, 1, 2, 3])
def test_seg_reduce_wrap_every_regime(fs, dt, regime):
    fs.force_seg_regime(regime)
    try:
        for nseg, L in SEG_SHAPES:
            for op in ("add", "argmin"):
                x = wrap_input(nseg * L, nseg + L, dt, op)
                eq(fs.seg_reduce(cu(x), nseg, L, op), oracle.seg_reduce(x, nseg, L, op),
                   f"seg_reduce {op} {nseg}x{L} regime {regime}")
    finally:
        fs.force_seg_regime(-1)


@pytest.mark.parametrize("dt", INTS)
@pytest.mark.parametrize("nseg,L", [(7, 3), (1000, 50), (5, 20_000), (100_000, 3), (4096, 64)])
def test_seg_reduce_col_wrap(fs, dt, nseg, L):
    x = workloads.full_range(nseg * L, 17, dt)
    eq(fs.seg_reduce(cu(x), nseg, L, "add", layout="col"), oracle.seg_reduce(x, nseg, L, "add", "col"),
       f"col {nseg}x{L}")


@pytest.mark.parametrize("dt", INTS)
@pytest.mark.parametrize("k", [1, 5, 34, 1024, 4096])
def test_vadd_wrap(fs, dt, k):
    n = 20_011 if k <= 34 else 3001
    x = workloads.full_range((n, k), k, dt)
    eq(fs.redomap(cu(x), "vadd"), oracle.vreduce(x, "add"), f"vadd k={k}")


@pytest.mark.parametrize("dt", INTS)
@pytest.mark.parametrize("k,w", [(5, 34), (32, 34), (32, 37), (7, 200), (300, 100)])
def test_stream_red_wrap(fs, dt, k, w):
    n = 30_011
    vals = workloads.full_range((n, w), k + w, dt)
    mem = workloads.ints(n, w, 0, k)
    sums, counts = fs.stream_red(cu(vals), cu(mem), k)
    ws, wc = oracle.stream_red(vals, mem, k)
    np.testing.assert_array_equal(host(counts), wc)
    np.testing.assert_array_equal(host(sums), ws)


@pytest.mark.parametrize("dt", INTS)
@pytest.mark.parametrize("op", ["add", "min", "max", "argmin", "vadd"])
def test_combine_int(fs, dt, op):
    """fs_combine on integer partials (the cross-GPU combine, A7): full range, ties."""
    if op == "vadd":
        parts = workloads.full_range((37, 9), 4, dt)
        eq(fs.combine(cu(parts), "vadd"), oracle.vreduce(parts, "add"), "combine vadd")
        return
    parts = workloads.full_range(37, 5, dt)
    parts[3] = parts[30] = parts.min()
    pidx = np.arange(37, dtype=np.int64) * 1000 + 5
    got = fs.combine(cu(parts), op, part_idx=cu(pidx) if op == "argmin" else None)
    want = oracle.reduce(parts, op)
    if op == "argmin":
        assert int(host(got[1])) == pidx[want[1]] and int(host(got[0])) == int(want[0])
    else:
        assert int(host(got)) == int(want)


@pytest.mark.parametrize("dt", INTS)
def test_scan_family_wrap_misc(fs, dt):
    """seg_map_reduce's map and reduce, and the KS regimes, on full-range integers."""
    x = workloads.full_range(333 * 1001, 8, dt)
    mp, rs = fs.seg_map_reduce(cu(x), 333, 1001, -(1 << 30) + 7, "add")
    wm, wr = oracle.seg_map_reduce(x, 333, 1001, -(1 << 30) + 7, "add")
    np.testing.assert_array_equal(host(mp).reshape(-1), wm)
    np.testing.assert_array_equal(host(rs), wr)


# ------------------------------------------------------------------ regimes: forced and reported
SCAN_REGIMES = [5, 7, 8, 9, 10, 11, 12]
SCAN_SHAPES = [(1001, 1), (777, 3), (256, 7), (300, 16), (200, 33), (64, 64), (100, 100), (50, 1000),
               (64, 2048), (9, 4097), (16, 8192), (150, 12_288), (160, 16_384), (3, 65_537)]


@pytest.mark.parametrize("regime", SCAN_REGIMES)
def test_seg_scan_forced_regimes(fs, regime):
    """Every row-major seg_scan regime forced where its preconditions hold (elsewhere the
    automatic choice stands): add/min/max on every dtype (the look-back scan, 5, is the only
    one the automatic plan no longer gives add/min/max on aligned buffers of these
    lengths), argmin; fs_last_seg_regime must equal fs_seg_regime under the same force."""
    fs.force_seg_regime(regime)
    try:
        for nseg, L in SCAN_SHAPES:
            for dt, op in ((np.float32, "add"), (np.int32, "add"), (np.int64, "add"), (np.int64, "min"),
                           (np.int32, "max"), (np.float32, "argmin")):
                if np.dtype(dt).kind == "i" and op == "add":
                    x = workloads.full_range(nseg * L, nseg + L, dt)
                else:
                    x = workloads.mixed(nseg * L, nseg + L, dt)
                if op == "argmin":
                    x[::7] = x.min()
                got = fs.seg_scan(cu(x), nseg, L, op)
                launched = fs.last_seg_regime()
                assert launched == fs.seg_regime(nseg, L, op=op, dtype=torch.from_numpy(x[:0]).dtype, scan=True), \
                    (nseg, L, dt, op, launched)
                want = oracle.seg_scan(x, nseg, L, op)
                if op == "add" and dt == np.float32:
                    asum = oracle.seg_scan(np.abs(x), nseg, L, "add")
                    err = np.abs(host(got).astype(np.float64) - want)
                    assert np.all(err <= 1e-4 * asum + 1e-30), (nseg, L, regime)
                else:
                    eq(got, want, f"seg_scan forced {regime} {nseg}x{L} {np.dtype(dt).name} {op}")
    finally:
        fs.force_seg_regime(-1)


def test_seg_scan_lookback_covers_every_op_and_dtype(fs):
    """With 5 forced the segmented look-back scan runs for add/min/max/argmin on every dtype
    (misaligned views included), which the automatic plan now reaches only in corners."""
    fs.force_seg_regime(5)
    try:
        for dt in (np.int32, np.int64, np.float32):
            for op in ("add", "min", "max", "argmin"):
                for nseg, L, off in ((300, 100, 0), (777, 64, 1), (5, 20_001, 0), (4, 70_001, 3)):
                    x = workloads.mixed(nseg * L, L + off, dt)
                    if np.dtype(dt).kind == "i" and op == "add":
                        x = workloads.full_range(nseg * L, L, dt)
                    got = fs.seg_scan(cu(x, off), nseg, L, op)
                    assert fs.last_seg_regime() == 5
                    want = oracle.seg_scan(x, nseg, L, op)
                    if op == "add" and dt == np.float32:
                        asum = oracle.seg_scan(np.abs(x), nseg, L, "add")
                        assert np.all(np.abs(host(got).astype(np.float64) - want) <= 1e-4 * asum + 1e-30)
                    else:
                        eq(got, want, f"look-back {np.dtype(dt).name} {op} {nseg}x{L}+{off}")
    finally:
        fs.force_seg_regime(-1)


def test_seg_regime_query_matches_launch(fs):
    """fs_seg_regime (the boundary's answer) equals the regime actually launched, for the C4
    seglen sweep shapes at 2^22 elements (2^27 for rows longer than 8192), every dtype, add and
    argmin, both primitives and both layouts (run-time multi-versioning)."""
    tdt = {np.int32: torch.int32, np.int64: torch.int64, np.float32: torch.float32}
    seen = set()
    for L in workloads.C4_SEGLENS:
        n = 1 << 22 if L <= 8192 else 1 << 27
        if L > n:
            continue
        nseg = n // L
        for dt in (np.float32, np.int32, np.int64):
            if dt == np.int64 and n > (1 << 22):
                continue
            x = torch.zeros(nseg * L, dtype=tdt[dt], device="cuda")
            for op in ("add", "argmin"):
                for layout in ("row", "col"):
                    for scan in (False, True):
                        if scan and n > (1 << 22) and op == "argmin":
                            continue
                        f = fs.seg_scan if scan else fs.seg_reduce
                        f(x, nseg, L, op, layout=layout)
                        got = fs.last_seg_regime()
                        want = fs.seg_regime(nseg, L, op=op, dtype=tdt[dt], layout=layout, scan=scan)
                        assert got == want, (L, nseg, dt, op, layout, scan, got, want)
                        seen.add((scan, got))
            del x
    torch.cuda.synchronize()
    assert {r for s, r in seen if s} >= {4, 5, 7, 9, 10, 11, 12}, seen  # (KS1, 8, is forced-only)
    assert {r for s, r in seen if not s} >= {0, 1, 2, 3, 4}, seen


# ------------------------------------------------------------------ R18 on the GPU
def _r18():
    with open(os.path.join(os.path.dirname(__file__), "golden", "kmeans_r18_fma.json")) as f:
        g = json.load(f)
    pts = np.array([[float.fromhex(v) for v in r] for r in g["points"]], np.float32)
    cen = np.array([[float.fromhex(v) for v in r] for r in g["centres"]], np.float32)
    return g, pts, cen


def test_kmeans_r18_fixture(fs):
    """Points whose R18 membership (exact rationals, tools/gen_golden_r18.py) differs from
    mul+add / reversed-order / exact / f64-accumulated / last-wins decisions: the fused
    kernel's certified argmin must reproduce R18 on every one, alone and tiled among
    ordinary points across many chunks, stages and CTAs."""
    g, pts, cen = _r18()
    m, _, counts, _, _ = fs.kmeans_step(cu(pts), cu(cen))
    np.testing.assert_array_equal(host(m), np.array(g["membership"], np.int32))
    r = np.random.default_rng(3)
    filler = (r.random((200_000, 34)) * 2 - 0.5).astype(np.float32)
    big = np.concatenate([filler, np.tile(pts, (50, 1))])
    perm = r.permutation(big.shape[0])
    big = big[perm]
    m, _, counts, _, _ = fs.kmeans_step(cu(big), cu(cen))
    wm = oracle.kmeans_step(big, cen)[0]
    np.testing.assert_array_equal(host(m), wm)
    pos = np.argsort(perm)[filler.shape[0]:]  # where the fixture's copies landed
    np.testing.assert_array_equal(host(m)[pos], np.tile(np.array(g["membership"], np.int32), 50))


# ------------------------------------------------------------------ full-size C5 legs
def _pool():
    return cf.ThreadPoolExecutor(max_workers=max(1, min(32, os.cpu_count() or 1)))


@pytest.mark.slow
def test_full_c5_kmeans_step(fs):
    """BASELINE configs[4] single-GPU shape: one fused K-means step over n = 2^26, d = 34,
    k = 32 (the bench's inputs and centres).  Membership compared on EVERY point with the
    oracle run chunk by chunk on the host cores (threads; the ctypes calls release the GIL),
    counts and delta exact, sums within 1e-4 of the f64 oracle."""
    pts, prev = workloads.c5_kmeans_shard(0, "cuda")
    n, d = pts.shape
    g = torch.Generator(device="cuda").manual_seed(77)
    cen = pts[torch.randint(0, n, (32,), device="cuda", generator=g)].clone()
    m, sums, counts, newc, delta = fs.kmeans_step(pts, cen, prev=prev)
    torch.cuda.synchronize()
    cen_h = host(cen)
    chunk = 1 << 20

    def work(a):
        p, pv, gm = host(pts[a:a + chunk]), host(prev[a:a + chunk]), host(m[a:a + chunk])
        wm, ws, wc, _, wd = oracle.kmeans_step(p, cen_h, pv)
        return int(np.count_nonzero(gm != wm)), ws, wc.astype(np.int64), wd

    ws = np.zeros((32, d))
    wc = np.zeros(32, np.int64)
    wd = 0
    bad = 0
    with _pool() as ex:
        for b, s, c, dl in ex.map(work, range(0, n, chunk)):
            bad += b
            ws += s
            wc += c
            wd += dl
    assert bad == 0, f"{bad} membership mismatches"
    np.testing.assert_array_equal(host(counts), wc.astype(np.int32))
    assert int(host(delta)[0]) == wd
    assert np.all(np.abs(host(sums).astype(np.float64) - ws) <= 1e-4 * ws)
    want_c = np.where(wc[:, None] > 0, ws / np.maximum(wc[:, None], 1), cen_h)
    assert np.all(np.abs(host(newc).astype(np.float64) - want_c) <= 1e-4 * np.abs(want_c))


@pytest.mark.slow
def test_full_c5_transpose_blocks_vs_oracle(fs):
    """The 2^14 x 2^14 f32 transpose (configs[4]) compared with oracle.transpose_2d on
    sampled row blocks: the oracle transposes the block [a, a+B) x [0, 2^14) and the result
    must equal the GPU result's column block (the first, the last and random blocks)."""
    from workloads import C5_T
    x = workloads.device_uniform((C5_T, C5_T), 6, "cuda")
    t = fs.transpose_2d(x)
    torch.cuda.synchronize()
    B = 256
    starts = sorted({0, C5_T - B} | set(int(a) * B for a in workloads.rng(5).integers(0, C5_T // B, 6)))
    for a in starts:
        want = oracle.transpose_2d(host(x[a:a + B]))
        np.testing.assert_array_equal(host(t[:, a:a + B]), want, err_msg=f"rows {a}..{a + B}")
    # a ragged block too (odd offset and width)
    want = oracle.transpose_2d(host(x[777:777 + 33, 5:5 + 1001]))
    np.testing.assert_array_equal(host(t[5:5 + 1001, 777:777 + 33]), want)


# ------------------------------------------------------------------ ring scan tile edges
# scan_ring_kernel (scanomap and the segmented look-back scan on 16-byte aligned buffers,
# add/min/max): tiles of 256 x 9 16-byte vectors = 9216 four-byte / 4608 eight-byte elements.
RING_TILE = {4: 9216, 8: 4608}


@pytest.mark.parametrize("dt", [np.int32, np.int64, np.float32])
@pytest.mark.parametrize("op", ["add", "min", "max"])
def test_scanomap_ring_tile_edges(fs, dt, op):
    """Sizes one element around a tile, a ragged sub-vector tail, one tile short of and just
    past a whole ring of tiles per SM, and a carry-in continuing a previous scan (F5)."""
    t = RING_TILE[np.dtype(dt).itemsize]
    for n in (1, 3, t - 1, t, t + 1, t + 3, 2 * t + 2, 6 * 148 * t - 1, 6 * 148 * t + 5):
        if np.dtype(dt).kind == "i":
            x = wrap_input(n, n % 89, dt, op)
        else:
            x = workloads.mixed(n, n % 89, dt)
        got = fs.scanomap(cu(x), op)
        want = oracle.scan(x, op)
        if dt == np.float32 and op == "add":
            asum = oracle.scan(np.abs(x), "add")
            assert np.all(np.abs(host(got).astype(np.float64) - want) <= 1e-4 * asum + 1e-30), n
        else:
            eq(got, want, f"ring scan {np.dtype(dt).name} {op} n={n}")
    if op == "add" and np.dtype(dt).kind == "i":
        x = workloads.full_range(5 * t + 7, 11, dt)
        h = 2 * t + 1
        a = fs.scanomap(cu(x[:h]), "add")
        b = fs.scanomap(cu(x[h:]), "add", carry=a[-1:].clone())
        eq(torch.cat([a, b]), oracle.scan(x, "add"), "ring scan carry")


@pytest.mark.parametrize("dt", [np.int32, np.int64, np.float32])
def test_seg_scan_ring_rows_around_tile(fs, dt):
    """Segmented ring scan: rows shorter than, equal to and longer than a tile, row starts
    inside and at tile boundaries (the look-back stops at the first flagged predecessor)."""
    t = RING_TILE[np.dtype(dt).itemsize]
    fs.force_seg_regime(5)
    try:
        for nseg, L in ((40, t - 1), (30, t), (20, t + 1), (7, 3 * t + 5), (3, 40 * t + 1)):
            for op in ("add", "max"):
                x = workloads.full_range(nseg * L, L, dt) if np.dtype(dt).kind == "i" else \
                    workloads.mixed(nseg * L, L, dt)
                got = fs.seg_scan(cu(x), nseg, L, op)
                want = oracle.seg_scan(x, nseg, L, op)
                if dt == np.float32 and op == "add":
                    asum = oracle.seg_scan(np.abs(x), nseg, L, "add")
                    assert np.all(np.abs(host(got).astype(np.float64) - want) <= 1e-4 * asum + 1e-30)
                else:
                    eq(got, want, f"ring seg_scan {np.dtype(dt).name} {op} {nseg}x{L}")
    finally:
        fs.force_seg_regime(-1)


# ------------------------------------------------------------------ long columns
@pytest.mark.parametrize("nseg,seglen", [(4, 700_001), (8, 400_003), (16, 200_000), (32, 90_001), (64, 47_777),
                                         (128, 23_333), (256, 12_001)])
def test_seg_scan_col_long(fs, nseg, seglen):
    """Column-major seg_scan of few long columns (the narrow and one-pass look-back column
    kernels, ragged row blocks); int wrap-around, min/max bit-exact, f32 add within R2."""
    for dt, op in ((np.float32, "add"), (np.int32, "add"), (np.int32, "max"), (np.float32, "min")):
        x = workloads.full_range(nseg * seglen, nseg + seglen, dt) if (op == "add" and dt == np.int32) else \
            workloads.mixed(nseg * seglen, nseg * 7 + seglen, dt)
        got = fs.seg_scan(cu(x), nseg, seglen, op, layout="col")
        want = oracle.seg_scan(x, nseg, seglen, op, "col")
        if op == "add" and dt == np.float32:
            asum = oracle.seg_scan(np.abs(x), nseg, seglen, "add", "col")
            assert np.all(np.abs(host(got).astype(np.float64) - want) <= 1e-4 * asum + 1e-30), (nseg, seglen)
        else:
            eq(got, want, f"col long {nseg}x{seglen} {np.dtype(dt).name} {op}")
