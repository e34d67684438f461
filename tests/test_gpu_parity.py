"""GPU parity: every libfutseg primitive (through the C ABI, via the binding)
against the sequential CPU oracle on the same seeded inputs.

Bar (BASELINE.json north_star):
  * integers, indices, argmin (value and index), min/max: bit-exact;
  * f32 add: |gpu - oracle_f64| <= 1e-4 * sum|x| (per output; for non-negative
    data this is the 1e-4 relative bound), every scan position checked.
Sizes span several tiles and a ragged tail; edge cases: empty, one element,
misaligned (offset) pointers, ties, every segmented regime forced.
"""
import numpy as np
import pytest
import torch

import oracle
import workloads

pytestmark = pytest.mark.gpu

DTYPES = [np.int32, np.int64, np.float32]
OPS = ["add", "min", "max", "argmin"]
TOL = 1e-4


@pytest.fixture(scope="module")
def fs():
    import paper_conf_pldi_henriksenseho17_b200 as m
    return m


def cu(a, offset=0):
    """numpy -> CUDA tensor; offset > 0 returns a view starting `offset` elements in (misaligned)."""
    a = np.ascontiguousarray(a)
    if offset:
        pad = np.zeros(offset, a.dtype)
        t = torch.from_numpy(np.concatenate([pad, a.reshape(-1)])).cuda()
        return t[offset:].view(a.shape) if a.ndim > 1 else t[offset:]
    return torch.from_numpy(a).cuda()


def host(t):
    return t.detach().cpu().numpy()


def assert_reduced(got, want, op, absx_sum=None, where=""):
    """got: GPU result (tensor or (v, i)); want: oracle result; absx_sum: oracle sum of |x| (f32 add)."""
    if op == "argmin":
        gv, gi = host(got[0]), host(got[1])
        wv, wi = want
        np.testing.assert_array_equal(gi, wi, err_msg=f"argmin index {where}")
        np.testing.assert_array_equal(gv, wv, err_msg=f"argmin value {where}")
        return
    g = host(got)
    w = np.asarray(want)
    if op == "add" and w.dtype == np.float64:
        bound = TOL * np.asarray(absx_sum, np.float64) + 1e-30
        err = np.abs(g.astype(np.float64) - w)
        assert np.all(err <= bound), f"f32 add {where}: max err {err.max()} bound {np.min(bound)}"
    else:
        np.testing.assert_array_equal(g, w, err_msg=f"{op} {where}")


# ------------------------------------------------------------------ redomap
@pytest.mark.parametrize("dt", DTYPES)
@pytest.mark.parametrize("op", OPS)
@pytest.mark.parametrize("n,offset", [(0, 0), (1, 0), (3, 1), (1000, 0), (65537, 3), (1 << 20, 0), (3_000_017, 1)])
def test_redomap(fs, dt, op, n, offset):
    x = workloads.mixed(n, 100 + n, dt)
    if n > 10 and op == "argmin":
        x[n // 3] = x[n // 2] = x.min()  # tie: the first occurrence must win
    got = fs.redomap(cu(x, offset), op)
    want = oracle.reduce(x, op)
    asum = oracle.reduce(np.abs(x), "add") if op == "add" and dt == np.float32 else None
    assert_reduced(got, want, op, asum, f"n={n} off={offset}")
    if op == "argmin" and n == 0:
        assert int(host(got[1])) == -1


def test_redomap_c1_full_range_bitexact(fs):
    """BASELINE configs[0]: i32 sum over 2^20 full-range values (wraps), bit-exact."""
    x = workloads.c1()
    assert int(host(fs.redomap(cu(x), "add"))) == int(oracle.reduce(x, "add"))
    xs = workloads.c1(small_range=True)
    assert int(host(fs.redomap(cu(xs), "add"))) == int(oracle.reduce(xs, "add"))
    for op in ("min", "max"):
        assert int(host(fs.redomap(cu(x), op))) == int(oracle.reduce(x, op))


@pytest.mark.parametrize("op", OPS)
def test_redomap_nn_c2(fs, op):
    """BASELINE configs[1]: Rodinia NN argmin over 855,280 (lat, lng) f32 records, duplicated 20x."""
    lat, lng, q = workloads.c2_nn()
    got = fs.redomap(cu(lat), op, map="nn_dist", lng=cu(lng), query=q)
    want = oracle.redomap(lat, op, "nn_dist", lng, q)
    asum = want if op == "add" else None  # distances are non-negative
    assert_reduced(got, want, op, asum, "nn")
    if op == "argmin":
        assert int(host(got[1])) < workloads.NN_BASE  # first of the 20 copies


def test_redomap_nn_misaligned_and_ibase(fs):
    lat, lng, q = workloads.c2_nn(base=5001, reps=3)
    got = fs.redomap(cu(lat, 1), "argmin", map="nn_dist", lng=cu(lng, 2), query=q, ibase=1000)
    v, i = oracle.redomap(lat, "argmin", "nn_dist", lng, q)
    assert float(host(got[0])) == float(v) and int(host(got[1])) == i + 1000


# ------------------------------------------------------------------ NEXT-1: kmeans_step
def _km_check(fs, pts, cen, prev=None, tag=""):
    m, sums, counts, newc, delta = fs.kmeans_step(cu(pts), cu(cen), prev=cu(prev) if prev is not None else None)
    wm, ws, wc, wn, wd = oracle.kmeans_step(pts, cen, prev)
    np.testing.assert_array_equal(host(m), wm)                 # bit-exact assignment
    np.testing.assert_array_equal(host(counts), wc)
    assert int(host(delta)[0]) == wd
    absum = np.zeros_like(ws)
    np.add.at(absum, wm, np.abs(pts).astype(np.float64))
    assert_reduced(sums, ws, "add", absum, f"kmeans sums {tag}")
    got_n = host(newc).astype(np.float64)
    scale = np.where(wc[:, None] > 0, absum / np.maximum(wc[:, None], 1), np.abs(cen))
    assert np.all(np.abs(got_n - wn) <= 1e-4 * scale + 1e-30), f"kmeans new centres {tag}"


@pytest.mark.parametrize("d,k", [(34, 5), (34, 32), (1, 3), (8, 8), (33, 17), (40, 32), (17, 1), (2, 32)])
def test_kmeans_step_shapes(fs, d, k):
    """Random centres picked from the points (so many near-ties on small d): membership
    bit-exact vs the f32 oracle, counts exact, sums/new centres within 1e-4."""
    r = np.random.default_rng(d * 100 + k)
    n = 50_021
    pts = r.random((n, d)).astype(np.float32)
    cen = pts[r.choice(n, k, replace=False)].copy()
    prev = r.integers(0, k, n).astype(np.int32)
    _km_check(fs, pts, cen, prev, f"d={d} k={k}")


def test_kmeans_step_c3_kdd_and_ties(fs):
    """kdd_cup shape (BASELINE configs[2]: n=494,019, d=34, k=5) with clustered points;
    duplicated centres (exact ties: the first wins) and an empty far-away cluster;
    signed data; a few points only; a second iteration from the new centres."""
    pts, mem = workloads.c3_kmeans(keys="clustered")
    cen = pts[:5].copy()
    m, _, _, newc, _ = fs.kmeans_step(cu(pts), cu(cen))
    _km_check(fs, pts, cen, None, "c3")
    _km_check(fs, pts, host(newc), host(m), "c3 iteration 2")
    dup = np.concatenate([cen, cen[:2], np.full((1, 34), 1e3, np.float32)])
    _km_check(fs, pts, dup, None, "duplicated + empty")
    sg = workloads.mixed((30_000, 34), 3, np.float32) * 100
    _km_check(fs, sg, sg[:32].copy(), None, "signed")
    for n in (0, 1, 15, 16, 17, 100):
        small = pts[:n].copy()
        _km_check(fs, small, cen, None, f"n={n}")


# ------------------------------------------------------------------ workspace contract
def test_dirty_workspace_body(fs):
    """The workspace body (past the control words and self-resetting tickets) is never
    assumed zero: fill it with garbage before every primitive and compare with the oracle."""
    HDR = 256 + 4 * 4096

    def dirty():
        ws = fs.workspace(1 << 26, "cuda")
        ws[HDR:].fill_(0xA5)
        torch.cuda.synchronize()

    lat, lng, q = workloads.c2_nn(base=20_000, reps=3)
    dirty()
    d, i = fs.nn_knn(cu(lat), cu(lng), q, 100)
    np.testing.assert_array_equal(host(i), oracle.nn_knn(lat, lng, q, 100)[1])
    pts, _ = workloads.c3_kmeans(n=40_000, d=34, k=32)
    prev = workloads.ints(40_000, 3, 0, 32)
    dirty()
    m, _, cnt, _, dl = fs.kmeans_step(cu(pts), cu(pts[:32].copy()), prev=cu(prev))
    wm, _, wc, _, wd = oracle.kmeans_step(pts, pts[:32].copy(), prev)
    np.testing.assert_array_equal(host(m), wm)
    np.testing.assert_array_equal(host(cnt), wc)
    assert int(host(dl)[0]) == wd
    x = workloads.mixed(3 * 70_001, 5, np.int32)
    dirty()
    mp, rs = fs.seg_map_reduce(cu(x), 3, 70_001, 2, "add")
    np.testing.assert_array_equal(host(rs), oracle.seg_map_reduce(x, 3, 70_001, 2, "add")[1])
    dirty()
    assert int(host(fs.scan_reduce(cu(x), "add"))) == int(oracle.scan_reduce(x, "add", "add"))
    dirty()
    assert int(host(fs.redomap(cu(x), "add"))) == int(oracle.reduce(x, "add"))
    dirty()
    np.testing.assert_array_equal(host(fs.scanomap(cu(x), "add")), oracle.scan(x, "add"))
    dirty()
    np.testing.assert_array_equal(host(fs.seg_reduce(cu(x), 3, 70_001, "max")), oracle.seg_reduce(x, 3, 70_001, "max"))
    dirty()  # the ring scan's segmented look-back (status words zeroed per call, payload never)
    np.testing.assert_array_equal(host(fs.seg_scan(cu(x), 3, 70_001, "add")), oracle.seg_scan(x, 3, 70_001, "add"))
    x8 = workloads.full_range(333_333, 6, np.int64)
    dirty()  # eight-byte tiles: status words plus separate aggregate / inclusive payload arrays
    np.testing.assert_array_equal(host(fs.scanomap(cu(x8), "add")), oracle.scan(x8, "add"))
    dirty()
    s_, c_ = fs.stream_red(cu(pts), cu(prev), 32)
    np.testing.assert_array_equal(host(c_), oracle.stream_red(pts, prev, 32)[1])


# ------------------------------------------------------------------ NEXT-3: scan_reduce
@pytest.mark.parametrize("n", [0, 1, 5, 127, 128, 4097, 1_000_003, 1 << 24])
def test_scan_reduce(fs, n):
    """Fig 10c fusion: reduce (scan x) in one pass, equal to the oracle's materialised scan +
    reduce: integers bit-exact (wrap-around), f32 within 1e-4 of the f64 oracle relative to
    the same computation on |x|."""
    for dt in DTYPES:
        for red in ("add", "max", "min"):
            # add: full-range integers (wrap-around is exact); max/min: no prefix overflow
            # (the max-prefix pair operator needs monotone addition, include/futseg.h)
            full = np.dtype(dt).kind == "i" and red == "add"
            x = workloads.full_range(n, n % 89, dt) if full else workloads.mixed(n, n % 89, dt)
            got = host(fs.scan_reduce(cu(x), red))
            want = oracle.scan_reduce(x, "add", red)
            if dt == np.float32 and n == 0:
                assert float(got) == float(want), (red, got, want)  # the neutral element
            elif dt == np.float32:
                scale = oracle.scan_reduce(np.abs(x), "add", "add") if red == "add" else np.abs(x).sum()
                assert abs(float(got) - float(want)) <= 1e-4 * scale + 1e-30, (n, red, got, want)
            else:
                assert got == want, (n, dt, red, got, want)


def test_scan_reduce_positive_closed_forms(fs):
    """Closed forms on the GPU directly: prefix sums of ones; the max prefix of a +-1 walk."""
    n = 1 << 20
    assert int(host(fs.scan_reduce(torch.ones(n, dtype=torch.int64, device="cuda"), "add"))) == n * (n + 1) // 2
    walk = np.where(np.arange(n) % 3 == 0, -1, 1).astype(np.int32)
    assert int(host(fs.scan_reduce(cu(walk), "max"))) == int(np.cumsum(walk.astype(np.int64)).max())


# ------------------------------------------------------------------ NEXT-4: seg_map_reduce
@pytest.mark.parametrize("nseg,seglen", [(1, 1), (1000, 1), (777, 3), (4096, 4), (300, 32), (1000, 33), (64, 128),
                                         (50, 1000), (9, 4097), (3, 65537), (2, 1_000_003), (0, 5), (7, 0),
                                         (700, 8192), (601, 10_001)])
def test_seg_map_reduce(fs, nseg, seglen):
    """L247-252 fused row nest: x + c written and each row reduced in one read; every op,
    all dtypes, short power-of-two rows (shuffle groups), warp rows, rows cut into pieces."""
    for dt, op in ((np.float32, "add"), (np.int32, "add"), (np.float32, "argmin"), (np.int64, "min"),
                   (np.int32, "max"), (np.int64, "argmin")):
        x = workloads.mixed(nseg * seglen, nseg * 5 + seglen, dt)
        if op == "argmin" and x.size > 10:
            x[::7] = x.min()
        c = 3 if np.dtype(dt).kind == "i" else 1.0
        got = fs.seg_map_reduce(cu(x), nseg, seglen, c, op)
        want = oracle.seg_map_reduce(x, nseg, seglen, c, op)
        np.testing.assert_array_equal(host(got[0]).reshape(-1), want[0])  # the map: exact
        rest_got = (got[1], got[2]) if op == "argmin" else got[1]
        rest_want = (want[1], want[2]) if op == "argmin" else want[1]
        asum = oracle.seg_reduce(np.abs(x), nseg, seglen, "add") if (op == "add" and dt == np.float32) else None
        assert_reduced(rest_got, rest_want, op, asum, f"seg_map_reduce {nseg}x{seglen} {dt.__name__} {op}")


def test_seg_map_reduce_misaligned(fs):
    """Input and output with different 16-byte phases (scalar map stores) and odd offsets."""
    x = workloads.mixed(37 * 1001, 9, np.float32)
    xin = cu(x, 1)
    om = torch.empty(x.size + 2, dtype=torch.float32, device="cuda")[2:]
    got = fs.seg_map_reduce(xin, 37, 1001, 0.5, "add", out_map=om)
    want = oracle.seg_map_reduce(x, 37, 1001, 0.5, "add")
    np.testing.assert_array_equal(host(got[0]), want[0])
    assert_reduced(got[1], want[1], "add", oracle.seg_reduce(np.abs(x), 37, 1001, "add"), "misaligned")


def test_kmeans_finish_matches_fused(fs):
    """fs_kmeans_finish (the multi-GPU layer's last step) = the fused step's own division,
    bit for bit; an empty cluster keeps its centre."""
    pts, _ = workloads.c3_kmeans(n=60_000, d=34, k=8)
    cen = np.concatenate([pts[:7], np.full((1, 34), 9.0, np.float32)])
    m, sums, counts, newc, _ = fs.kmeans_step(cu(pts), cu(cen))
    fin = fs.kmeans_finish(sums, counts, cu(cen))
    np.testing.assert_array_equal(host(fin), host(newc))
    assert int(host(counts)[7]) == 0 and np.all(host(fin)[7] == 9.0)


# ------------------------------------------------------------------ NEXT-2: nn_knn
def _knn_check(fs, lat, lng, q, kk, off=0):
    d, i = fs.nn_knn(cu(lat, off), cu(lng, off), q, kk)
    wd, wi = oracle.nn_knn(lat, lng, q, kk)
    np.testing.assert_array_equal(host(i), wi)                                  # bit-exact indices
    np.testing.assert_array_equal(host(d).view(np.uint32), wd.view(np.uint32))  # and distances


@pytest.mark.parametrize("kk", [1, 5, 100, 257, 1024])
def test_nn_knn_c2(fs, kk):
    """NEXT-2 at the C2 shape: 855,280 records (base duplicated 20x, L1637), the paper's
    100 argmin rounds (L1653-1655) plus other kk; bit-exact against kk oracle rounds."""
    lat, lng, q = workloads.c2_nn()
    _knn_check(fs, lat, lng, q, kk)


@pytest.mark.parametrize("n,kk", [(0, 3), (1, 1), (5, 7), (2047, 100), (2048, 100), (2049, 1024), (4097, 2),
                                  (100_003, 1000), (1_000_003, 100)])
def test_nn_knn_sizes(fs, n, kk):
    """Empty, fewer records than kk (neutral padding), one tile +-1, ragged chunks, many CTAs."""
    base = max(1, n // 7)
    lat, lng, q = workloads.c2_nn(base=base, reps=8, seed=n % 97)
    lat, lng = lat[:n], lng[:n]
    if n == 0:
        d, i = fs.nn_knn(torch.zeros(0, device="cuda"), torch.zeros(0, device="cuda"), q, kk)
        assert host(i).tolist() == [-1] * kk and np.all(np.isinf(host(d)))
        return
    _knn_check(fs, lat, lng, q, kk, off=1 if n % 2 else 0)


def test_nn_knn_adversarial_order(fs):
    """Records sorted by decreasing distance: every tile improves on the running list, so
    the selection keeps flushing (the worst case of the threshold filter); all-equal
    distances: pure index order."""
    lat, lng, q = workloads.c2_nn(base=50_000, reps=1, seed=9)
    dd = oracle.nn_dist(lat, lng, *q)
    order = np.argsort(-dd, kind="stable")
    _knn_check(fs, lat[order].copy(), lng[order].copy(), q, 1024)
    flat = np.full(70_000, 1.5, np.float32)
    _knn_check(fs, flat, flat.copy(), (1.5, 1.5), 300)


@pytest.mark.parametrize("dt", DTYPES)
@pytest.mark.parametrize("k", [1, 5, 34, 100, 1024, 4096])
def test_redomap_vadd(fs, dt, k):
    """VADD(k) over [n][k] = column sums (Fig 4b map(+), G5)."""
    n = 20_011 if k <= 100 else 3001
    x = workloads.mixed((n, k), 7 + k, dt)
    got = fs.redomap(cu(x), "vadd")
    want = oracle.vreduce(x, "add")
    asum = oracle.vreduce(np.abs(x), "add") if dt == np.float32 else None
    assert_reduced(got, want, "add", asum, f"vadd k={k}")


def test_redomap_vadd_empty(fs):
    got = fs.redomap(torch.zeros((0, 7), dtype=torch.float32, device="cuda"), "vadd")
    assert host(got).tolist() == [0.0] * 7


# ------------------------------------------------------------------ combine
@pytest.mark.parametrize("op", OPS)
def test_combine(fs, op):
    parts = workloads.mixed(37, 5, np.float32)
    parts[3] = parts[30] = parts.min()
    pidx = np.arange(37, dtype=np.int64) * 1000 + 5
    got = fs.combine(cu(parts), op, part_idx=cu(pidx) if op == "argmin" else None)
    want = oracle.reduce(parts, op)
    if op == "argmin":
        assert int(host(got[1])) == pidx[want[1]] and float(host(got[0])) == float(want[0])
    else:
        assert_reduced(got, want, op, oracle.reduce(np.abs(parts), "add"), "combine")


# ------------------------------------------------------------------ scanomap
@pytest.mark.parametrize("dt", DTYPES)
@pytest.mark.parametrize("op", OPS)
@pytest.mark.parametrize("n,offset", [(1, 0), (5, 1), (4096, 0), (100_003, 0), (1_000_003, 2), (5_000_011, 0)])
def test_scanomap(fs, dt, op, n, offset):
    x = workloads.mixed(n, 200 + n, dt)
    got = fs.scanomap(cu(x, offset), op)
    want = oracle.scan(x, op)
    asum = oracle.scan(np.abs(x), "add") if op == "add" and dt == np.float32 else None
    assert_reduced(got, want, op, asum, f"scan n={n}")


def test_scanomap_full_range_i32_and_carry(fs):
    x = workloads.c1(1 << 20)
    np.testing.assert_array_equal(host(fs.scanomap(cu(x), "add")), oracle.scan(x, "add"))
    # carry-in (F5's accumulator a): scan of the second half continued from the first
    h = x.size // 2
    first = fs.scanomap(cu(x[:h]), "add")
    second = fs.scanomap(cu(x[h:]), "add", carry=first[-1:].clone())
    np.testing.assert_array_equal(np.concatenate([host(first), host(second)]), oracle.scan(x, "add"))
    y = workloads.mixed(50_000, 3, np.float32)
    y[10] = y[40_000] = y.min()
    a = fs.scanomap(cu(y[:25_000]), "argmin")
    b = fs.scanomap(cu(y[25_000:]), "argmin", carry=a[0][-1:].clone(), carry_idx=a[1][-1:].clone(), ibase=25_000)
    wv, wi = oracle.scan(y, "argmin")
    np.testing.assert_array_equal(np.concatenate([host(a[1]), host(b[1])]), wi)
    np.testing.assert_array_equal(np.concatenate([host(a[0]), host(b[0])]), wv)


@pytest.mark.parametrize("op", ["add", "min", "argmin"])
def test_scanomap_nn(fs, op):
    lat, lng, q = workloads.c2_nn(base=30_011, reps=3)
    got = fs.scanomap(cu(lat), op, map="nn_dist", lng=cu(lng), query=q)
    want = oracle.scanomap(lat, op, "nn_dist", lng, q)
    assert_reduced(got, want, op, want if op == "add" else None, "scan nn")


# ------------------------------------------------------------------ seg_reduce
SEG_SHAPES = [(1, 1), (1000, 1), (777, 3), (513, 7), (300, 16), (200, 33), (64, 64), (100, 100), (50, 1000),
              (9, 4097), (3, 65537), (2, 300_001), (1, 1_000_003)]


@pytest.mark.parametrize("nseg,seglen", SEG_SHAPES)
@pytest.mark.parametrize("regime", [-1, 0, 1, 2, 3])
def test_seg_reduce_regimes_f32_and_i32(fs, nseg, seglen, regime):
    fs.force_seg_regime(regime)
    try:
        for dt, op in ((np.float32, "add"), (np.int32, "add"), (np.float32, "argmin"), (np.int64, "max")):
            x = workloads.mixed(nseg * seglen, nseg + seglen, dt)
            got = fs.seg_reduce(cu(x), nseg, seglen, op)
            want = oracle.seg_reduce(x, nseg, seglen, op)
            asum = oracle.seg_reduce(np.abs(x), nseg, seglen, "add") if (op == "add" and dt == np.float32) else None
            assert_reduced(got, want, op, asum, f"seg {nseg}x{seglen} r={regime} {dt.__name__} {op}")
    finally:
        fs.force_seg_regime(-1)


@pytest.mark.parametrize("dt", DTYPES)
@pytest.mark.parametrize("op", OPS)
def test_seg_reduce_all_ops_misaligned(fs, dt, op):
    for nseg, seglen in [(333, 5), (65, 129), (5, 20_001)]:
        x = workloads.mixed(nseg * seglen, 9, dt)
        got = fs.seg_reduce(cu(x, 1), nseg, seglen, op)
        want = oracle.seg_reduce(x, nseg, seglen, op)
        asum = oracle.seg_reduce(np.abs(x), nseg, seglen, "add") if (op == "add" and dt == np.float32) else None
        assert_reduced(got, want, op, asum, f"seg misaligned {nseg}x{seglen}")


@pytest.mark.parametrize("dt", DTYPES)
@pytest.mark.parametrize("op", OPS)
@pytest.mark.parametrize("nseg,seglen", [(1, 1), (1, 5000), (7, 3), (1000, 50), (5, 20_000), (100_000, 3), (4096, 64)])
def test_seg_reduce_col_major(fs, dt, op, nseg, seglen):
    """as_column_major (L1431): same logical rows, stored column-major."""
    x = workloads.mixed(nseg * seglen, 31, dt)
    cm = np.ascontiguousarray(x.reshape(nseg, seglen).T).reshape(-1)
    got = fs.seg_reduce(cu(cm), nseg, seglen, op, layout="col")
    want = oracle.seg_reduce(cm, nseg, seglen, op, "col")
    asum = oracle.seg_reduce(np.abs(cm), nseg, seglen, "add", "col") if (op == "add" and dt == np.float32) else None
    assert_reduced(got, want, op, asum, f"col {nseg}x{seglen}")
    if dt != np.float32 or op != "add":  # C-13: col(transpose X) == row(X) bit for bit
        row = fs.seg_reduce(cu(x), nseg, seglen, op)
        if op == "argmin":
            np.testing.assert_array_equal(host(row[1]), host(got[1]))
        else:
            np.testing.assert_array_equal(host(row), host(got))


@pytest.mark.parametrize("dt", DTYPES)
@pytest.mark.parametrize("op", OPS)
@pytest.mark.parametrize("nseg,seglen,layout", [
    (3 * 2560 + 17, 3, "row"), (8192 * 2 + 5, 1, "row"), (1001, 33, "row"), (777, 63, "row"), (2049, 31, "row"),
    (310_001, 3, "col"), (303_105, 7, "col"), (256, 100_003, "col"), (5, 200_003, "col"), (64, 400_009, "col"),
    (268, 5_003, "col"), (1024, 4_099, "col"), (1000, 4_096, "col"), (3, 9_001, "col"), (1, 70_001, "col"),
    (1025, 5_000, "col")])
def test_seg_reduce_tiled_rows_and_split_columns(fs, dt, op, nseg, seglen, layout):
    """Row layout, odd seglen <= 63: whole rows staged by TMA, one thread per row, several tiles
    and a ragged last tile.  Column layout: m <= 8 rows of >= 148*8*256 columns (the short-rows
    kernel), narrow w <= 1024 read as one flat vector stream (periods of rows, leftover rows), and
    hundreds of row splits (the two-level combine of partial rows)."""
    x = workloads.mixed(nseg * seglen, nseg ^ seglen, dt)
    got = fs.seg_reduce(cu(x), nseg, seglen, op, layout=layout)
    want = oracle.seg_reduce(x, nseg, seglen, op, layout)
    asum = oracle.seg_reduce(np.abs(x), nseg, seglen, "add", layout) if (op == "add" and dt == np.float32) else None
    assert_reduced(got, want, op, asum, f"{layout} {nseg}x{seglen}")
    if layout == "col" and nseg * seglen < (1 << 22):  # misaligned base: the short-rows kernel takes any phase
        got = fs.seg_reduce(cu(x, 1), nseg, seglen, op, layout=layout)
        assert_reduced(got, want, op, asum, f"{layout} {nseg}x{seglen} misaligned")


def test_seg_reduce_empty(fs):
    for op in OPS:
        got = fs.seg_reduce(torch.zeros(0, dtype=torch.float32, device="cuda"), 5, 0, op)
        want = oracle.seg_reduce(np.zeros(0, np.float32), 5, 0, op)
        if op == "argmin":
            assert host(got[1]).tolist() == [-1] * 5
        else:
            np.testing.assert_array_equal(host(got), want.astype(np.float32))
    assert fs.seg_reduce(torch.zeros(0, dtype=torch.int32, device="cuda"), 0, 7, "add").numel() == 0


# ------------------------------------------------------------------ seg_scan
@pytest.mark.parametrize("nseg,seglen", [(1, 1), (1000, 1), (777, 3), (300, 16), (200, 33), (50, 1000), (9, 4097),
                                         (3, 65537), (1, 1_000_003)])
@pytest.mark.parametrize("layout", ["row", "col"])
def test_seg_scan(fs, nseg, seglen, layout):
    for dt, op in ((np.float32, "add"), (np.int32, "add"), (np.float32, "argmin"), (np.int64, "min"),
                   (np.int32, "max")):
        x = workloads.mixed(nseg * seglen, nseg * 3 + seglen, dt)
        got = fs.seg_scan(cu(x), nseg, seglen, op, layout=layout)
        want = oracle.seg_scan(x, nseg, seglen, op, layout)
        asum = oracle.seg_scan(np.abs(x), nseg, seglen, "add", layout) if (op == "add" and dt == np.float32) else None
        assert_reduced(got, want, op, asum, f"segscan {layout} {nseg}x{seglen} {dt.__name__} {op}")


@pytest.mark.parametrize("seglen", [1, 2, 4, 8, 16, 32, 64, 128, 256, 512, 1024, 2048, 4096, 8192])
@pytest.mark.parametrize("nseg", [1, 3, 1001, 7_001])
def test_seg_scan_short_pow2(fs, nseg, seglen):
    """KS0 (regime 7): power-of-two rows by in-register + shuffle scans (one warp) and a
    shared-memory combine across warps (256..1024 f32, 128..512 8-byte), rows of 2-8
    chunks (2048..8192 f32, 1024..4096 8-byte; 8-byte 8192 takes the look-back scan); every
    op and dtype, ragged vector tails for
    L < 4, argmin ties, int wrap-around."""
    for dt, op in ((np.float32, "add"), (np.int32, "add"), (np.float32, "argmin"), (np.int64, "min"),
                   (np.int32, "max"), (np.int64, "add"), (np.int64, "argmin"), (np.float32, "max")):
        x = workloads.mixed(nseg * seglen, nseg + seglen, dt)
        if op == "argmin" and x.size > 8:
            x[::5] = x.min()  # ties inside segments: the first index must win
        if dt == np.int32 and op == "add":
            x = workloads.full_range(x.size, seglen, np.int32)
        got = fs.seg_scan(cu(x), nseg, seglen, op)
        want = oracle.seg_scan(x, nseg, seglen, op)
        asum = oracle.seg_scan(np.abs(x), nseg, seglen, "add") if (op == "add" and dt == np.float32) else None
        assert_reduced(got, want, op, asum, f"segscan short {nseg}x{seglen} {dt.__name__} {op}")


@pytest.mark.parametrize("nseg,seglen", [(4, 70_001), (8, 4096), (16, 100_003), (32, 9_999), (2, 300_007),
                                         (4, 2_000_000)])
def test_seg_scan_col_narrow(fs, nseg, seglen):
    """Column-major seg_scan with few columns (rows of <= 8 16-byte vectors): the one-pass
    look-back kernel (blocks stacked down the columns, per-column look-back); ragged row
    blocks; argmin ties; 8-byte types."""
    for dt, op in ((np.float32, "add"), (np.int32, "add"), (np.float32, "argmin"), (np.int64, "min"),
                   (np.int64, "add"), (np.int32, "max")):
        if np.dtype(dt).itemsize == 8 and nseg > 16:
            continue
        x = workloads.mixed(nseg * seglen, nseg * 7 + seglen, dt)
        if op == "argmin":
            x[::3] = x.min()
        got = fs.seg_scan(cu(x), nseg, seglen, op, layout="col")
        want = oracle.seg_scan(x, nseg, seglen, op, "col")
        asum = oracle.seg_scan(np.abs(x), nseg, seglen, "add", "col") if (op == "add" and dt == np.float32) else None
        assert_reduced(got, want, op, asum, f"segscan col narrow {nseg}x{seglen} {dt.__name__} {op}")


@pytest.mark.parametrize("nseg,seglen", [(128, 64), (128, 100_003), (256, 65), (1024, 1000), (4096, 3001),
                                         (128 * 37, 777), (1 << 17, 64)])
def test_seg_scan_col_wide(fs, nseg, seglen):
    """Column-major seg_scan with wide rows (multiples of 128 four-byte columns, 16-byte
    vectors): the one-pass look-back kernel over several column tiles (or one thread per
    column when no row split is needed) with ragged row blocks, int wrap-around, 8-byte
    types and argmin."""
    for dt, op in ((np.float32, "add"), (np.int32, "add"), (np.int32, "min"), (np.float32, "max"),
                   (np.float32, "min"), (np.int64, "add"), (np.float32, "argmin")):
        x = workloads.mixed(nseg * seglen, nseg * 5 + seglen, dt)
        if dt == np.int32 and op == "add":
            x = workloads.full_range(x.size, seglen, np.int32)
        got = fs.seg_scan(cu(x), nseg, seglen, op, layout="col")
        want = oracle.seg_scan(x, nseg, seglen, op, "col")
        asum = oracle.seg_scan(np.abs(x), nseg, seglen, "add", "col") if (op == "add" and dt == np.float32) else None
        assert_reduced(got, want, op, asum, f"segscan col wide {nseg}x{seglen} {dt.__name__} {op}")


@pytest.mark.parametrize("nseg,seglen,offset", [(303_105, 3, 0), (310_001, 7, 1), (303_104, 2, 0), (5, 100_003, 0),
                                                (37, 20_011, 0), (3, 1_000_003, 0), (200, 5_000, 1), (33, 40_000, 2)])
def test_seg_scan_col_short_and_scalar(fs, nseg, seglen, offset):
    """Column layout: m <= 8 rows of >= 148 * 2048 columns (the short-rows kernel, any phase),
    and widths that are not multiples of the vector (or misaligned views): scalar columns
    through the one-pass look-back kernel."""
    for dt, op in ((np.float32, "add"), (np.int32, "add"), (np.float32, "argmin"), (np.int64, "min"),
                   (np.int32, "max")):
        x = workloads.mixed(nseg * seglen, nseg * 11 + seglen, dt)
        if op == "argmin":
            x[::4] = x.min()
        got = fs.seg_scan(cu(x, offset), nseg, seglen, op, layout="col")
        want = oracle.seg_scan(x, nseg, seglen, op, "col")
        asum = oracle.seg_scan(np.abs(x), nseg, seglen, "add", "col") if (op == "add" and dt == np.float32) else None
        assert_reduced(got, want, op, asum, f"segscan col {nseg}x{seglen}+{offset} {dt.__name__} {op}")


def test_seg_scan_few_long_rows(fs):
    """Fewer rows than SMs, each >= 2^26 long and 16-byte aligned: one flat slab scan per
    row (indices restart at every row: checked by argmin on the second row's ties)."""
    nseg, seglen = 2, 1 << 26
    for dt, op in ((np.float32, "add"), (np.int32, "max"), (np.int32, "argmin")):
        x = workloads.mixed(nseg * seglen, 4242, dt)
        if op == "argmin":
            x[seglen + 5::9] = x.min()
        got = fs.seg_scan(cu(x), nseg, seglen, op)
        want = oracle.seg_scan(x, nseg, seglen, op)
        asum = oracle.seg_scan(np.abs(x), nseg, seglen, "add") if (op == "add" and dt == np.float32) else None
        assert_reduced(got, want, op, asum, f"segscan long rows {nseg}x{seglen} {dt.__name__} {op}")
        del got, want, asum


@pytest.mark.parametrize("seglen", [4, 64, 512])
def test_seg_scan_pow2_misaligned_falls_back(fs, seglen):
    """KS0 needs 16-byte aligned buffers: a misaligned view of power-of-two rows falls back
    -- to KS1 / KS3 (element-aligned shared-memory staging) for add/min/max at L = 4 / 64,
    512, to the segmented look-back scan for argmin -- and still matches the oracle
    (test_gpu_edges forces the look-back scan for every op and dtype)."""
    nseg = 777
    for dt, op in ((np.float32, "add"), (np.int32, "max"), (np.float32, "argmin")):
        x = workloads.mixed(nseg * seglen, seglen, dt)
        got = fs.seg_scan(cu(x, 1), nseg, seglen, op)
        want = oracle.seg_scan(x, nseg, seglen, op)
        asum = oracle.seg_scan(np.abs(x), nseg, seglen, "add") if (op == "add" and dt == np.float32) else None
        assert_reduced(got, want, op, asum, f"segscan misaligned {seglen} {op}")


@pytest.mark.parametrize("seglen", [3, 5, 7, 9, 12, 17, 31])
@pytest.mark.parametrize("nseg", [1, 2, 255, 256, 257, 100_001])
@pytest.mark.parametrize("regime", [-1, 8])
def test_seg_scan_short_rows_tile(fs, nseg, seglen, regime):
    """Short non-power-of-two rows: KS3 with the TMA ring (regime 11, the default for aligned
    buffers: tiles of R rows, R a multiple of the rows that fill whole 16-byte vectors, the
    leftover rows by the staged-load KS3) and KS1 forced (regime 8: tiles of 256 rows, a ragged
    last tile, scalar tails of the vector loads); add/min/max on every dtype."""
    fs.force_seg_regime(regime)
    try:
        for dt, op in ((np.float32, "add"), (np.int32, "add"), (np.int64, "min"), (np.int32, "max"),
                       (np.int64, "add")):
            x = workloads.full_range(nseg * seglen, seglen, dt) if (op == "add" and dt != np.float32) else \
                workloads.mixed(nseg * seglen, nseg + seglen, dt)
            got = fs.seg_scan(cu(x), nseg, seglen, op)
            if nseg > 1:
                want_rg = 8 if regime == 8 else 11
                assert fs.last_seg_regime() == want_rg, (fs.last_seg_regime(), want_rg)
            want = oracle.seg_scan(x, nseg, seglen, op)
            asum = oracle.seg_scan(np.abs(x), nseg, seglen, "add") if (op == "add" and dt == np.float32) else None
            assert_reduced(got, want, op, asum, f"segscan tile {nseg}x{seglen} {dt.__name__} {op} r={regime}")
    finally:
        fs.force_seg_regime(-1)


@pytest.mark.parametrize("seglen", [33, 100, 1000, 1023, 4097, 8191, 9000, 16_383])
@pytest.mark.parametrize("nseg,offset", [(1, 0), (7, 1), (1001, 0), (300, 3)])
def test_seg_scan_rows_ks3(fs, nseg, seglen, offset):
    """KS3: rows of 32 < L <= 16384 (8192 for 8-byte types) staged R whole rows per CTA in
    shared memory: several rows per CTA and a row per CTA, pieces that straddle row heads,
    a partial last chunk, misaligned views, int wrap-around; argmin and long 8-byte rows
    keep the look-back scan."""
    for dt, op in ((np.float32, "add"), (np.int32, "add"), (np.int64, "min"), (np.int64, "add"),
                   (np.int32, "max"), (np.float32, "min"), (np.float32, "argmin")):
        x = workloads.full_range(nseg * seglen, seglen, dt) if (op == "add" and dt != np.float32) else \
            workloads.mixed(nseg * seglen, nseg * 13 + seglen, dt)
        got = fs.seg_scan(cu(x, offset), nseg, seglen, op)
        want = oracle.seg_scan(x, nseg, seglen, op)
        asum = oracle.seg_scan(np.abs(x), nseg, seglen, "add") if (op == "add" and dt == np.float32) else None
        assert_reduced(got, want, op, asum, f"segscan ks3 {nseg}x{seglen}+{offset} {dt.__name__} {op}")


@pytest.mark.parametrize("nseg,seglen", [(253, 3 * 8192 + 4), (300, 20_000), (256, 65_536), (1000, 12_292)])
def test_seg_scan_row_stream(fs, nseg, seglen):
    """KS2 through the TMA ring (regime 9: >= 1.7 x SMs rows, 16-byte aligned, seglen a multiple
    of the vector): rows of several 8192-element tiles and a partial last tile; add/min/max
    on every dtype, int wrap-around."""
    for dt, op in ((np.float32, "add"), (np.int32, "add"), (np.int64, "min"), (np.int64, "add"),
                   (np.int32, "max"), (np.float32, "min")):
        x = workloads.full_range(nseg * seglen, seglen, dt) if (op == "add" and dt != np.float32) else \
            workloads.mixed(nseg * seglen, nseg + seglen, dt)
        got = fs.seg_scan(cu(x), nseg, seglen, op)
        assert fs.last_seg_regime() == 9, fs.last_seg_regime()
        want = oracle.seg_scan(x, nseg, seglen, op)
        asum = oracle.seg_scan(np.abs(x), nseg, seglen, "add") if (op == "add" and dt == np.float32) else None
        assert_reduced(got, want, op, asum, f"segscan stream {nseg}x{seglen} {dt.__name__} {op}")


@pytest.mark.parametrize("seglen", [2048, 4097, 12_289, 16_384, 65_537])
def test_seg_scan_cta_rows(fs, seglen):
    """KS2 (regime 9): a CTA owns whole rows (>= 4 rows per SM): whole and partial chunks,
    misaligned row starts (odd lengths), argmin indices, int wrap-around; and a misaligned
    view (head elements)."""
    nseg = 4 * 148 + 7
    for dt, op in ((np.float32, "add"), (np.int32, "add"), (np.float32, "argmin"), (np.int64, "min"),
                   (np.int64, "add"), (np.int32, "max")):
        x = workloads.full_range(nseg * seglen, seglen, dt) if (op == "add" and dt != np.float32) else \
            workloads.mixed(nseg * seglen, nseg + seglen, dt)
        if op == "argmin":
            x[::9] = x.min()
        got = fs.seg_scan(cu(x, 1 if seglen % 2 else 0), nseg, seglen, op)
        want = oracle.seg_scan(x, nseg, seglen, op)
        asum = oracle.seg_scan(np.abs(x), nseg, seglen, "add") if (op == "add" and dt == np.float32) else None
        assert_reduced(got, want, op, asum, f"segscan cta {nseg}x{seglen} {dt.__name__} {op}")


def test_seg_scan_misaligned(fs):
    x = workloads.mixed(50 * 999, 4, np.int64)
    got = fs.seg_scan(cu(x, 1), 50, 999, "add")
    np.testing.assert_array_equal(host(got), oracle.seg_scan(x, 50, 999, "add"))


# ------------------------------------------------------------------ stream_red
@pytest.mark.parametrize("keys", ["uniform", "clustered", "skewed"])
def test_stream_red_c3_kdd_shape(fs, keys):
    """BASELINE configs[2]: kdd_cup shape n=494,019, d=34, k=5; counts bit-exact, sums 1e-4."""
    pts, mem = workloads.c3_kmeans(keys=keys)
    sums, counts = fs.stream_red(cu(pts), cu(mem), 5)
    ws, wc = oracle.stream_red(pts, mem, 5)
    np.testing.assert_array_equal(host(counts), wc)
    absum, _ = oracle.stream_red(np.abs(pts), mem, 5)
    assert_reduced(sums, ws, "add", absum, "kmeans c3")


@pytest.mark.parametrize("dt", DTYPES)
@pytest.mark.parametrize("k,w", [(1, 1), (3, 7), (8, 32), (5, 33), (16, 64), (32, 34), (32, 36), (32, 37),
                                 (9, 35), (32, 64), (33, 10), (100, 70), (7, 200), (300, 100), (2000, 40)])
def test_stream_red_shapes(fs, dt, k, w):
    n = 30_011
    vals = workloads.mixed((n, w), k * 100 + w, dt)
    mem = workloads.ints(n, k + w, 0, k)
    sums, counts = fs.stream_red(cu(vals), cu(mem), k)
    ws, wc = oracle.stream_red(vals, mem, k)
    np.testing.assert_array_equal(host(counts), wc)
    absum = oracle.stream_red(np.abs(vals), mem, k)[0] if dt == np.float32 else None
    assert_reduced(sums, ws, "add", absum, f"stream_red k={k} w={w}")


@pytest.mark.parametrize("k,w", [(32, 34), (5, 34), (32, 36), (8, 40)])
def test_stream_red_skewed_staged(fs, k, w):
    """TMA-staged path with skewed keys (90% in cluster 0): the cluster-owner lane of the
    extra features walks up to a whole stage of rows; every chunk's ragged tail too."""
    n = 200_003
    pts, mem = workloads.c3_kmeans(n=n, d=w, k=k, keys="skewed", seed=11)
    sums, counts = fs.stream_red(cu(pts), cu(mem), k)
    ws, wc = oracle.stream_red(pts, mem, k)
    np.testing.assert_array_equal(host(counts), wc)
    assert_reduced(sums, ws, "add", ws, f"stream_red skewed k={k} w={w}")


def test_stream_red_bad_key_staged(fs):
    """An out-of-range key inside a TMA stage is skipped (trash row) and flagged; the
    other rows of that stage still count."""
    n = 100_000
    vals = workloads.mixed((n, 34), 5, np.float32)
    mem = workloads.ints(n, 6, 0, 32)
    bad = [17, 40_000, 99_999]
    fs.check_device_error()
    mem_bad = mem.copy()
    mem_bad[bad] = [32, -1, 1 << 30]
    sums, counts = fs.stream_red(cu(vals), cu(mem_bad), 32)
    with pytest.raises(fs.FutsegError, match="BOUNDS"):
        fs.check_device_error()
    keep = np.ones(n, bool)
    keep[bad] = False
    ws, wc = oracle.stream_red(vals[keep], mem[keep], 32)
    np.testing.assert_array_equal(host(counts), wc)
    absum, _ = oracle.stream_red(np.abs(vals[keep]), mem[keep], 32)
    assert_reduced(sums, ws, "add", absum, "stream_red bad keys staged")


def test_stream_red_small_and_empty(fs):
    for n in (0, 1, 17):
        vals = workloads.mixed((n, 34), 1, np.float32)
        mem = workloads.ints(n, 2, 0, 5)
        sums, counts = fs.stream_red(cu(vals) if n else torch.zeros((0, 34), device="cuda"),
                                     cu(mem) if n else torch.zeros(0, dtype=torch.int32, device="cuda"), 5)
        ws, wc = oracle.stream_red(vals, mem, 5)
        np.testing.assert_array_equal(host(counts), wc)
        np.testing.assert_allclose(host(sums), ws, rtol=1e-5, atol=1e-6)


def test_stream_red_bad_key_raises(fs):
    vals = workloads.mixed((1000, 4), 1, np.float32)
    mem = workloads.ints(1000, 2, 0, 5)
    mem[123] = 9
    fs.check_device_error()  # clear state
    fs.stream_red(cu(vals), cu(mem), 5)
    with pytest.raises(fs.FutsegError, match="BOUNDS"):
        fs.check_device_error()
    fs.check_device_error()  # cleared


# ------------------------------------------------------------------ transpose
@pytest.mark.parametrize("dt", DTYPES)
@pytest.mark.parametrize("r,c", [(1, 1), (1, 1000), (1000, 1), (32, 32), (33, 65), (1000, 777), (4096, 4096)])
def test_transpose(fs, dt, r, c):
    x = workloads.mixed((r, c), r + c, dt)
    got = fs.transpose_2d(cu(x))
    np.testing.assert_array_equal(host(got), oracle.transpose_2d(x))


# ------------------------------------------------------------------ full BASELINE sizes
_C4 = []


def _c4():
    if not _C4:
        _C4.append(workloads.c4())
    return _C4[0]


@pytest.mark.slow
def test_full_c1_seg_reduce_1024x1024(fs):
    x = workloads.c1()
    for regime in (-1, 0, 1, 2, 3):
        fs.force_seg_regime(regime)
        try:
            got = fs.seg_reduce(cu(x), 1024, 1024, "add")
        finally:
            fs.force_seg_regime(-1)
        np.testing.assert_array_equal(host(got), oracle.seg_reduce(x, 1024, 1024, "add"))


@pytest.mark.slow
@pytest.mark.parametrize("seglen", [1, 32, 1024, 65536, 1 << 28])
def test_full_c4_seg_reduce_and_scan(fs, seglen):
    """BASELINE configs[3] at full size (2^28 f32): seg_reduce compared everywhere; seg_scan
    compared on a sample of 4096 positions plus every segment end."""
    x = _c4()
    nseg = (1 << 28) // seglen
    xt = cu(x)
    got = host(fs.seg_reduce(xt, nseg, seglen, "add"))
    want = oracle.seg_reduce(x, nseg, seglen, "add")
    err = np.abs(got.astype(np.float64) - want)
    assert np.all(err <= TOL * want + 1e-30), err.max()  # non-negative data: relative bound
    sc = fs.seg_scan(xt, nseg, seglen, "add")
    del xt
    r = workloads.rng(99)
    pos = np.unique(np.concatenate([r.integers(0, 1 << 28, 4096), np.arange(nseg)[:4096] * seglen + seglen - 1]))
    gs = host(sc[torch.from_numpy(pos).cuda()]).astype(np.float64)
    ws = oracle.seg_scan(x, nseg, seglen, "add")[pos] if seglen <= 65536 else oracle.scan(x, "add")[pos]
    assert np.all(np.abs(gs - ws) <= TOL * ws + 1e-30)


@pytest.mark.slow
def test_full_c5_transpose_and_kmeans(fs):
    """BASELINE configs[4] single-GPU legs: transpose 2^14 x 2^14 f32 (sampled rows) and the
    k-means update n=2^26, d=34, k=32 checked against the oracle chunk by chunk (F3 combine)."""
    from workloads import C5_T
    x = workloads.device_uniform((C5_T, C5_T), 6, "cuda")
    t = fs.transpose_2d(x)
    rows = workloads.rng(5).integers(0, C5_T, 16)
    for j in rows:
        np.testing.assert_array_equal(host(t[j]), host(x[:, j]))
    del x, t
    pts, mem = workloads.c5_kmeans_shard(0, "cuda")
    sums, counts = fs.stream_red(pts, mem, 32)
    ws = np.zeros((32, 34))
    wc = np.zeros(32, np.int64)
    chunk = 1 << 22
    for a in range(0, pts.shape[0], chunk):
        s, c = oracle.stream_red(host(pts[a:a + chunk]), host(mem[a:a + chunk]), 32)
        ws += s
        wc += c
    np.testing.assert_array_equal(host(counts), wc.astype(np.int32))
    assert np.all(np.abs(host(sums).astype(np.float64) - ws) <= TOL * ws)
