"""Pins for the CPU oracle, CPU only.

The oracle is trusted only because of these checks, none of which re-types
its arithmetic: hand-computed fixtures from the paper's definitions
(tests/golden), closed forms, library routines (numpy) on special cases,
brute force over partitions and bracketings on tiny inputs (P-1, P-2),
algebraic identities from the paper (F3/F5 L1067-1074, G5 L1313-1319,
Fig 4a = 4b = 4c L469-505, banana split L203-204) and invariants.
"""
import itertools
import json
import os

import numpy as np
import pytest

import oracle
import workloads

GOLD = os.path.join(os.path.dirname(__file__), "golden")
DTYPES = [np.int32, np.int64, np.float32]
OPS = ["add", "min", "max", "argmin"]


def gold(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


# ---------------------------------------------------------------- golden fixtures
def test_golden_reduce_scan_iota9():
    g = gold("l128_reduce_iota9.json")
    x = np.array(g["input"], np.int32)
    assert oracle.reduce(x, "add") == g["reduce"]
    assert oracle.scan(x, "add").tolist() == g["scan"]


def test_golden_row_sums_l247():
    g = gold("l247_row_sums.json")
    x = np.array(g["input"], np.float32)
    got = oracle.seg_reduce(x, g["nseg"], g["seglen"], "add")
    assert got.tolist() == g["row_sums"]


def test_golden_fig4_counts_and_sums():
    g = gold("fig4_counts.json")
    pts = np.array(g["points"], np.float32)
    mem = np.array(g["membership"], np.int32)
    sums, counts = oracle.stream_red(pts, mem, g["k"])
    assert counts.tolist() == g["counts"]
    assert sums.tolist() == g["sums"]


def test_golden_nn_argmin_ties():
    g = gold("nn_argmin_ties.json")
    x = np.array(g["values"], np.float32)
    v, i = oracle.reduce(x, "argmin")
    assert [float(v), i] == g["argmin"]
    sv, si = oracle.scan(x, "argmin")
    assert sv.tolist() == g["scan_values"] and si.tolist() == g["scan_index"]


def test_golden_column_major_l1431():
    g = gold("l1431_column_major.json")
    rm = np.array(g["row_major"], np.int32)
    cm = np.array(g["col_major"], np.int32)
    assert oracle.transpose_2d(rm.reshape(3, 2)).tolist() == g["transpose_of_3x2"]
    assert oracle.seg_reduce(rm, 3, 2, "add", "row").tolist() == g["row_sums"]
    assert oracle.seg_reduce(cm, 3, 2, "add", "col").tolist() == g["row_sums"]
    assert oracle.seg_scan(rm, 3, 2, "add", "row").tolist() == g["row_scans_row_major"]
    assert oracle.seg_scan(cm, 3, 2, "add", "col").tolist() == g["row_scans_col_major"]


# ---------------------------------------------------------------- P-4 closed forms
@pytest.mark.parametrize("n", [0, 1, 2, 1000, 1 << 17, 100_003])
def test_closed_form_sum_iota_wraps(n):
    x32 = np.arange(n, dtype=np.int64).astype(np.int32)  # iota n (wraps past 2^31 only for huge n)
    want = (n * (n - 1) // 2) % (1 << 32)
    want = want - (1 << 32) if want >= (1 << 31) else want
    assert int(oracle.reduce(x32, "add")) == want
    x64 = np.arange(n, dtype=np.int64) * (1 << 40)  # forces i64 wrap for large n
    w64 = (n * (n - 1) // 2 * (1 << 40)) % (1 << 64)
    w64 = w64 - (1 << 64) if w64 >= (1 << 63) else w64
    assert int(oracle.reduce(x64, "add")) == w64


@pytest.mark.parametrize("dt", DTYPES)
def test_closed_form_scan_of_ones(dt):
    n = 5000
    got = oracle.scan(np.ones(n, dt), "add")
    assert got.tolist() == list(range(1, n + 1))


@pytest.mark.parametrize("dt", DTYPES)
def test_closed_form_permutation_extrema(dt):
    n = 777
    perm = workloads.rng(11).permutation(n).astype(dt)
    assert oracle.reduce(perm, "min") == 0
    assert oracle.reduce(perm, "max") == n - 1
    v, i = oracle.reduce(perm, "argmin")
    assert v == 0 and i == int(np.nonzero(perm == 0)[0][0])
    v, i = oracle.reduce(np.full(33, 7, dt), "argmin")
    assert v == 7 and i == 0


@pytest.mark.parametrize("k", [1, 3, 7])
def test_closed_form_counts_mod_k(k):
    n = 1000
    keys = (np.arange(n) % k).astype(np.int32)
    vals = np.ones((n, 1), np.int32)
    sums, counts = oracle.stream_red(vals, keys, k)
    want = [len(range(r, n, k)) for r in range(k)]
    assert counts.tolist() == want and sums[:, 0].tolist() == want


def test_closed_form_seg_sum_of_iota_rows():
    nseg, L = 37, 53
    x = np.arange(nseg * L, dtype=np.int64)
    got = oracle.seg_reduce(x, nseg, L, "add")
    assert got.tolist() == [s * L * L + L * (L - 1) // 2 for s in range(nseg)]


def test_empty_inputs_give_neutral():
    for dt in DTYPES:
        e = np.zeros(0, dt)
        assert oracle.reduce(e, "add") == 0
        v, i = oracle.reduce(e, "argmin")
        assert i == -1
        assert oracle.scan(e, "add").size == 0
        z = oracle.seg_reduce(e, 4, 0, "max")
        assert z.size == 4
        assert (z == (-np.inf if dt == np.float32 else np.iinfo(dt).min)).all()


# ---------------------------------------------------------------- P-10 library routines
@pytest.mark.parametrize("dt", DTYPES)
def test_library_reduce_scan(dt):
    x = workloads.mixed(4099, 21, dt)
    if dt == np.float32:
        assert oracle.reduce(x, "add") == pytest.approx(np.sum(x, dtype=np.float64), rel=1e-12, abs=1e-9)
        np.testing.assert_allclose(oracle.scan(x, "add"), np.cumsum(x, dtype=np.float64), rtol=1e-12, atol=1e-9)
    else:
        assert oracle.reduce(x, "add") == np.sum(x, dtype=dt)
        np.testing.assert_array_equal(oracle.scan(x, "add"), np.cumsum(x, dtype=dt))
    assert oracle.reduce(x, "min") == x.min()
    assert oracle.reduce(x, "max") == x.max()
    v, i = oracle.reduce(x, "argmin")
    assert i == int(np.argmin(x)) and v == x.min()
    np.testing.assert_array_equal(oracle.scan(x, "min"), np.minimum.accumulate(x))
    np.testing.assert_array_equal(oracle.scan(x, "max"), np.maximum.accumulate(x))
    sv, si = oracle.scan(x, "argmin")
    want_i = np.array([int(np.argmin(x[: j + 1])) for j in range(0, x.size, 97)])
    np.testing.assert_array_equal(si[::97], want_i)
    np.testing.assert_array_equal(sv, np.minimum.accumulate(x))


def test_library_full_range_i32_wraps():
    x = workloads.c1(1 << 16)
    assert oracle.reduce(x, "add") == np.sum(x, dtype=np.int32)  # numpy wraps modulo 2^32
    np.testing.assert_array_equal(oracle.scan(x, "add"), np.cumsum(x, dtype=np.int32))
    x64 = workloads.full_range(5000, 3, np.int64)
    assert oracle.reduce(x64, "add") == np.sum(x64, dtype=np.int64)


@pytest.mark.parametrize("dt", DTYPES)
@pytest.mark.parametrize("nseg,seglen", [(1, 1), (7, 1), (13, 5), (5, 64), (3, 1000), (1, 4097)])
def test_library_seg_ops(dt, nseg, seglen):
    x = workloads.mixed(nseg * seglen, 5, dt)
    rows = x.reshape(nseg, seglen)
    acc = np.float64 if dt == np.float32 else dt
    np.testing.assert_allclose(oracle.seg_reduce(x, nseg, seglen, "add"), rows.sum(1, dtype=acc), rtol=1e-12)
    np.testing.assert_array_equal(oracle.seg_reduce(x, nseg, seglen, "min"), rows.min(1))
    v, i = oracle.seg_reduce(x, nseg, seglen, "argmin")
    np.testing.assert_array_equal(i, rows.argmin(1))
    np.testing.assert_array_equal(v, rows.min(1))
    colstore = np.ascontiguousarray(rows.T).reshape(-1)
    np.testing.assert_array_equal(oracle.seg_reduce(colstore, nseg, seglen, "max", "col"), rows.max(1))
    np.testing.assert_allclose(oracle.seg_scan(x, nseg, seglen, "add").reshape(nseg, seglen),
                               np.cumsum(rows, 1, dtype=acc), rtol=1e-12, atol=1e-12)
    cs = oracle.seg_scan(colstore, nseg, seglen, "max", "col").reshape(seglen, nseg)
    np.testing.assert_array_equal(cs, np.maximum.accumulate(rows, 1).T)


def test_library_stream_red_bincount_and_add_at():
    pts, mem = workloads.c3_kmeans(n=20_000, d=34, k=5)
    sums, counts = oracle.stream_red(pts, mem, 5)
    np.testing.assert_array_equal(counts, np.bincount(mem, minlength=5))
    want = np.zeros((5, 34))
    np.add.at(want, mem, pts.astype(np.float64))
    np.testing.assert_allclose(sums, want, rtol=1e-12)


def test_library_transpose():
    for dt in (np.int32, np.int64, np.float32):
        x = workloads.mixed((37, 129), 9, dt)
        np.testing.assert_array_equal(oracle.transpose_2d(x), x.T)


def test_library_nn_dist_bitexact_with_numpy_f32():
    lat, lng, q = workloads.c2_nn(base=5000, reps=2)
    d0 = lat - np.float32(q[0])
    d1 = lng - np.float32(q[1])
    want = np.sqrt(d0 * d0 + d1 * d1)  # numpy f32 ops: separately rounded, no contraction
    got = oracle.nn_dist(lat, lng, *q)
    assert got.dtype == np.float32
    np.testing.assert_array_equal(got.view(np.uint32), want.view(np.uint32))
    v, i = oracle.redomap(lat, "argmin", "nn_dist", lng, q)
    assert i == int(np.argmin(want)) and i < 5000  # first copy wins (duplicated data, L1637)


def test_golden_nn_knn_hand():
    g = gold("nn_knn_hand.json")
    d, i = oracle.nn_knn(np.array(g["lat"], np.float32), np.array(g["lng"], np.float32), g["q"], g["kk"])
    assert d.tolist() == [float(v) for v in g["dist"]] and i.tolist() == g["idx"]


def test_library_nn_knn_is_a_lexicographic_sort():
    """kk rounds of argmin-with-exclusion = the first kk of the records sorted by
    (distance, index) (np.lexsort, a different algorithm), incl. the 20x ties (L1637)."""
    lat, lng, q = workloads.c2_nn(base=3000, reps=20)
    d0 = lat - np.float32(q[0])
    d1 = lng - np.float32(q[1])
    dist = np.sqrt(d0 * d0 + d1 * d1)
    order = np.lexsort((np.arange(dist.size), dist))
    for kk in (1, 7, 100, 257):
        d, i = oracle.nn_knn(lat, lng, q, kk)
        np.testing.assert_array_equal(i, order[:kk])
        np.testing.assert_array_equal(d.view(np.uint32), dist[order[:kk]].view(np.uint32))
    # closed form of the duplication: each distance recurs at stride base, in index order
    d, i = oracle.nn_knn(lat, lng, q, 60)
    assert i[:20].tolist() == [int(i[0]) + 3000 * r for r in range(20)]
    assert np.all(d[:20] == d[0]) and d[20] > d[0]
    # kk = 1 is the argmin redomap (pinned above); kk > n pads with the neutral element
    v, j = oracle.redomap(lat, "argmin", "nn_dist", lng, q)
    assert oracle.nn_knn(lat, lng, q, 1)[1][0] == j
    d, i = oracle.nn_knn(lat[:5], lng[:5], q, 7)
    assert sorted(i[:5].tolist()) == list(range(5)) and i[5:].tolist() == [-1, -1]
    assert np.all(np.isinf(d[5:])) and np.all(np.diff(d[:5]) >= 0)


def test_golden_kmeans_step_hand():
    g = gold("kmeans_step_hand.json")
    m, sums, counts, newc, delta = oracle.kmeans_step(np.array(g["points"], np.float32),
                                                      np.array(g["centres"], np.float32), np.array(g["prev"]))
    assert m.tolist() == g["membership"] and counts.tolist() == g["counts"] and delta == g["delta"]
    assert sums.tolist() == g["sums"]
    np.testing.assert_allclose(newc, g["new_centres"], rtol=1e-15)


def test_kmeans_step_against_float64_brute_force():
    """Assignment: the f32 fma distance argmin is the float64 argmin except at f32-level
    near-ties, where it is still a valid minimum; centre update = numpy bincount / add.at /
    mean (library routines); the empty cluster keeps its centre; delta = changed labels."""
    r = np.random.default_rng(17)
    x = r.random((20_000, 34)).astype(np.float32)
    cen = x[r.choice(x.shape[0], 31, replace=False)].copy()
    cen = np.concatenate([cen, np.full((1, 34), 50.0, np.float32)])  # far away: stays empty
    prev = r.integers(0, 32, x.shape[0]).astype(np.int32)
    m, sums, counts, newc, delta = oracle.kmeans_step(x, cen, prev)
    e64 = ((x.astype(np.float64)[:, None, :] - cen.astype(np.float64)[None]) ** 2).sum(-1)
    best = e64.min(1)
    assert np.all(e64[np.arange(x.shape[0]), m] <= best * (1 + 1e-5))
    assert np.mean(m == e64.argmin(1)) > 0.999
    np.testing.assert_array_equal(counts, np.bincount(m, minlength=32))
    want = np.zeros((32, 34))
    np.add.at(want, m, x.astype(np.float64))
    np.testing.assert_allclose(sums, want, rtol=1e-12)
    assert counts[31] == 0 and np.all(newc[31] == 50.0)
    for c in range(31):
        np.testing.assert_allclose(newc[c], x[m == c].astype(np.float64).mean(0), rtol=1e-12)
    assert delta == int(np.count_nonzero(m != prev))


def test_kmeans_step_closed_forms():
    r = np.random.default_rng(5)
    x = r.random((500, 7)).astype(np.float32)
    # centres taken from the points: those points are at distance exactly 0
    idx = np.array([3, 100, 250, 499])
    m, *_ = oracle.kmeans_step(x, x[idx])
    assert m[idx].tolist() == [0, 1, 2, 3]
    # a duplicated centre never wins (ties go to the first)
    cen = np.concatenate([x[idx], x[idx[:1]]])
    m2, _, counts, _, _ = oracle.kmeans_step(x, cen)
    assert counts[4] == 0 and np.array_equal(m2, m)
    # k = 1: every point in cluster 0; the new centre is the column mean; no prev -> delta 0
    m1, s1, c1, n1, d1 = oracle.kmeans_step(x, x[:1])
    assert np.all(m1 == 0) and c1.tolist() == [500] and d1 == 0
    np.testing.assert_allclose(n1[0], x.astype(np.float64).mean(0), rtol=1e-12)
    # banana split / Fig 4c: the centre sums are stream_red over the new membership
    s_sr, c_sr = oracle.stream_red(x, m, 4)
    _, s_k, c_k, _, _ = oracle.kmeans_step(x, x[idx])
    np.testing.assert_array_equal(c_sr, c_k)
    np.testing.assert_allclose(s_sr, s_k, rtol=1e-12)


def test_golden_l247_map_reduce():
    g = gold("l247_map_reduce.json")
    x = np.array(g["matrix"], np.float32)
    mapped, sums = oracle.seg_map_reduce(x, 2, 3, g["c"])
    assert mapped.reshape(2, 3).tolist() == g["mapped"] and sums.tolist() == g["sums"]


@pytest.mark.parametrize("dt", DTYPES)
def test_seg_map_reduce_against_numpy(dt):
    """The mapped output is numpy's x + c (f32: the same single rounding; ints: wrap-around);
    the reduced output is seg_reduce of the ORIGINAL rows (pinned above)."""
    x = workloads.full_range((37, 129), 11, dt) if np.dtype(dt).kind == "i" else workloads.mixed((37, 129), 11, dt)
    c = 7 if np.dtype(dt).kind == "i" else 0.37
    for op in OPS:
        r = oracle.seg_map_reduce(x, 37, 129, c, op)
        want_map = (x.reshape(-1) + np.array(c, dt)).astype(dt) if np.dtype(dt).kind == "f" else \
            (x.reshape(-1).astype(np.int64 if dt == np.int32 else np.uint64) + c).astype(dt)
        np.testing.assert_array_equal(r[0], want_map)
        want_red = oracle.seg_reduce(x, 37, 129, op)
        if op == "argmin":
            np.testing.assert_array_equal(r[1], want_red[0])
            np.testing.assert_array_equal(r[2], want_red[1])
        else:
            np.testing.assert_array_equal(r[1], want_red)


@pytest.mark.parametrize("dt", DTYPES)
def test_scan_reduce_against_numpy_and_closed_forms(dt):
    """Fig 10a: reduce (scan x) = numpy cumsum then sum / max / min (f64 for f32, wrapping
    int64 arithmetic for ints); closed forms: sum of the prefix sums of ones = n(n+1)/2,
    of iota = sum_i i(i+1)/2; max prefix sum of a +1/-1 walk = its running maximum."""
    x = workloads.mixed(10_007, 21, dt)
    wide = x.astype(np.float64) if dt == np.float32 else x.astype(np.int64)
    cs = np.cumsum(wide)
    def wrap(v):
        return np.array(v).astype(np.int64).astype(dt) if dt != np.float32 else v
    if dt == np.float32:  # numpy sums pairwise: same f64 value up to rounding order
        assert abs(oracle.scan_reduce(x, "add", "add") - np.sum(cs)) <= 1e-12 * np.sum(np.abs(cs))
    else:
        assert oracle.scan_reduce(x, "add", "add") == wrap(np.sum(cs))
    assert oracle.scan_reduce(x, "add", "max") == (cs.max() if dt == np.float32 else wrap(cs.max()))
    assert oracle.scan_reduce(x, "add", "min") == (cs.min() if dt == np.float32 else wrap(cs.min()))
    n = 1000
    assert oracle.scan_reduce(np.ones(n, dt), "add", "add") == n * (n + 1) // 2
    assert oracle.scan_reduce(np.arange(n, dtype=dt), "add", "add") == sum(i * (i + 1) // 2 for i in range(n))
    walk = np.where(np.arange(n) % 3 == 0, -1, 1).astype(dt)
    assert oracle.scan_reduce(walk, "add", "max") == np.cumsum(walk.astype(np.int64)).max()
    assert oracle.scan_reduce(np.zeros(0, dt), "add", "add") == 0  # empty: the reduce's neutral


def test_invalid_key_is_rejected():
    with pytest.raises(ValueError):
        oracle.stream_red(np.ones((3, 2), np.float32), np.array([0, 5, 1]), 3)


# ---------------------------------------------------------------- P-1 brute force partitions
def _partitions(n):
    for cuts in range(1 << max(n - 1, 0)):
        bounds = [0] + [i + 1 for i in range(n - 1) if cuts >> i & 1] + [n]
        yield list(zip(bounds[:-1], bounds[1:]))


@pytest.mark.parametrize("op", OPS)
def test_bruteforce_sfold_partitions(op):
    """sFold (+) f (v1 # ... # vk) = (f e) (+) (f v1) (+) ... (+) (f vk) is the
    same for every partition iff f is a fold with (+) (L255-263, L167-170):
    check the oracle's reduce on all 2^(n-1) contiguous partitions (F3, L1067)."""
    for dt in (np.int32, np.int64):
        x = workloads.mixed(9, 77, dt)
        x[3] = x[7]  # force an argmin tie
        whole = oracle.reduce(x, op)
        for parts in _partitions(x.size):
            if op == "argmin":
                vals = np.array([oracle.reduce(x[a:b], op)[0] for a, b in parts], dt)
                idxs = [oracle.reduce(x[a:b], op)[1] + a for a, b in parts]
                # combining chunk results with (+) = argmin over the per-chunk winners,
                # evaluated by the oracle itself on the chunk-result array
                cv, ci = oracle.reduce(vals, op)
                assert (cv, idxs[ci]) == whole
            else:
                chunk = np.array([oracle.reduce(x[a:b], op) for a, b in parts], dt)
                assert oracle.reduce(chunk, op) == whole


# ---------------------------------------------------------------- P-2 tree shapes
def _brackets(items):
    if len(items) == 1:
        yield items[0]
        return
    for k in range(1, len(items)):
        for left in _brackets(items[:k]):
            for right in _brackets(items[k:]):
                yield ("node", left, right)


def _eval(tree, op, dt):
    """Evaluate a bracketing using only the oracle: a (+) b = reduce [a, b]."""
    if tree[0] != "node":
        return tree
    a = _eval(tree[1], op, dt)
    b = _eval(tree[2], op, dt)
    if op == "argmin":
        v, i = oracle.reduce(np.array([a[0], b[0]], dt), op)
        return (v, (a[1], b[1])[i])
    return (oracle.reduce(np.array([a[0], b[0]], dt), op),)


@pytest.mark.parametrize("op", OPS)
@pytest.mark.parametrize("dt", [np.int32, np.int64])
def test_bruteforce_bracketings(op, dt):
    x = workloads.mixed(6, 5, dt)
    x[1] = x[4]
    leaves = [(x[i], i) if op == "argmin" else (x[i],) for i in range(x.size)]
    whole = oracle.reduce(x, op)
    for tree in _brackets(leaves):
        r = _eval(tree, op, dt)
        assert (r if op == "argmin" else r[0]) == whole


def test_neutral_element_invariants():
    """x (+) 0(+) = 0(+) (+) x = x (L132-133) on extreme samples (P-3)."""
    samples = {
        np.int32: [np.iinfo(np.int32).min, -1, 0, 1, np.iinfo(np.int32).max],
        np.int64: [np.iinfo(np.int64).min, -1, 0, 1, np.iinfo(np.int64).max],
        np.float32: [-np.inf, -1.5, -0.0, 0.0, 3.25, np.inf],
    }
    for dt, vals in samples.items():
        for v in vals:
            one = np.array([v], dt)
            neutral = {"add": 0,
                       "min": np.inf if dt == np.float32 else np.iinfo(dt).max,
                       "max": -np.inf if dt == np.float32 else np.iinfo(dt).min}
            for op in ("add", "min", "max"):
                assert oracle.reduce(one, op) == one[0]  # 0(+) (+) x
                assert oracle.reduce(np.array([v, neutral[op]], dt), op) == one[0]  # x (+) 0(+)
            av, ai = oracle.reduce(one, "argmin")
            assert av == one[0] and ai == 0


# ---------------------------------------------------------------- paper identities
def test_f5_chunk_scan_plus_carry_is_scan():
    """F5 (L1071-1074): scan each chunk, add the carry of the previous chunks."""
    x = workloads.mixed(200, 8, np.int64)
    whole = oracle.scan(x, "add")
    r = workloads.rng(3)
    for _ in range(20):
        cuts = np.sort(r.choice(np.arange(1, 200), size=5, replace=False))
        out, carry = [], np.int64(0)
        for a, b in zip([0, *cuts], [*cuts, 200]):
            yc = oracle.scan(x[a:b], "add") + carry
            out.append(yc)
            carry = yc[-1]
        np.testing.assert_array_equal(np.concatenate(out), whole)


@pytest.mark.parametrize("op", ["add", "min", "max", "argmin"])
def test_g5_vreduce_equals_seg_reduce_of_transpose(op):
    """G5 (L1313-1319): reduce (map (+)) (replicate k 0) zs = map (reduce (+) 0) (transpose zs)."""
    for dt in DTYPES:
        z = workloads.mixed((301, 7), 4, dt)
        a = oracle.vreduce(z, op)
        b = oracle.seg_reduce(oracle.transpose_2d(z), 7, 301, op, "row")
        c = oracle.seg_reduce(z, 7, 301, op, "col")  # as_column_major view (L1431)
        for u, v in ((a, b), (a, c)):
            if op == "argmin":
                np.testing.assert_array_equal(u[0], v[0])
                np.testing.assert_array_equal(u[1], v[1])
            else:
                np.testing.assert_array_equal(u, v)


def test_fig4_three_formulations_agree():
    """Fig 4a (sequential loop) = 4b (reduce map(+) of one-hot increments) = 4c (stream_red)."""
    k = 6
    mem = workloads.ints(3000, 12, 0, k)
    _, counts_a = oracle.stream_red(np.zeros((3000, 0), np.int32), mem, k)
    increments = np.eye(k, dtype=np.int32)[mem]  # Fig 4b's [n][k] one-hot rows
    counts_b = oracle.vreduce(increments, "add")
    # Fig 4c: chunks of arbitrary sizes, each starting from zeros (L529-531), combined by map(+)
    parts = [(0, 1), (1, 700), (700, 701), (701, 3000)]
    per_chunk = np.stack([oracle.stream_red(np.zeros((b - a, 0), np.int32), mem[a:b], k)[1] for a, b in parts])
    counts_c = oracle.vreduce(per_chunk, "add")
    np.testing.assert_array_equal(counts_a, counts_b)
    np.testing.assert_array_equal(counts_a, counts_c)
    np.testing.assert_array_equal(counts_a, np.bincount(mem, minlength=k))


def test_banana_split_sums_and_counts():
    """fold((+)*(+))(f,g) = (fold (+) f, fold (+) g) (L203-204): tupled sums+counts
    equal a sums-only pass and a counts-only pass; counts equal a ones column."""
    pts, mem = workloads.c3_kmeans(n=5000, d=3, k=4)
    sums, counts = oracle.stream_red(pts, mem, 4)
    only_counts = oracle.stream_red(np.zeros((5000, 0), np.float32), mem, 4)[1]
    ones = oracle.stream_red(np.ones((5000, 1), np.int32), mem, 4)[0][:, 0]
    np.testing.assert_array_equal(counts, only_counts)
    np.testing.assert_array_equal(counts, ones)
    for c in range(4):
        np.testing.assert_allclose(sums[c], oracle.vreduce(pts[mem == c], "add"), rtol=1e-12)


def test_segmented_equals_per_segment_flat():
    """P-8: seg_reduce(X)[s] = reduce(X[s]); seg_scan(X)[s] = scan(X[s])."""
    for dt in DTYPES:
        nseg, L = 11, 37
        x = workloads.mixed(nseg * L, 2, dt)
        for op in OPS:
            sr = oracle.seg_reduce(x, nseg, L, op)
            ss = oracle.seg_scan(x, nseg, L, op)
            for s in range(nseg):
                row = x[s * L:(s + 1) * L]
                if op == "argmin":
                    assert (sr[0][s], sr[1][s]) == oracle.reduce(row, op)
                    np.testing.assert_array_equal(ss[1][s * L:(s + 1) * L], oracle.scan(row, op)[1])
                else:
                    assert sr[s] == oracle.reduce(row, op)
                    np.testing.assert_array_equal(ss[s * L:(s + 1) * L], oracle.scan(row, op))


def test_redomap_is_reduce_of_map():
    """fold (+,0) g = reduce (+,0) . map g  (L254) with g = the NN distance."""
    lat, lng, q = workloads.c2_nn(base=300, reps=3)
    d = oracle.nn_dist(lat, lng, *q)
    assert oracle.redomap(lat, "min", "nn_dist", lng, q) == d.min()
    np.testing.assert_array_equal(oracle.scanomap(lat, "max", "nn_dist", lng, q), np.maximum.accumulate(d))


def _r18_fixture():
    g = gold("kmeans_r18_fma.json")
    pts = np.array([[float.fromhex(v) for v in row] for row in g["points"]], np.float32)
    cen = np.array([[float.fromhex(v) for v in row] for row in g["centres"]], np.float32)
    return g, pts, cen


def test_golden_kmeans_r18_fma_rounding():
    """Reading R18 pinned: points whose R18 membership (exact rationals, one rounding per
    fma, index order, first centre on ties; tools/gen_golden_r18.py) differs from the
    decision under separately rounded mul+add, reversed order, exact real arithmetic, an f64
    accumulator, or last-wins ties.  An oracle making any of those mistakes fails here."""
    g, pts, cen = _r18_fixture()
    assert set(g["discriminates"]) == {"mul_add", "reversed", "exact", "f64_acc", "le_ties"}
    m, _, counts, _, _ = oracle.kmeans_step(pts, cen)
    bad = [(i, w) for i, (a, b, w) in enumerate(zip(m.tolist(), g["membership"], g["discriminates"])) if a != b]
    assert not bad, bad
    assert counts[2] == 0
