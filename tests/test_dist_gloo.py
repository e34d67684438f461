"""Multi-process (world_size 2, gloo, CPU) tests of the sharded path in
paper_conf_pldi_henriksenseho17_b200/dist.py: shard ranges, global indices,
rank-ordered argmin combine, scan carries (F5) and the all_reduce of k-means
partials, against the oracle on the unsharded input.

The local primitive runs through an oracle-backed shim with the binding's
signatures (the CUDA library needs a GPU); the collectives are the real
torch.distributed ones.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as tdist
import torch.multiprocessing as mp

import oracle
import workloads


class OracleShim:
    """CPU stand-in for the CUDA binding: same call signatures, oracle arithmetic; results
    are written into ``out=`` views when given (the binding's contract)."""

    @staticmethod
    def _put(res, out):
        if out is None:
            return res
        out.copy_(res.reshape(out.shape))
        return out

    def redomap(self, x, op="add", ibase=0, out=None, **kw):
        a = x.numpy()
        if op == "argmin":
            v, i = oracle.reduce(a, "argmin")
            return torch.tensor(v, dtype=x.dtype), torch.tensor(i + ibase if i >= 0 else -1)
        return self._put(torch.tensor(oracle.reduce(a, op)).to(x.dtype), out)

    def combine(self, parts, op="add", part_idx=None, out=None, out_idx=None):
        a = parts.numpy()
        if op == "argmin":
            v, i = oracle.reduce(a, "argmin")
            return torch.tensor(v, dtype=parts.dtype), part_idx[i].clone()
        return self._put(torch.tensor(oracle.reduce(a, op)).to(parts.dtype), out)

    def scanomap(self, x, op="add", carry=None, carry_idx=None, ibase=0, out=None, **kw):
        a = x.numpy()
        if carry is None:
            r = oracle.scan(a, op)
            if op == "argmin":
                return torch.from_numpy(r[0]), torch.from_numpy(r[1] + ibase)
            return self._put(torch.from_numpy(r.astype(a.dtype)), out)
        # F5: c (+) scan(x) = scan(c # x)[1:]
        r = oracle.scan(np.concatenate([carry.numpy(), a]), op)
        if op == "argmin":
            v, i = r[0][1:], r[1][1:]
            gi = np.where(i == 0, int(carry_idx.item()), i - 1 + ibase)
            return torch.from_numpy(v.copy()), torch.from_numpy(gi)
        return self._put(torch.from_numpy(r[1:].astype(a.dtype)), out)

    # the exchange packing (fs_argmin_pack / _unpack, fs_partials_pack / _unpack): numpy
    @staticmethod
    def argmin_pack(values, idx):
        v, i = values.numpy(), idx.numpy()
        if v.dtype == np.int64:
            return torch.from_numpy(np.stack([v, i], 1).astype(np.int64))
        if v.dtype == np.float32:
            b = np.where(v == 0, np.float32(0), v).view(np.uint32).astype(np.uint64)
            o = np.where(b >> 31 == 1, (~b) & 0xFFFFFFFF, b | 0x80000000)
        else:
            o = (v.view(np.uint32).astype(np.uint64) ^ 0x80000000)
        u = (o << np.uint64(32)) | (i.astype(np.int64).view(np.uint64) & np.uint64(0xFFFFFFFF))
        u = np.where(i < 0, np.uint64(0xFFFFFFFFFFFFFFFF), u)  # "no element" orders last
        return torch.from_numpy((u ^ np.uint64(1 << 63)).view(np.int64).copy())

    @staticmethod
    def argmin_unpack(keys, dtype, P=1):
        k = keys.numpy().reshape(-1)
        if dtype == torch.int64:
            rec = k.reshape(-1, 2)[:P]
            best = (np.iinfo(np.int64).max, -1)
            for v, i in rec:
                if i >= 0 and (best[1] < 0 or (v, i) < best):
                    best = (int(v), int(i))
            return torch.tensor(best[0]), torch.tensor(best[1])
        u = k[:1].view(np.uint64)[0] ^ np.uint64(1 << 63)
        lo, hi = int(u & np.uint64(0xFFFFFFFF)), int(u >> np.uint64(32))
        if lo == 0xFFFFFFFF:
            return (torch.tensor(np.inf, dtype=torch.float32) if dtype == torch.float32
                    else torch.tensor(np.iinfo(np.int32).max, dtype=torch.int32)), torch.tensor(-1)
        if dtype == torch.float32:
            b = np.uint32(hi & 0x7FFFFFFF) if hi >> 31 else np.uint32(~hi & 0xFFFFFFFF)
            return torch.tensor(np.array([b], np.uint32).view(np.float32)[0]), torch.tensor(lo)
        return torch.tensor(np.array([hi ^ 0x80000000], np.uint32).view(np.int32)[0]), torch.tensor(lo)

    @staticmethod
    def partials_pack(sums, counts=None, extra=None):
        s = sums.numpy().reshape(-1)
        c = counts.numpy().reshape(-1) if counts is not None else np.zeros(0)
        e = [int(extra.reshape(-1)[0])] if extra is not None else [0]
        if s.dtype == np.float32:
            return torch.from_numpy(np.concatenate([s.astype(np.float64), c.astype(np.float64), np.array(e, np.float64)]))
        return torch.from_numpy(np.concatenate([s.astype(np.int64), c.astype(np.int64), np.array(e, np.int64)]))

    @staticmethod
    def partials_unpack(packed, sums, counts=None, extra=None):
        p = packed.numpy()
        kw = sums.numel()
        if sums.dtype == torch.float32:
            sums.copy_(torch.from_numpy(p[:kw].astype(np.float32)).reshape(sums.shape))
        else:
            sums.copy_(torch.from_numpy(p[:kw].astype(np.int64).astype(sums.numpy().dtype)).reshape(sums.shape))
        if counts is not None:
            counts.copy_(torch.from_numpy(p[kw:kw + counts.numel()].astype(np.int64).astype(np.int32)))
        if extra is not None:
            extra.copy_(torch.tensor([int(p[-1])], dtype=torch.int64).reshape(extra.shape))
        return sums, counts, extra

    @staticmethod
    def copy_2d(src, rows, cols, src_ld, dst, dst_ld):
        for r in range(rows):
            dst[r * dst_ld:r * dst_ld + cols] = src[r * src_ld:r * src_ld + cols]
        return dst

    def stream_red(self, vals, keys, k):
        s, c = oracle.stream_red(vals.numpy(), keys.numpy(), k)
        return torch.from_numpy(s.astype(vals.numpy().dtype)), torch.from_numpy(c)

    def seg_reduce(self, x, nseg, seglen, op="add", layout="row", out=None):
        return self._put(torch.from_numpy(np.asarray(oracle.seg_reduce(x.numpy(), nseg, seglen, op, layout))
                                          .astype(x.numpy().dtype)), out)

    def seg_scan(self, x, nseg, seglen, op="add", layout="row", out=None):
        return self._put(torch.from_numpy(np.asarray(oracle.seg_scan(x.numpy(), nseg, seglen, op, layout))
                                          .astype(x.numpy().dtype)), out)

    def transpose_2d(self, x):
        return torch.from_numpy(oracle.transpose_2d(x.numpy()))

    def kmeans_step(self, pts, cen, prev=None):
        m, s, c, n, d = oracle.kmeans_step(pts.numpy(), cen.numpy(), None if prev is None else prev.numpy())
        return (torch.from_numpy(m), torch.from_numpy(s.astype(np.float32)), torch.from_numpy(c),
                torch.from_numpy(n.astype(np.float32)), torch.tensor([d], dtype=torch.int64))

    def kmeans_finish(self, sums, counts, cen):
        c = counts.numpy()[:, None]
        return torch.from_numpy(np.where(c > 0, sums.numpy() / np.maximum(c, 1), cen.numpy()).astype(np.float32))

    def seg_map_reduce(self, x, nseg, seglen, c, op="add"):
        r = oracle.seg_map_reduce(x.numpy(), nseg, seglen, c, op)
        return tuple(torch.from_numpy(np.asarray(v)) for v in r)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _check_dist(rank, world, fd, be, to, host):
    """The dist layer against the oracle on the unsharded input; ``to`` moves a numpy array to
    the backend's device, ``host`` brings a result back."""
    # ---- redomap / scanomap over a global array, uneven shards, argmin ties across shards
    for dt in (np.int32, np.int64, np.float32):
        n = 10_007
        x = workloads.mixed(n, 3, dt)
        if np.dtype(dt).kind == "i":
            x[::5] = workloads.full_range(x[::5].size, 7, dt)  # sums wrap (R1)
        x[17] = x[9000] = x.min()  # tie across the shards: the lower global index wins
        lo, hi = fd.shard_range(n, rank, world)
        xl = to(x[lo:hi].copy())
        for op in ("add", "min", "max"):
            r = host(fd.redomap(xl, op, group=None, backend=be))
            w = oracle.reduce(x, op)
            if dt == np.float32 and op == "add":
                assert abs(float(r) - w) <= 1e-4 * oracle.reduce(np.abs(x), "add")
            else:
                assert r.item() == w, (dt, op, r, w)
        v, i = fd.redomap(xl, "argmin", ibase=lo, backend=be)
        wv, wi = oracle.reduce(x, "argmin")
        assert (host(v).item(), host(i).item()) == (wv, wi), (dt, host(v), host(i), wv, wi)
        for op in ("add", "max"):
            s = host(fd.scanomap(xl, op, ibase=lo, backend=be))
            w = oracle.scan(x, op)[lo:hi]
            if dt == np.float32 and op == "add":
                assert np.all(np.abs(s - w) <= 1e-4 * oracle.scan(np.abs(x), "add")[lo:hi] + 1e-12)
            else:
                np.testing.assert_array_equal(s, w)
        sv, si = fd.scanomap(xl, "argmin", ibase=lo, backend=be)
        wv, wi = oracle.scan(x, "argmin")
        np.testing.assert_array_equal(host(si), wi[lo:hi])
        np.testing.assert_array_equal(host(sv), wv[lo:hi])
    # ---- an empty shard (more ranks than elements on some): argmin neutral handling
    x = workloads.mixed(world - 1, 4, np.float32)
    lo, hi = fd.shard_range(x.size, rank, world)
    v, i = fd.redomap(to(x[lo:hi].copy()), "argmin", ibase=lo, backend=be)
    assert (host(v).item(), host(i).item()) == oracle.reduce(x, "argmin")
    # ---- k-means partial centroids: rows sharded, ONE all_reduce of packed sums + counts
    pts, mem = workloads.c3_kmeans(n=9_001, d=34, k=5)
    lo, hi = fd.shard_range(pts.shape[0], rank, world)
    sums, counts = fd.stream_red(to(pts[lo:hi].copy()), to(mem[lo:hi].copy()), 5, backend=be)
    ws, wc = oracle.stream_red(pts, mem, 5)
    np.testing.assert_array_equal(host(counts), wc)
    np.testing.assert_allclose(host(sums), ws, rtol=1e-4)  # R2 (non-negative data)
    for dt in (np.int32, np.int64):  # integer sums: exact modulo 2^32 / 2^64 through the f64-free packing
        vals = workloads.full_range((5_003, 7), 11, dt)
        keys = workloads.ints(5_003, 12, 0, 4)
        lo, hi = fd.shard_range(vals.shape[0], rank, world)
        sums, counts = fd.stream_red(to(vals[lo:hi].copy()), to(keys[lo:hi].copy()), 4, backend=be)
        ws, wc = oracle.stream_red(vals, keys, 4)
        np.testing.assert_array_equal(host(sums), ws)
        np.testing.assert_array_equal(host(counts), wc)
    # ---- one K-means iteration over sharded points: local fused step + one all_reduce
    prev = workloads.ints(pts.shape[0], 8, 0, 5)
    cen = pts[:5].copy()
    lo, hi = fd.shard_range(pts.shape[0], rank, world)
    m, ks, kc, kn, kd = fd.kmeans_step(to(pts[lo:hi].copy()), to(cen), prev_local=to(prev[lo:hi].copy()), backend=be)
    wm, wsum, wcnt, wnew, wdel = oracle.kmeans_step(pts, cen, prev)
    np.testing.assert_array_equal(host(m), wm[lo:hi])
    np.testing.assert_array_equal(host(kc), wcnt)
    assert int(host(kd).reshape(-1)[0]) == wdel
    np.testing.assert_allclose(host(ks), wsum, rtol=1e-4)  # R2 (non-negative data)
    np.testing.assert_allclose(host(kn), wnew, rtol=1e-4)
    # ---- NEXT-4 row nest, rows sharded
    xr = workloads.mixed(50 * 33, 6, np.float32)
    rlo2, rhi2 = fd.shard_range(50, rank, world)
    mp, rs = fd.seg_map_reduce(to(xr[rlo2 * 33:rhi2 * 33].copy()), rhi2 - rlo2, 33, 1.0, backend=be)
    wmp, wrs = oracle.seg_map_reduce(xr, 50, 33, 1.0)
    np.testing.assert_array_equal(host(mp).reshape(-1), wmp[rlo2 * 33:rhi2 * 33])
    bound = 1e-4 * oracle.seg_reduce(np.abs(xr), 50, 33, "add")[rlo2:rhi2] + 1e-30  # R2 (f32 reassociated)
    assert np.all(np.abs(host(rs).astype(np.float64) - wrs[rlo2:rhi2]) <= bound)
    # ---- outer segments sharded, no exchange
    nseg, L = 101, 37
    xs = workloads.mixed(nseg * L, 4, np.int32)
    slo, shi = fd.shard_range(nseg, rank, world)
    part = fd.seg_reduce(to(xs[slo * L:shi * L].copy()), shi - slo, L, "add", backend=be)
    np.testing.assert_array_equal(host(part), oracle.seg_reduce(xs, nseg, L, "add")[slo:shi])
    # ---- fewer segments than GPUs (and more): elements sharded inside the rows
    for nseg, L, dt in ((1, 10_001, np.float32), (2, 7_777, np.int64), (world - 1 or 1, 5_003, np.int32),
                        (5, 3_001, np.int32), (3 * world + 1, 97, np.float32), (1, 3, np.int32)):
        xs = workloads.mixed(nseg * L, nseg + L, dt)
        lo, hi = fd.shard_range(nseg * L, rank, world)
        for op in ("add", "min", "max"):
            o0, red = fd.seg_reduce_elems(to(xs[lo:hi].copy()), nseg, L, op, backend=be)
            want = oracle.seg_reduce(xs, nseg, L, op)[o0:o0 + red.numel()]
            _, _, (w0, w1), _ = fd.elem_plan(nseg, L, rank, world)
            assert (o0, red.numel()) == (w0, w1 - w0)
            sc = host(fd.seg_scan_elems(to(xs[lo:hi].copy()), nseg, L, op, backend=be))
            wsc = oracle.seg_scan(xs, nseg, L, op)[lo:hi]
            if dt == np.float32 and op == "add":
                assert np.all(np.abs(host(red) - want) <= 1e-4 * oracle.seg_reduce(np.abs(xs), nseg, L, "add")[o0:o0 + red.numel()] + 1e-12)
                assert np.all(np.abs(sc - wsc) <= 1e-4 * oracle.seg_scan(np.abs(xs), nseg, L, "add")[lo:hi] + 1e-12)
            else:
                np.testing.assert_array_equal(host(red), want)
                np.testing.assert_array_equal(sc, wsc)
    # ---- transpose of a row block = column block of the global transpose
    m = workloads.mixed((64, 48), 5, np.float32)
    rlo, rhi = fd.shard_range(64, rank, world)
    tb = fd.transpose_2d(to(m[rlo:rhi].copy()), backend=be)
    np.testing.assert_array_equal(host(tb), oracle.transpose_2d(m)[:, rlo:rhi])
    # ---- NEXT-4: the distributed all-to-all transpose (row-sharded in, row-sharded out)
    for rows, cols, dt in ((64, 48, np.float32), (37, 101, np.int64), (5, 3, np.int32), (130, 257, np.float32)):
        m = workloads.mixed((rows, cols), rows + cols, dt)
        rlo, rhi = fd.shard_range(rows, rank, world)
        y = host(fd.transpose_2d_global(to(m[rlo:rhi].copy()), rows, cols, backend=be))
        clo, chi = fd.shard_range(cols, rank, world)
        np.testing.assert_array_equal(y, oracle.transpose_2d(m)[clo:chi])


def _worker(rank, world, port, fails):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    tdist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_pldi_henriksenseho17_b200 import dist as fd
        _check_dist(rank, world, fd, OracleShim(), lambda a: torch.from_numpy(np.ascontiguousarray(a)),
                    lambda t: t.numpy() if isinstance(t, torch.Tensor) else np.asarray(t))
    except Exception as e:  # noqa: BLE001
        import traceback
        fails.put(f"rank {rank}: {type(e).__name__}: {e}\n{traceback.format_exc()}")
        raise
    finally:
        tdist.destroy_process_group()


def test_shard_range_partitions():
    from paper_conf_pldi_henriksenseho17_b200 import dist as fd
    for n in (0, 1, 7, 100):
        for world in (1, 2, 3, 8):
            got = [fd.shard_range(n, r, world) for r in range(world)]
            assert got[0][0] == 0 and got[-1][1] == n
            assert all(a[1] == b[0] for a, b in zip(got, got[1:]))
            sizes = [h - l for l, h in got]
            assert max(sizes) - min(sizes) <= 1


@pytest.mark.parametrize("world", [2, 3])
def test_dist_gloo(world):
    ctx = mp.get_context("spawn")
    fails = ctx.Queue()
    try:
        mp.start_processes(_worker, args=(world, _free_port(), fails), nprocs=world, join=True, start_method="spawn")
    finally:
        msgs = []
        while not fails.empty():
            msgs.append(fails.get())
        assert not msgs, "\n".join(msgs)
