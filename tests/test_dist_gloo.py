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
    """CPU stand-in for the CUDA binding: same call signatures, oracle arithmetic."""

    @staticmethod
    def _out(x, like):
        return torch.from_numpy(np.asarray(x).astype(like.numpy().dtype).reshape(-1))

    def redomap(self, x, op="add", ibase=0, **kw):
        a = x.numpy()
        if op == "argmin":
            v, i = oracle.reduce(a, "argmin")
            return torch.tensor(v, dtype=x.dtype), torch.tensor(i + ibase if i >= 0 else -1)
        return torch.tensor(oracle.reduce(a, op)).to(x.dtype)

    def combine(self, parts, op="add", part_idx=None):
        a = parts.numpy()
        if op == "argmin":
            v, i = oracle.reduce(a, "argmin")
            return torch.tensor(v, dtype=parts.dtype), part_idx[i].clone()
        return torch.tensor(oracle.reduce(a, op)).to(parts.dtype)

    def scanomap(self, x, op="add", carry=None, carry_idx=None, ibase=0, **kw):
        a = x.numpy()
        if carry is None:
            r = oracle.scan(a, op)
            if op == "argmin":
                return torch.from_numpy(r[0]), torch.from_numpy(r[1] + ibase)
            return torch.from_numpy(r.astype(a.dtype))
        # F5: c (+) scan(x) = scan(c # x)[1:]
        r = oracle.scan(np.concatenate([carry.numpy(), a]), op)
        if op == "argmin":
            v, i = r[0][1:], r[1][1:]
            gi = np.where(i == 0, int(carry_idx.item()), i - 1 + ibase)
            return torch.from_numpy(v.copy()), torch.from_numpy(gi)
        return torch.from_numpy(r[1:].astype(a.dtype))

    def stream_red(self, vals, keys, k):
        s, c = oracle.stream_red(vals.numpy(), keys.numpy(), k)
        return torch.from_numpy(s.astype(vals.numpy().dtype)), torch.from_numpy(c)

    def seg_reduce(self, x, nseg, seglen, op="add", layout="row"):
        return torch.from_numpy(np.asarray(oracle.seg_reduce(x.numpy(), nseg, seglen, op, layout)))

    def seg_scan(self, x, nseg, seglen, op="add", layout="row"):
        return torch.from_numpy(np.asarray(oracle.seg_scan(x.numpy(), nseg, seglen, op, layout)))

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


def _worker(rank, world, port, fails):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    tdist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_pldi_henriksenseho17_b200 import dist as fd
        be = OracleShim()
        # ---- redomap / scanomap over a global i32 / f32 array, uneven shards
        for dt in (np.int32, np.int64, np.float32):
            n = 10_007
            x = workloads.mixed(n, 3, dt)
            x[17] = x[9000] = x.min()  # tie across the two shards: rank 0's index wins
            lo, hi = fd.shard_range(n, rank, world)
            xl = torch.from_numpy(x[lo:hi].copy())
            for op in ("add", "min", "max"):
                r = fd.redomap(xl, op, group=None, backend=be)
                w = oracle.reduce(x, op)
                if dt == np.float32 and op == "add":
                    assert abs(float(r) - w) <= 1e-4 * oracle.reduce(np.abs(x), "add")
                else:
                    assert r.item() == w, (dt, op, r, w)
            v, i = fd.redomap(xl, "argmin", ibase=lo, backend=be)
            wv, wi = oracle.reduce(x, "argmin")
            assert (v.item(), i.item()) == (wv, wi)
            for op in ("add", "max"):
                s = fd.scanomap(xl, op, ibase=lo, backend=be).numpy()
                w = oracle.scan(x, op)[lo:hi]
                if dt == np.float32 and op == "add":
                    assert np.all(np.abs(s - w) <= 1e-4 * oracle.scan(np.abs(x), "add")[lo:hi] + 1e-12)
                else:
                    np.testing.assert_array_equal(s, w)
            sv, si = fd.scanomap(xl, "argmin", ibase=lo, backend=be)
            wv, wi = oracle.scan(x, "argmin")
            np.testing.assert_array_equal(si.numpy(), wi[lo:hi])
            np.testing.assert_array_equal(sv.numpy(), wv[lo:hi])
        # ---- k-means partial centroids: rows sharded, one all_reduce
        pts, mem = workloads.c3_kmeans(n=9_001, d=34, k=5)
        lo, hi = fd.shard_range(pts.shape[0], rank, world)
        sums, counts = fd.stream_red(torch.from_numpy(pts[lo:hi].copy()), torch.from_numpy(mem[lo:hi].copy()), 5,
                                     backend=be)
        ws, wc = oracle.stream_red(pts, mem, 5)
        np.testing.assert_array_equal(counts.numpy(), wc)
        np.testing.assert_allclose(sums.numpy(), ws, rtol=1e-5)
        # ---- one K-means iteration over sharded points: local fused step + one all_reduce
        prev = workloads.ints(pts.shape[0], 8, 0, 5)
        cen = pts[:5].copy()
        m, ks, kc, kn, kd = fd.kmeans_step(torch.from_numpy(pts[lo:hi].copy()), torch.from_numpy(cen),
                                           prev_local=torch.from_numpy(prev[lo:hi].copy()), backend=be)
        wm, wsum, wcnt, wnew, wdel = oracle.kmeans_step(pts, cen, prev)
        np.testing.assert_array_equal(m.numpy(), wm[lo:hi])
        np.testing.assert_array_equal(kc.numpy(), wcnt)
        assert int(kd.item()) == wdel
        np.testing.assert_allclose(ks.numpy(), wsum, rtol=1e-5)
        np.testing.assert_allclose(kn.numpy(), wnew, rtol=1e-5)
        # ---- NEXT-4 row nest, rows sharded
        xr = workloads.mixed(50 * 33, 6, np.float32)
        rlo2, rhi2 = fd.shard_range(50, rank, world)
        mp, rs = fd.seg_map_reduce(torch.from_numpy(xr[rlo2 * 33:rhi2 * 33].copy()), rhi2 - rlo2, 33, 1.0, backend=be)
        wmp, wrs = oracle.seg_map_reduce(xr, 50, 33, 1.0)
        np.testing.assert_array_equal(mp.numpy(), wmp[rlo2 * 33:rhi2 * 33])
        np.testing.assert_allclose(rs.numpy(), wrs[rlo2:rhi2], rtol=1e-6)
        # ---- outer segments sharded, no exchange
        nseg, L = 101, 37
        xs = workloads.mixed(nseg * L, 4, np.int32)
        slo, shi = fd.shard_range(nseg, rank, world)
        part = fd.seg_reduce(torch.from_numpy(xs[slo * L:shi * L].copy()), shi - slo, L, "add", backend=be)
        np.testing.assert_array_equal(part.numpy(), oracle.seg_reduce(xs, nseg, L, "add")[slo:shi])
        # ---- transpose of a row block = column block of the global transpose
        m = workloads.mixed((64, 48), 5, np.float32)
        rlo, rhi = fd.shard_range(64, rank, world)
        tb = fd.transpose_2d(torch.from_numpy(m[rlo:rhi].copy()), backend=be)
        np.testing.assert_array_equal(tb.numpy(), oracle.transpose_2d(m)[:, rlo:rhi])
    except Exception as e:  # noqa: BLE001
        fails.put(f"rank {rank}: {type(e).__name__}: {e}")
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


def test_dist_world2_gloo():
    ctx = mp.get_context("spawn")
    fails = ctx.Queue()
    mp.start_processes(_worker, args=(2, _free_port(), fails), nprocs=2, join=True, start_method="spawn")
    assert fails.empty()
