"""The multi-GPU layer (paper_conf_pldi_henriksenseho17_b200/dist.py) with the REAL CUDA
backend: two ranks on cuda:0 (this box has one GPU; NCCL refuses two ranks on one device), the
collectives over gloo with the tensors bounced through host memory.  Every local step -- the
primitives, the exchange packing (fs_argmin_pack / _unpack, fs_partials_pack / _unpack) and the
column-block gather of the distributed transpose (fs_copy_2d) -- runs in libfutseg's kernels and
is checked against the oracle on the unsharded input (the same checks as the gloo CPU test)."""
import os
import types

import numpy as np
import pytest
import torch
import torch.distributed as tdist
import torch.multiprocessing as mp

from test_dist_gloo import _check_dist, _free_port

pytestmark = pytest.mark.gpu


def _bounced():
    """torch.distributed with CUDA tensors staged through host memory (gloo on one GPU)."""
    def wrap(fn):
        def call(*args, **kw):
            tens = [a for a in args if isinstance(a, torch.Tensor)]
            host = [t.cpu() for t in tens]
            it = iter(host)
            args2 = [next(it) if isinstance(a, torch.Tensor) else a for a in args]
            torch.cuda.synchronize()
            r = fn(*args2, **kw)
            for t, h in zip(tens, host):
                t.copy_(h)
            return r
        return call
    ns = types.SimpleNamespace(**{k: getattr(tdist, k) for k in dir(tdist) if not k.startswith("__")})
    for name in ("all_reduce", "all_gather_into_tensor", "all_to_all_single"):
        setattr(ns, name, wrap(getattr(tdist, name)))
    return ns


def _worker(rank, world, port, fails):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    tdist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_pldi_henriksenseho17_b200 as fs
        from paper_conf_pldi_henriksenseho17_b200 import dist as fd
        fd.dist = _bounced()
        _check_dist(rank, world, fd, fs, lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda(),
                    lambda t: t.detach().cpu().numpy() if isinstance(t, torch.Tensor) else np.asarray(t))
        torch.cuda.synchronize()
    except Exception as e:  # noqa: BLE001
        import traceback
        fails.put(f"rank {rank}: {type(e).__name__}: {e}\n{traceback.format_exc()}")
        raise
    finally:
        tdist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_dist_cuda_backend_one_gpu(world):
    ctx = mp.get_context("spawn")
    fails = ctx.Queue()
    try:
        mp.start_processes(_worker, args=(world, _free_port(), fails), nprocs=world, join=True, start_method="spawn")
    finally:
        msgs = []
        while not fails.empty():
            msgs.append(fails.get())
        assert not msgs, "\n".join(msgs)


def test_exchange_packing_direct():
    """fs_argmin_pack keys order exactly as R3's (value, index) order (checked on every pair,
    incl. -0 / +0, infinities, INT32 extremes and the 'no element' index -1); fs_partials_pack /
    _unpack round-trip (integer sums modulo 2^32 / 2^64); fs_copy_2d on misaligned views."""
    import paper_conf_pldi_henriksenseho17_b200 as fs
    r = np.random.default_rng(3)
    for dt in (np.float32, np.int32):
        if dt == np.float32:
            v = np.array([-np.inf, -3.5, -0.0, 0.0, 1e-30, 2.0, 2.0, np.inf, 7.0], np.float32)
        else:
            v = np.array([np.iinfo(np.int32).min, -5, 0, 0, 3, 3, np.iinfo(np.int32).max, 9], np.int32)
        idx = r.integers(0, 50, v.size).astype(np.int64)
        idx[-1] = -1  # a rank with no element
        keys = fs.argmin_pack(torch.from_numpy(v).cuda(), torch.from_numpy(idx).cuda()).cpu().numpy()
        for a in range(v.size):
            for b in range(v.size):
                def rk(j):  # R3 order; index -1 (no element) after everything
                    return (1, 0, 0) if idx[j] < 0 else (0, float(v[j]), int(idx[j]))
                assert (keys[a] < keys[b]) == (rk(a) < rk(b)) or (rk(a) == rk(b)), (dt, a, b)
        for j in range(v.size):
            val, ii = fs.argmin_unpack(torch.from_numpy(keys[j:j + 1]).cuda(), torch.from_numpy(v[:1]).dtype)
            if idx[j] < 0:
                assert int(ii) == -1
            else:
                assert int(ii) == idx[j] and float(val) == float(v[j])
    for dt in (np.float32, np.int32, np.int64):
        sums = (r.random((5, 7)) * 100).astype(dt) if dt == np.float32 else \
            r.integers(np.iinfo(dt).min, np.iinfo(dt).max, (5, 7), dtype=dt)
        cnt = r.integers(0, 1000, 5).astype(np.int32)
        ext = torch.tensor([123456789], dtype=torch.int64).cuda()
        p = fs.partials_pack(torch.from_numpy(sums).cuda(), torch.from_numpy(cnt).cuda(), ext)
        p2 = p + p  # two identical ranks
        s2, c2, e2 = torch.empty((5, 7), dtype=torch.from_numpy(sums).dtype, device="cuda"), \
            torch.empty(5, dtype=torch.int32, device="cuda"), torch.empty(1, dtype=torch.int64, device="cuda")
        fs.partials_unpack(p2, s2, c2, e2)
        if dt == np.float32:
            np.testing.assert_array_equal(s2.cpu().numpy(), (sums.astype(np.float64) * 2).astype(np.float32))
        else:
            with np.errstate(over="ignore"):
                np.testing.assert_array_equal(s2.cpu().numpy(), sums + sums)  # wraps (R1)
        np.testing.assert_array_equal(c2.cpu().numpy(), cnt * 2)
        assert int(e2.cpu()) == 2 * 123456789
    src = torch.arange(1, 1 + 7 * 13, dtype=torch.float32, device="cuda")
    dst = torch.zeros(5 * 9 + 1, dtype=torch.float32, device="cuda")
    fs.copy_2d(src[1:], 5, 6, 13, dst[1:], 9)
    want = np.zeros(5 * 9 + 1, np.float32)
    s_ = np.arange(1, 1 + 7 * 13, dtype=np.float32)[1:]
    for rr in range(5):
        want[1 + rr * 9:1 + rr * 9 + 6] = s_[rr * 13:rr * 13 + 6]
    np.testing.assert_array_equal(dst.cpu().numpy(), want)
