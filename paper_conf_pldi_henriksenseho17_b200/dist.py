"""Multi-GPU layer: one process per GPU, the primitives sharded where they shard
naturally, and ONE collective where the method has a real exchange step
(BASELINE.json north_star: "Outer segments are split across
GPUs.  Whole-array reductions and k-means partial centroids are combined with
one NCCL allreduce over NVLink").

  redomap     contiguous shards; local fold; partials combined by all_reduce
              (add/min/max/vadd) or all_gather + rank-ordered fs_combine (argmin,
              exact and deterministic: the smallest global index wins ties)
  scanomap    contiguous shards; local total -> all_gather of the P totals ->
              carry = combine of the totals of ranks < r (F5's accumulator a,
              L1071-1074) -> local scanomap with carry-in
  stream_red  rows sharded; local chunk results combined by all_reduce (map(+))
  kmeans_step (NEXT-1) points sharded; fused local step, one all_reduce of
              (sums, counts, delta), new centres from the global sums
  seg_reduce, seg_scan, transpose_2d, seg_map_reduce (NEXT-4)
              outer segments / row blocks sharded; no collective

The collectives go through ``torch.distributed`` (NCCL over NVLink on GPUs,
gloo in the CPU tests) on the current stream, with no host synchronisation.
``backend`` is the module that runs the local primitive: the CUDA binding by
default; the CPU tests pass an oracle-backed shim with the same signatures so
the sharding, offsets, rank order and carries are exercised on CPU.
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def _default_backend():
    import paper_conf_pldi_henriksenseho17_b200 as fs
    return fs


def shard_range(n: int, rank: int, world: int):
    """Contiguous block partition of range(n): rank r gets [lo, hi)."""
    base, rem = divmod(n, world)
    lo = rank * base + min(rank, rem)
    return lo, lo + base + (1 if rank < rem else 0)


def _world(group):
    return dist.get_world_size(group), dist.get_rank(group)


_REDUCE_OPS = {"add": dist.ReduceOp.SUM, "vadd": dist.ReduceOp.SUM, "min": dist.ReduceOp.MIN,
               "max": dist.ReduceOp.MAX}


def redomap(x_local, op="add", ibase: int = 0, group=None, backend=None, **map_kw):
    """Global fold of the concatenation of every rank's ``x_local`` (rank order).
    ``ibase`` = global index of x_local[0] (argmin indices are global)."""
    be = backend or _default_backend()
    world, _ = _world(group)
    if op == "argmin":
        v, i = be.redomap(x_local, "argmin", ibase=ibase, **map_kw)
        vs = [torch.empty_like(v.reshape(1)) for _ in range(world)]
        is_ = [torch.empty_like(i.reshape(1)) for _ in range(world)]
        dist.all_gather(vs, v.reshape(1), group=group)
        dist.all_gather(is_, i.reshape(1), group=group)
        return be.combine(torch.cat(vs), "argmin", part_idx=torch.cat(is_))
    r = be.redomap(x_local, op, **map_kw)
    dist.all_reduce(r, op=_REDUCE_OPS[op], group=group)
    return r


def scanomap(x_local, op="add", ibase: int = 0, group=None, backend=None, **map_kw):
    """Global inclusive scan; rank r returns its slice of the result."""
    be = backend or _default_backend()
    world, rank = _world(group)
    if op == "argmin":
        v, i = be.redomap(x_local, "argmin", ibase=ibase, **map_kw)
        vs = [torch.empty_like(v.reshape(1)) for _ in range(world)]
        is_ = [torch.empty_like(i.reshape(1)) for _ in range(world)]
        dist.all_gather(vs, v.reshape(1), group=group)
        dist.all_gather(is_, i.reshape(1), group=group)
        if rank == 0:
            return be.scanomap(x_local, "argmin", ibase=ibase, **map_kw)
        cv, ci = be.combine(torch.cat(vs[:rank]), "argmin", part_idx=torch.cat(is_[:rank]))
        return be.scanomap(x_local, "argmin", carry=cv.reshape(1), carry_idx=ci.reshape(1), ibase=ibase, **map_kw)
    t = be.redomap(x_local, op, **map_kw)
    ts = [torch.empty_like(t.reshape(1)) for _ in range(world)]
    dist.all_gather(ts, t.reshape(1), group=group)
    if rank == 0:
        return be.scanomap(x_local, op, **map_kw)
    carry = be.combine(torch.cat(ts[:rank]), op)
    return be.scanomap(x_local, op, carry=carry.reshape(1), **map_kw)


def stream_red(vals_local, keys_local, k: int, group=None, backend=None):
    """K-means sums/counts over every rank's rows: local stream_red + all_reduce (map(+))."""
    be = backend or _default_backend()
    sums, counts = be.stream_red(vals_local, keys_local, k)
    dist.all_reduce(sums, op=dist.ReduceOp.SUM, group=group)
    dist.all_reduce(counts, op=dist.ReduceOp.SUM, group=group)
    return sums, counts


def kmeans_step(points_local, centres, prev_local=None, group=None, backend=None):
    """One K-means iteration over every rank's points (NEXT-1): the fused local step on the
    shard, then ONE exchange -- all_reduce of the partial sums, counts and changed-label
    count -- and the new centres from the global sums (fs_kmeans_finish).  Returns
    (membership of the local points, sums, counts, new centres, delta)."""
    be = backend or _default_backend()
    m, sums, counts, _, delta = be.kmeans_step(points_local, centres, prev=prev_local)
    dist.all_reduce(sums, op=dist.ReduceOp.SUM, group=group)
    dist.all_reduce(counts, op=dist.ReduceOp.SUM, group=group)
    dist.all_reduce(delta, op=dist.ReduceOp.SUM, group=group)
    return m, sums, counts, be.kmeans_finish(sums, counts, centres), delta


def seg_map_reduce(x_local, nseg_local: int, seglen: int, c, op="add", backend=None):
    """NEXT-4 rows sharded (rank r owns a block of rows): no exchange."""
    be = backend or _default_backend()
    return be.seg_map_reduce(x_local, nseg_local, seglen, c, op)


def seg_reduce(x_local, nseg_local: int, seglen: int, op="add", layout="row", backend=None):
    """Outer segments sharded (rank r owns a contiguous block of rows): no exchange."""
    be = backend or _default_backend()
    return be.seg_reduce(x_local, nseg_local, seglen, op, layout=layout)


def seg_scan(x_local, nseg_local: int, seglen: int, op="add", layout="row", backend=None):
    be = backend or _default_backend()
    return be.seg_scan(x_local, nseg_local, seglen, op, layout=layout)


def transpose_2d(block, backend=None):
    """Rank r transposes its row block [rows_r][cols]; the result is column block r of
    the global transpose (no exchange; a globally row-sharded result would need an
    all-to-all, which the hot path does not require)."""
    be = backend or _default_backend()
    return be.transpose_2d(block)
