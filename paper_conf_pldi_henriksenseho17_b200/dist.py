"""Multi-GPU layer: one process per GPU, the primitives sharded where they shard
naturally, and ONE collective per exchange step (BASELINE.json
north_star: "Outer segments are split across GPUs.  Whole-array reductions and
k-means partial centroids are combined with one NCCL allreduce over NVLink").

  redomap     contiguous shards; local fold; ONE all_reduce of the partials: SUM / MIN /
              MAX (integer SUM wraps, reading R1), ARGMIN as packed keys (fs_argmin_pack:
              the key order is R3's (value, index) order, so MIN is the exact argmin;
              int64 values: one all_gather of (value, index) records)
  scanomap    contiguous shards; local total -> ONE all_gather of the P totals (keys for
              ARGMIN) -> carry = combine of the totals of ranks < r (F5's accumulator a,
              L1071-1074) -> local scanomap with carry-in
  stream_red  rows sharded; local chunk results packed (fs_partials_pack: sums and counts
              in one f64 / int64 buffer) -> ONE all_reduce SUM -> unpacked (map(+), Fig 4c)
  kmeans_step (NEXT-1) points sharded; fused local step; sums, counts and the changed-label
              count packed -> ONE all_reduce -> new centres from the global sums
  seg_reduce, seg_scan, seg_map_reduce (NEXT-4)
              outer segments sharded (nseg >= P): no exchange.  With fewer segments than
              GPUs (e.g. seglen = 2^28, the C4 endpoint) the ELEMENTS are sharded instead
              (seg_reduce_elems / seg_scan_elems): each rank folds its pieces of the rows it
              touches, ONE all_gather of every rank's last-row partial, and the owner of a
              row (the rank holding its last element) combines the partials of the ranks
              before it in rank order (a scan takes them as the carry of its first piece)
  transpose_2d   a row block -> the matching column block of the result (no exchange)
  transpose_2d_global (NEXT-4) a globally row-sharded matrix -> the row-sharded transpose:
              column blocks gathered (fs_copy_2d), ONE all_to_all, one local transpose

The collectives go through ``torch.distributed`` (NCCL over NVLink on GPUs, gloo in the
CPU tests and the one-GPU functional test) on the current stream, with no host
synchronisation.  ``backend`` is the module that runs the local primitive and the
pack / unpack steps: the CUDA binding by default; the CPU tests pass an oracle-backed
shim with the same signatures.
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


def _gather(t, world, group):
    """ONE all_gather of a small contiguous tensor -> [world, *t.shape] (contiguous)."""
    flat = t.contiguous().reshape(-1)
    out = torch.empty(world * flat.numel(), dtype=t.dtype, device=t.device)
    dist.all_gather_into_tensor(out, flat, group=group)  # rank-ordered concatenation
    return out.reshape((world,) + tuple(t.shape))


def _argmin_exchange(be, v, i, world, group):
    """Global argmin of per-rank (value, index) partials with ONE collective."""
    keys = be.argmin_pack(v.reshape(1), i.reshape(1))
    if v.dtype == torch.int64:  # (value, index) records: all_gather, folded in rank order
        return be.argmin_unpack(_gather(keys.reshape(2), world, group), v.dtype, P=world)
    dist.all_reduce(keys, op=dist.ReduceOp.MIN, group=group)
    return be.argmin_unpack(keys, v.dtype, P=1)


def _argmin_prefix(be, keys_all, rank, dtype):
    """ARGMIN of the gathered partials of ranks < rank (keys as packed by argmin_pack)."""
    if dtype == torch.int64:
        return be.argmin_unpack(keys_all[:rank].reshape(-1, 2), dtype, P=rank)
    k = be.redomap(keys_all[:rank].reshape(-1), "min")  # signed key order = R3 order
    return be.argmin_unpack(k.reshape(1), dtype, P=1)


def redomap(x_local, op="add", ibase: int = 0, group=None, backend=None, **map_kw):
    """Global fold of the concatenation of every rank's ``x_local`` (rank order).
    ``ibase`` = global index of x_local[0] (argmin indices are global)."""
    be = backend or _default_backend()
    world, _ = _world(group)
    if op == "argmin":
        v, i = be.redomap(x_local, "argmin", ibase=ibase, **map_kw)
        return _argmin_exchange(be, v, i, world, group)
    r = be.redomap(x_local, op, **map_kw)
    dist.all_reduce(r, op=_REDUCE_OPS[op], group=group)
    return r


def scanomap(x_local, op="add", ibase: int = 0, group=None, backend=None, **map_kw):
    """Global inclusive scan; rank r returns its slice of the result."""
    be = backend or _default_backend()
    world, rank = _world(group)
    if op == "argmin":
        v, i = be.redomap(x_local, "argmin", ibase=ibase, **map_kw)
        keys = _gather(be.argmin_pack(v.reshape(1), i.reshape(1)).reshape(-1), world, group)
        if rank == 0:
            return be.scanomap(x_local, "argmin", ibase=ibase, **map_kw)
        cv, ci = _argmin_prefix(be, keys, rank, v.dtype)
        return be.scanomap(x_local, "argmin", carry=cv.reshape(1), carry_idx=ci.reshape(1), ibase=ibase, **map_kw)
    t = be.redomap(x_local, op, **map_kw)
    ts = _gather(t.reshape(1), world, group).reshape(-1)
    if rank == 0:
        return be.scanomap(x_local, op, **map_kw)
    carry = be.combine(ts[:rank], op)
    return be.scanomap(x_local, op, carry=carry.reshape(1), **map_kw)


def stream_red(vals_local, keys_local, k: int, group=None, backend=None):
    """K-means sums/counts over every rank's rows: local stream_red, then sums and counts
    packed into one buffer and combined by ONE all_reduce SUM (map(+), Fig 4c)."""
    be = backend or _default_backend()
    sums, counts = be.stream_red(vals_local, keys_local, k)
    packed = be.partials_pack(sums, counts)
    dist.all_reduce(packed, op=dist.ReduceOp.SUM, group=group)
    be.partials_unpack(packed, sums, counts)
    return sums, counts


def kmeans_step(points_local, centres, prev_local=None, group=None, backend=None):
    """One K-means iteration over every rank's points (NEXT-1): the fused local step on the
    shard, then ONE exchange -- the partial sums, counts and changed-label count packed into
    one buffer, one all_reduce -- and the new centres from the global sums (fs_kmeans_finish).
    Returns (membership of the local points, sums, counts, new centres, delta)."""
    be = backend or _default_backend()
    m, sums, counts, _, delta = be.kmeans_step(points_local, centres, prev=prev_local)
    packed = be.partials_pack(sums, counts, extra=delta)
    dist.all_reduce(packed, op=dist.ReduceOp.SUM, group=group)
    be.partials_unpack(packed, sums, counts, extra=delta)
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


# ------------------------------------------------------------------ element-sharded segments
def elem_plan(nseg: int, seglen: int, rank: int, world: int):
    """Host-side plan of the element-sharded segmented ops (every rank computes every rank's
    plan; no communication).  Rank r holds elements [lo, hi) of the row-major [nseg][seglen]
    array.  Returns (lo, hi, owned rows [o0, o1), for each rank p the row of its last element)."""
    n = nseg * seglen
    lo, hi = shard_range(n, rank, world)
    last = []
    for p in range(world):
        plo, phi = shard_range(n, p, world)
        last.append((phi - 1) // seglen if phi > plo else -1)
    # row s is owned by the rank holding its last element (s + 1) * seglen - 1
    o0 = (lo + seglen - 1) // seglen if hi > lo else 0   # first row whose last element is >= lo
    o1 = hi // seglen if hi > lo else 0                   # rows whose last element is < hi
    return lo, hi, (o0, max(o0, o1)), last


def _first_rank_of_row(s, nseg, seglen, world):
    """The rank holding element s * seglen (the first rank touching row s)."""
    n = nseg * seglen
    e = s * seglen
    for p in range(world):
        plo, phi = shard_range(n, p, world)
        if plo <= e < phi:
            return p
    return world - 1


def seg_reduce_elems(x_local, nseg: int, seglen: int, op="add", group=None, backend=None):
    """Segmented reduce of a row-major [nseg][seglen] array whose ELEMENTS are sharded
    (rank r holds shard_range(nseg * seglen, r, P)): for nseg < P (long rows split across
    GPUs).  ONE all_gather of each rank's last-row partial; rank r returns (o0, out) with
    out[s - o0] the result of every row s it owns (its last element is on rank r).
    ops add / min / max."""
    if op not in ("add", "min", "max"):
        raise ValueError("seg_reduce_elems: add / min / max")
    be = backend or _default_backend()
    world, rank = _world(group)
    L = seglen
    lo, hi, (o0, o1), _ = elem_plan(nseg, seglen, rank, world)
    x = x_local.reshape(-1)
    # this rank's partial of its last row (the piece after the last row start in [lo, hi))
    if hi > lo:
        l = (hi - 1) // L
        tail = be.redomap(x[max(lo, l * L) - lo:], op)
    else:
        tail = be.redomap(x[:0], op)
    parts = _gather(tail.reshape(1), world, group).reshape(-1)
    out = torch.empty(o1 - o0, dtype=x.dtype, device=x.device)
    if o1 == o0:
        return o0, out
    s = o0
    if lo > o0 * L:  # the first owned row starts on earlier ranks: their partials, then ours
        r0 = _first_rank_of_row(o0, nseg, L, world)
        pair = torch.empty(2, dtype=x.dtype, device=x.device)
        be.combine(parts[r0:rank], op, out=pair[0:1].reshape(()))
        be.redomap(x[:(o0 + 1) * L - lo], op, out=pair[1:2].reshape(()))
        be.combine(pair, op, out=out[0:1].reshape(()))
        s += 1
    if o1 > s:  # whole rows inside this rank
        a = s * L - lo
        be.seg_reduce(x[a:a + (o1 - s) * L], o1 - s, L, op, out=out[s - o0:])
    return o0, out


def seg_scan_elems(x_local, nseg: int, seglen: int, op="add", group=None, backend=None):
    """Segmented inclusive scan with the ELEMENTS sharded (see seg_reduce_elems): the first
    piece of a rank continues a row begun on earlier ranks, so it takes their combined
    partials as its carry (F5); whole rows and the last piece scan locally.  ONE all_gather.
    Returns the rank's slice of the result.  ops add / min / max."""
    if op not in ("add", "min", "max"):
        raise ValueError("seg_scan_elems: add / min / max")
    be = backend or _default_backend()
    world, rank = _world(group)
    L = seglen
    lo, hi, _, _ = elem_plan(nseg, seglen, rank, world)
    x = x_local.reshape(-1)
    if hi > lo:
        l = (hi - 1) // L
        tail = be.redomap(x[max(lo, l * L) - lo:], op)
    else:
        tail = be.redomap(x[:0], op)
    parts = _gather(tail.reshape(1), world, group).reshape(-1)
    out = torch.empty_like(x)
    if hi == lo:
        return out
    f = lo // L
    head_end = min(hi, (f + 1) * L) - lo  # the piece of row f on this rank
    if lo > f * L:  # row f began on earlier ranks: carry = their partials in rank order
        r0 = _first_rank_of_row(f, nseg, L, world)
        carry = be.combine(parts[r0:rank], op)
        be.scanomap(x[:head_end], op, carry=carry.reshape(1), out=out[:head_end])
        a = head_end
    else:
        a = 0
    if hi - lo > a:  # rows (or a row's first piece) starting inside this rank
        m = hi - lo - a
        nfull, rest = divmod(m, L)
        if nfull:
            be.seg_scan(x[a:a + nfull * L], nfull, L, op, out=out[a:a + nfull * L])
        if rest:
            b = a + nfull * L
            be.scanomap(x[b:], op, out=out[b:])
    return out


# ------------------------------------------------------------------ transpose
def transpose_2d(block, backend=None):
    """Rank r transposes its row block [rows_r][cols]; the result is column block r of
    the global transpose (no exchange)."""
    be = backend or _default_backend()
    return be.transpose_2d(block)


def transpose_2d_global(block, rows: int, cols: int, group=None, backend=None):
    """NEXT-4: rearrange (1,0) of a globally row-sharded matrix X [rows][cols] (rank r holds
    rows shard_range(rows, r, P)) into the row-sharded transpose Y = X^T [cols][rows] (rank r
    returns rows shard_range(cols, r, P) of Y).  Rank r gathers, for every destination p, its
    rows' column block [rows_r][cols_p] (fs_copy_2d), ONE all_to_all exchanges the blocks,
    and the received [rows][cols_r] (all ranks' rows, this rank's columns, in rank order) is
    transposed locally (fs_transpose_2d)."""
    be = backend or _default_backend()
    world, rank = _world(group)
    rlo, rhi = shard_range(rows, rank, world)
    nr = rhi - rlo
    x = block.reshape(-1)
    send = torch.empty(nr * cols, dtype=block.dtype, device=block.device)
    in_split, out_split = [], []
    clo_r, chi_r = shard_range(cols, rank, world)
    off = 0
    for p in range(world):
        clo, chi = shard_range(cols, p, world)
        w = chi - clo
        if nr and w:
            be.copy_2d(x[clo:], nr, w, cols, send[off:], w)
        off += nr * w
        in_split.append(nr * w)
        plo, phi = shard_range(rows, p, world)
        out_split.append((phi - plo) * (chi_r - clo_r))
    recv = torch.empty(sum(out_split), dtype=block.dtype, device=block.device)
    dist.all_to_all_single(recv, send, output_split_sizes=out_split, input_split_sizes=in_split, group=group)
    return be.transpose_2d(recv.reshape(rows, chi_r - clo_r))
