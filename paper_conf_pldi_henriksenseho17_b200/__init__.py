"""libfutseg: the B200 hot path of Futhark-compiled code (Henriksen et al., PLDI'17).

Thin Python binding over the C ABI in ``include/futseg.h`` (ctypes, argument
marshalling only -- every step of every primitive runs in the CUDA kernels of
``libfutseg.so``).  PyTorch provides device memory and the current stream.

    import paper_conf_pldi_henriksenseho17_b200 as futseg
    s = futseg.redomap(x, "add")                       # reduce (+) 0 x
    v, i = futseg.redomap(lat, "argmin", map="nn_dist", lng=lng, query=(30., 90.))
    y = futseg.scanomap(x, "max")                      # inclusive scan
    r = futseg.seg_reduce(xss, nseg, seglen, "min", layout="row")
    sums, counts = futseg.stream_red(points, membership, k)
    t = futseg.transpose_2d(m)

Importing fails loudly (ImportError) if the CUDA library has not been built;
every call requires CUDA tensors.  There is no CPU fallback.
"""
from __future__ import annotations

import ctypes
import os

import torch

__all__ = [
    "FutsegError", "redomap", "scanomap", "stream_red", "seg_reduce", "seg_scan", "transpose_2d",
    "combine", "argmin_pack", "argmin_unpack", "partials_pack", "partials_unpack", "copy_2d", "nn_knn", "kmeans_step", "kmeans_finish", "seg_map_reduce", "scan_reduce", "check_device_error", "seg_regime", "last_seg_regime", "force_seg_regime", "library_path", "version",
]

_HERE = os.path.dirname(os.path.abspath(__file__))
# FUTSEG_LIB: an alternative build of the same library (A/B measurement of build variants)
_LIB_PATH = os.environ.get("FUTSEG_LIB") or os.path.join(_HERE, "libfutseg.so")

if not os.path.exists(_LIB_PATH):
    raise ImportError(
        f"libfutseg.so not found at {_LIB_PATH}; build it with "
        "`python paper_conf_pldi_henriksenseho17_b200/build.py` (or __graft_entry__.build())")

_lib = ctypes.CDLL(_LIB_PATH)

FS_I32, FS_I64, FS_F32 = 0, 1, 2
OPS = {"add": 0, "min": 1, "max": 2, "argmin": 3, "vadd": 4}
MAPS = {"id": 0, "nn_dist": 1}
LAYOUTS = {"row": 0, "col": 1}
_DT = {torch.int32: FS_I32, torch.int64: FS_I64, torch.float32: FS_F32}
REGIMES = {0: "KG0/KG1 short rows (shuffle groups / smem tile)", 1: "KG2 warp/segment", 2: "KG3 block/segment",
           3: "KG4 multi-block/segment", 4: "column (col-major)", 5: "segmented look-back scan", 6: "empty",
           7: "KS0 short power-of-two scan (register + shuffle)", 8: "KS1 short-row scan (shared-memory tile)",
           9: "KS2 CTA-per-row scan with a running carry", 10: "KS0-BIG power-of-two rows of 2-8 CTA steps",
           11: "KS3 whole rows staged in shared memory (TMA ring when aligned)", 12: "flat slab scan per row"}


class fs_opdesc(ctypes.Structure):
    _fields_ = [("op", ctypes.c_int32), ("dtype", ctypes.c_int32), ("width", ctypes.c_int64)]


class fs_mapdesc(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int32), ("q0", ctypes.c_float), ("q1", ctypes.c_float), ("ibase", ctypes.c_int64)]


_P, _L, _I, _SZ = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32, ctypes.POINTER(ctypes.c_size_t)
_SIG = {
    "fs_redomap_workspace": [fs_opdesc, _L, _SZ],
    "fs_scanomap_workspace": [fs_opdesc, _L, _SZ],
    "fs_seg_reduce_workspace": [fs_opdesc, _L, _L, _I, _SZ],
    "fs_seg_scan_workspace": [fs_opdesc, _L, _L, _I, _SZ],
    "fs_stream_red_workspace": [_I, _L, _L, _L, _SZ],
    "fs_redomap": [fs_opdesc, fs_mapdesc, _P, _P, _L, _P, _P, _P, ctypes.c_size_t, _P],
    "fs_scanomap": [fs_opdesc, fs_mapdesc, _P, _P, _L, _P, _P, _P, _P, _P, ctypes.c_size_t, _P],
    "fs_combine": [fs_opdesc, _P, _P, _L, _P, _P, _P],
    "fs_stream_red": [_I, _P, _P, _L, _L, _L, _P, _P, _P, ctypes.c_size_t, _P],
    "fs_seg_reduce": [fs_opdesc, _P, _L, _L, _I, _P, _P, _P, ctypes.c_size_t, _P],
    "fs_seg_scan": [fs_opdesc, _P, _L, _L, _I, _P, _P, _P, ctypes.c_size_t, _P],
    "fs_transpose_2d": [_I, _P, _L, _L, _P, _P],
    "fs_nn_knn_workspace": [_L, _L, _SZ],
    "fs_nn_knn": [_P, _P, _L, ctypes.c_float, ctypes.c_float, _L, _P, _P, _P, ctypes.c_size_t, _P],
    "fs_kmeans_step_workspace": [_L, _L, _L, _SZ],
    "fs_kmeans_step": [_P, _L, _L, _P, _L, _P, _P, _P, _P, _P, _P, _P, ctypes.c_size_t, _P],
    "fs_seg_map_reduce_workspace": [fs_opdesc, _L, _L, _SZ],
    "fs_seg_map_reduce": [fs_opdesc, _P, _L, _L, _L, ctypes.c_float, _P, _P, _P, _P, ctypes.c_size_t, _P],
    "fs_scan_reduce_workspace": [_I, _L, _SZ],
    "fs_scan_reduce": [_I, _I, _I, _P, _L, _P, _P, ctypes.c_size_t, _P],
    "fs_kmeans_finish": [_P, _P, _P, _L, _L, _P, _P],
    "fs_check_device_error": [_P, _P],
    "fs_argmin_pack": [_I, _P, _P, _L, _P, _P],
    "fs_argmin_unpack": [_I, _P, _L, _P, _P, _P],
    "fs_partials_pack": [_I, _P, _P, _P, _L, _L, _P, _P],
    "fs_partials_unpack": [_I, _P, _L, _L, _P, _P, _P, _P],
    "fs_copy_2d": [_I, _P, _L, _L, _L, _P, _L, _P],
    "fs_seg_regime": [_I, fs_opdesc, _L, _L, _I],
    "fs_force_seg_regime": [_I],
    "fs_last_seg_regime": [],
    "fs_status_string": [_I],
    "fs_version": [],
    "fs_launch_count": [],
}
for _name, _args in _SIG.items():
    _f = getattr(_lib, _name)
    _f.argtypes = _args
    _f.restype = _I
_lib.fs_status_string.restype = ctypes.c_char_p
_lib.fs_version.restype = ctypes.c_char_p
_lib.fs_launch_count.restype = ctypes.c_uint64

C = _lib  # raw C ABI (ctypes), for callers that manage their own device pointers

# NVTX ranges (tracing): FUTSEG_NVTX=1 wraps every primitive of this module in an
# NVTX range named "futseg.<primitive>" (visible in nsys / ncu --nvtx); off by default so that
# the ~1 us of range push/pop never perturbs a timed region.
_NVTX = os.environ.get("FUTSEG_NVTX", "0") not in ("", "0")


def _traced(fn):
    if not _NVTX:
        return fn
    import functools

    @functools.wraps(fn)
    def wrapper(*args, **kw):
        torch.cuda.nvtx.range_push("futseg." + fn.__name__)
        try:
            return fn(*args, **kw)
        finally:
            torch.cuda.nvtx.range_pop()
    return wrapper


class FutsegError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        super().__init__(f"{where}: {_lib.fs_status_string(status).decode()}")


def _ok(status: int, where: str):
    if status != 0:
        raise FutsegError(status, where)


def library_path() -> str:
    return _LIB_PATH


def version() -> str:
    return _lib.fs_version().decode()


def launch_count() -> int:
    """Kernels launched by libfutseg in this process so far."""
    return int(_lib.fs_launch_count())


# ------------------------------------------------------------------ helpers
def _dev(t: torch.Tensor, name: str) -> torch.Tensor:
    if not isinstance(t, torch.Tensor):
        raise TypeError(f"{name}: expected a torch.Tensor")
    if not t.is_cuda:
        raise ValueError(f"{name}: libfutseg runs on CUDA tensors only (got {t.device}); there is no CPU path")
    if not t.is_contiguous():
        raise ValueError(f"{name}: tensor must be contiguous")
    return t


def _dt(t: torch.Tensor) -> int:
    try:
        return _DT[t.dtype]
    except KeyError:
        raise TypeError(f"unsupported dtype {t.dtype} (int32, int64, float32)") from None


def _ptr(t):
    return None if t is None or t.numel() == 0 else ctypes.c_void_p(t.data_ptr())


def _stream(device) -> ctypes.c_void_p:
    return ctypes.c_void_p(torch.cuda.current_stream(device).cuda_stream)


_ws_cache: dict = {}


def workspace(nbytes: int, device) -> torch.Tensor:
    """Zero-initialised workspace for ``device`` and its current stream (grown on demand)."""
    device = torch.device(device)
    key = (device.index, torch.cuda.current_stream(device).cuda_stream)
    ws = _ws_cache.get(key)
    if ws is None or ws.numel() < nbytes:
        ws = torch.zeros(max(int(nbytes), 1 << 16), dtype=torch.uint8, device=device)
        _ws_cache[key] = ws
    return ws


def _query(fn, *args) -> int:
    sz = ctypes.c_size_t(0)
    _ok(fn(*args, ctypes.byref(sz)), fn.__name__)
    return sz.value


def _op(op: str, dt: int, width: int = 1) -> fs_opdesc:
    if op not in OPS:
        raise ValueError(f"unknown op {op!r}; expected one of {sorted(OPS)}")
    return fs_opdesc(OPS[op], dt, width)


# ------------------------------------------------------------------ primitives
def redomap(x, op: str = "add", map: str = "id", lng=None, query=(0.0, 0.0), ibase: int = 0, out=None, out_idx=None):
    """fold (+, 0(+)) f x = reduce (+) (map f x).

    op in add/min/max/argmin (scalar result) or vadd (x is [n][k] -> [k]).
    map="nn_dist": x = lat, lng = lng (f32), f = distance to ``query``.
    Returns a 0-d tensor, a [k] tensor (vadd) or (value, index) for argmin.
    """
    x = _dev(x, "x")
    dt = _dt(x)
    width = 1
    if op == "vadd":
        if x.dim() != 2:
            raise ValueError("vadd expects a 2-D [n][k] tensor")
        n, width = x.shape
    else:
        n = x.numel()
    o = _op(op, dt, width)
    m = fs_mapdesc(MAPS[map], float(query[0]), float(query[1]), int(ibase))
    if map == "nn_dist":
        lng = _dev(lng, "lng")
        if lng.numel() != n:
            raise ValueError("lat/lng sizes differ")
    if out is None:
        out = torch.empty(width if op == "vadd" else (), dtype=x.dtype, device=x.device)
    if op == "argmin" and out_idx is None:
        out_idx = torch.empty((), dtype=torch.int64, device=x.device)
    ws = workspace(_query(_lib.fs_redomap_workspace, o, n), x.device)
    _ok(_lib.fs_redomap(o, m, _ptr(x), _ptr(lng) if map == "nn_dist" else None, n, ctypes.c_void_p(out.data_ptr()),
                        ctypes.c_void_p(out_idx.data_ptr()) if out_idx is not None else None,
                        ctypes.c_void_p(ws.data_ptr()), ws.numel(), _stream(x.device)), "fs_redomap")
    return (out, out_idx) if op == "argmin" else out


def scanomap(x, op: str = "add", map: str = "id", lng=None, query=(0.0, 0.0), carry=None, carry_idx=None,
             ibase: int = 0, out=None, out_idx=None):
    """out[i] = c (+) f(x0) (+) ... (+) f(xi): the inclusive scan of map f x (L129-130, F5)."""
    x = _dev(x, "x")
    dt = _dt(x)
    n = x.numel()
    o = _op(op, dt)
    m = fs_mapdesc(MAPS[map], float(query[0]), float(query[1]), int(ibase))
    if map == "nn_dist":
        lng = _dev(lng, "lng")
    if out is None:
        out = torch.empty(n, dtype=x.dtype, device=x.device)
    if op == "argmin" and out_idx is None:
        out_idx = torch.empty(n, dtype=torch.int64, device=x.device)
    ws = workspace(_query(_lib.fs_scanomap_workspace, o, n), x.device)
    _ok(_lib.fs_scanomap(o, m, _ptr(x), _ptr(lng) if map == "nn_dist" else None, n, _ptr(out), _ptr(out_idx),
                         _ptr(carry), _ptr(carry_idx), ctypes.c_void_p(ws.data_ptr()), ws.numel(),
                         _stream(x.device)), "fs_scanomap")
    return (out, out_idx) if op == "argmin" else out


def combine(parts, op: str = "add", part_idx=None, width: int = 1, out=None, out_idx=None):
    """parts[0] (+) ... (+) parts[P-1] (the final combine of per-chunk / per-GPU partials)."""
    parts = _dev(parts, "parts")
    dt = _dt(parts)
    P = parts.shape[0] if parts.dim() > 0 else 1
    if op == "vadd":
        width = parts.shape[1]
    o = _op(op, dt, width)
    if out is None:
        out = torch.empty(width if op == "vadd" else (), dtype=parts.dtype, device=parts.device)
    if op == "argmin" and out_idx is None:
        out_idx = torch.empty((), dtype=torch.int64, device=parts.device)
    _ok(_lib.fs_combine(o, _ptr(parts), _ptr(part_idx), P, ctypes.c_void_p(out.data_ptr()),
                        _ptr(out_idx) if out_idx is not None else None, _stream(parts.device)), "fs_combine")
    return (out, out_idx) if op == "argmin" else out


def argmin_pack(values, idx, out=None):
    """ARGMIN partials -> int64 keys whose signed MIN is the R3 argmin (i32 / f32: [n] keys;
    i64: [n][2] (value, index) records for an all_gather).  One collective per exchange."""
    values, idx = _dev(values, "values"), _dev(idx, "idx")
    dt = _dt(values)
    n = values.numel()
    if out is None:
        out = torch.empty((n, 2) if dt == FS_I64 else n, dtype=torch.int64, device=values.device)
    _ok(_lib.fs_argmin_pack(dt, _ptr(values), _ptr(idx), n, _ptr(out), _stream(values.device)), "fs_argmin_pack")
    return out


def argmin_unpack(keys, dtype, P: int = 1, out=None, out_idx=None):
    """The reduced key (i32 / f32, P = 1) or the P gathered records (i64) -> (value, index)."""
    keys = _dev(keys, "keys")
    dt = _DT[dtype]
    if out is None:
        out = torch.empty((), dtype=dtype, device=keys.device)
    if out_idx is None:
        out_idx = torch.empty((), dtype=torch.int64, device=keys.device)
    _ok(_lib.fs_argmin_unpack(dt, _ptr(keys), P, ctypes.c_void_p(out.data_ptr()), ctypes.c_void_p(out_idx.data_ptr()),
                              _stream(keys.device)), "fs_argmin_unpack")
    return out, out_idx


def partials_pack(sums, counts=None, extra=None, out=None):
    """sums [k][w] (+ counts [k], + one extra int64 such as delta) -> ONE buffer of k*w + k + 1
    f64 (f32 sums) or int64 (integer sums) for a single all_reduce SUM."""
    sums = _dev(sums, "sums")
    dt = _dt(sums)
    k, w = (sums.shape[0], sums.shape[1]) if sums.dim() == 2 else (sums.numel(), 1)
    if out is None:
        out = torch.empty(k * w + k + 1, dtype=torch.float64 if dt == FS_F32 else torch.int64, device=sums.device)
    _ok(_lib.fs_partials_pack(dt, _ptr(sums), _ptr(counts), _ptr(extra), k, w, ctypes.c_void_p(out.data_ptr()),
                              _stream(sums.device)), "fs_partials_pack")
    return out


def partials_unpack(packed, sums, counts=None, extra=None):
    """Inverse of partials_pack after the reduction, into the given sums / counts / extra."""
    packed, sums = _dev(packed, "packed"), _dev(sums, "sums")
    dt = _dt(sums)
    k, w = (sums.shape[0], sums.shape[1]) if sums.dim() == 2 else (sums.numel(), 1)
    _ok(_lib.fs_partials_unpack(dt, ctypes.c_void_p(packed.data_ptr()), k, w, _ptr(sums), _ptr(counts), _ptr(extra),
                                _stream(sums.device)), "fs_partials_unpack")
    return sums, counts, extra


def copy_2d(src, rows: int, cols: int, src_ld: int, dst, dst_ld: int):
    """dst[r][c] = src[r][c] for r < rows, c < cols with leading dimensions src_ld / dst_ld
    (elements; tensors are flat views starting at element (0, 0))."""
    src, dst = _dev(src, "src"), _dev(dst, "dst")
    _ok(_lib.fs_copy_2d(src.element_size(), _ptr(src), src_ld, rows, cols, _ptr(dst), dst_ld, _stream(src.device)),
        "fs_copy_2d")
    return dst


def nn_knn(lat, lng, query, kk: int, out_dist=None, out_idx=None):
    """NEXT-2: Rodinia NN's kk nearest neighbours of ``query`` = kk argmin rounds with
    exclusion (L1653-1655): the kk smallest (distance, index) in ascending order, one launch.
    Returns (dist[kk] f32, idx[kk] int64); rounds beyond n give (+inf, -1)."""
    lat = _dev(lat, "lat")
    lng = _dev(lng, "lng")
    if lat.dtype != torch.float32 or lng.dtype != torch.float32 or lat.shape != lng.shape:
        raise TypeError("nn_knn: lat and lng must be float32 tensors of the same shape")
    n = lat.numel()
    if out_dist is None:
        out_dist = torch.empty(kk, dtype=torch.float32, device=lat.device)
    if out_idx is None:
        out_idx = torch.empty(kk, dtype=torch.int64, device=lat.device)
    ws = workspace(_query(_lib.fs_nn_knn_workspace, n, kk), lat.device)
    _ok(_lib.fs_nn_knn(_ptr(lat), _ptr(lng), n, float(query[0]), float(query[1]), kk, _ptr(out_dist), _ptr(out_idx),
                       ctypes.c_void_p(ws.data_ptr()), ws.numel(), _stream(lat.device)), "fs_nn_knn")
    return out_dist, out_idx


def kmeans_step(points, centres, prev=None, membership=None, sums=None, counts=None, new_centres=None,
                delta=None, with_membership: bool = True):
    """NEXT-1: one fused Rodinia K-means iteration (Sec. 2.4; F6 fusion):
    assignment (first centre on ties) + stream_red centre sums/counts + new centres.
    points [n][d] f32 (16-byte aligned), centres [k][d] f32; k <= 32, d <= 40.
    Returns (membership [n] i32 or None, sums [k][d], counts [k], new_centres [k][d],
    delta (1-element int64 tensor; 0 without prev))."""
    points = _dev(points, "points")
    centres = _dev(centres, "centres")
    if points.dtype != torch.float32 or centres.dtype != torch.float32 or points.dim() != 2 or centres.dim() != 2:
        raise TypeError("kmeans_step: points [n][d] and centres [k][d] must be float32 matrices")
    n, d = points.shape
    k = centres.shape[0]
    if centres.shape[1] != d:
        raise ValueError("kmeans_step: centres must have the points' width")
    dev = points.device
    if prev is not None:
        prev = _dev(prev, "prev")
    if membership is None and with_membership:
        membership = torch.empty(n, dtype=torch.int32, device=dev)
    sums = torch.empty((k, d), dtype=torch.float32, device=dev) if sums is None else sums
    counts = torch.empty(k, dtype=torch.int32, device=dev) if counts is None else counts
    new_centres = torch.empty((k, d), dtype=torch.float32, device=dev) if new_centres is None else new_centres
    delta = torch.empty(1, dtype=torch.int64, device=dev) if delta is None else delta
    ws = workspace(_query(_lib.fs_kmeans_step_workspace, n, d, k), dev)
    _ok(_lib.fs_kmeans_step(_ptr(points), n, d, _ptr(centres), k, _ptr(prev), _ptr(membership), _ptr(sums),
                            _ptr(counts), _ptr(new_centres), _ptr(delta), ctypes.c_void_p(ws.data_ptr()), ws.numel(),
                            _stream(dev)), "fs_kmeans_step")
    return membership, sums, counts, new_centres, delta


def seg_map_reduce(x, nseg: int, seglen: int, c, op: str = "add", out_map=None, out=None, out_idx=None):
    """NEXT-4, L247-252: for every row of the row-major [nseg][seglen] x, in one read:
    (map (+c) row, reduce op row).  Returns (mapped [like x], reduced [nseg] [, idx])."""
    x = _dev(x, "x")
    dt = _dt(x)
    if x.numel() != nseg * seglen:
        raise ValueError("seg_map_reduce: x must hold nseg * seglen elements")
    o = _op(op, dt)
    if out_map is None:
        out_map = torch.empty_like(x)
    if out is None:
        out = torch.empty(nseg, dtype=x.dtype, device=x.device)
    if op == "argmin" and out_idx is None:
        out_idx = torch.empty(nseg, dtype=torch.int64, device=x.device)
    ci = int(c) if dt != FS_F32 else 0
    ws = workspace(_query(_lib.fs_seg_map_reduce_workspace, o, nseg, seglen), x.device)
    _ok(_lib.fs_seg_map_reduce(o, _ptr(x), nseg, seglen, ci, float(c), _ptr(out_map), _ptr(out), _ptr(out_idx),
                               ctypes.c_void_p(ws.data_ptr()), ws.numel(), _stream(x.device)), "fs_seg_map_reduce")
    return (out_map, out, out_idx) if op == "argmin" else (out_map, out)


def kmeans_finish(sums, counts, centres, out=None):
    """new centres = sums / counts, an empty cluster keeps its centre (R19)."""
    sums, counts, centres = _dev(sums, "sums"), _dev(counts, "counts"), _dev(centres, "centres")
    k, d = centres.shape
    out = torch.empty_like(centres) if out is None else out
    _ok(_lib.fs_kmeans_finish(_ptr(sums), _ptr(counts), _ptr(centres), k, d, _ptr(out), _stream(sums.device)),
        "fs_kmeans_finish")
    return out


def scan_reduce(x, red: str = "add", scan: str = "add", out=None):
    """NEXT-3, Fig 10c: reduce red (scan (+) x) in one read, the scan never materialised.
    red in add (sum of prefix sums) / max / min (extreme prefix sum)."""
    x = _dev(x, "x")
    dt = _dt(x)
    if out is None:
        out = torch.empty((), dtype=x.dtype, device=x.device)
    ws = workspace(_query(_lib.fs_scan_reduce_workspace, dt, x.numel()), x.device)
    _ok(_lib.fs_scan_reduce(OPS[scan], OPS[red], dt, _ptr(x), x.numel(), _ptr(out), ctypes.c_void_p(ws.data_ptr()),
                            ws.numel(), _stream(x.device)), "fs_scan_reduce")
    return out


def stream_red(vals, keys, k: int, sums=None, counts=None, with_counts: bool = True):
    """K-means centre sums [k][w] and counts [k] as stream_red (map(+)) (Fig 4c)."""
    vals = _dev(vals, "vals")
    keys = _dev(keys, "keys")
    if keys.dtype != torch.int32:
        raise TypeError("keys must be int32")
    dt = _dt(vals)
    n = keys.numel()
    w = vals.shape[1] if vals.dim() == 2 else 0
    if vals.shape[0] != n:
        raise ValueError("vals and keys disagree on n")
    if sums is None:
        sums = torch.empty((k, w), dtype=vals.dtype, device=vals.device)
    if counts is None and with_counts:
        counts = torch.empty(k, dtype=torch.int32, device=vals.device)
    ws = workspace(_query(_lib.fs_stream_red_workspace, dt, n, w, k), vals.device)
    _ok(_lib.fs_stream_red(dt, _ptr(vals), _ptr(keys), n, w, k, _ptr(sums), _ptr(counts),
                           ctypes.c_void_p(ws.data_ptr()), ws.numel(), _stream(vals.device)), "fs_stream_red")
    return sums, counts


def seg_reduce(x, nseg: int, seglen: int, op: str = "add", layout: str = "row", out=None, out_idx=None):
    """out[s] = reduce (+) 0(+) xss[s] over the logical [nseg][seglen] array (footnote 5)."""
    x = _dev(x, "x")
    dt = _dt(x)
    if x.numel() != nseg * seglen:
        raise ValueError("x.numel() != nseg * seglen")
    o = _op(op, dt)
    if out is None:
        out = torch.empty(nseg, dtype=x.dtype, device=x.device)
    if op == "argmin" and out_idx is None:
        out_idx = torch.empty(nseg, dtype=torch.int64, device=x.device)
    ws = workspace(_query(_lib.fs_seg_reduce_workspace, o, nseg, seglen, LAYOUTS[layout]), x.device)
    _ok(_lib.fs_seg_reduce(o, _ptr(x), nseg, seglen, LAYOUTS[layout], _ptr(out), _ptr(out_idx),
                           ctypes.c_void_p(ws.data_ptr()), ws.numel(), _stream(x.device)), "fs_seg_reduce")
    return (out, out_idx) if op == "argmin" else out


def seg_scan(x, nseg: int, seglen: int, op: str = "add", layout: str = "row", out=None, out_idx=None):
    """Inclusive scan of every row of the logical [nseg][seglen] array; same shape and layout."""
    x = _dev(x, "x")
    dt = _dt(x)
    if x.numel() != nseg * seglen:
        raise ValueError("x.numel() != nseg * seglen")
    o = _op(op, dt)
    if out is None:
        out = torch.empty(nseg * seglen, dtype=x.dtype, device=x.device)
    if op == "argmin" and out_idx is None:
        out_idx = torch.empty(nseg * seglen, dtype=torch.int64, device=x.device)
    ws = workspace(_query(_lib.fs_seg_scan_workspace, o, nseg, seglen, LAYOUTS[layout]), x.device)
    _ok(_lib.fs_seg_scan(o, _ptr(x), nseg, seglen, LAYOUTS[layout], _ptr(out), _ptr(out_idx),
                         ctypes.c_void_p(ws.data_ptr()), ws.numel(), _stream(x.device)), "fs_seg_scan")
    return (out, out_idx) if op == "argmin" else out


def transpose_2d(x, out=None):
    """out[j][i] = x[i][j]  (rearrange (1,0), L1389-1393)."""
    x = _dev(x, "x")
    if x.dim() != 2:
        raise ValueError("transpose_2d expects a 2-D tensor")
    r, c = x.shape
    if out is None:
        out = torch.empty((c, r), dtype=x.dtype, device=x.device)
    _ok(_lib.fs_transpose_2d(_dt(x), _ptr(x), r, c, _ptr(out), _stream(x.device)), "fs_transpose_2d")
    return out


def check_device_error(device=None):
    """Synchronise and raise FutsegError(FS_ERR_BOUNDS) if a kernel flagged bad input."""
    device = torch.device(device if device is not None else torch.cuda.current_device())
    ws = workspace(4096, device)
    _ok(_lib.fs_check_device_error(ctypes.c_void_p(ws.data_ptr()), _stream(device)), "fs_check_device_error")


def seg_regime(nseg: int, seglen: int, op: str = "add", dtype=torch.float32, layout: str = "row",
               scan: bool = False) -> int:
    return int(_lib.fs_seg_regime(1 if scan else 0, _op(op, _DT[dtype]), nseg, seglen, LAYOUTS[layout]))


def last_seg_regime() -> int:
    """The regime the last seg_reduce / seg_scan call of this thread launched (include/futseg.h)."""
    return int(_lib.fs_last_seg_regime())


def force_seg_regime(regime: int):
    _ok(_lib.fs_force_seg_regime(int(regime)), "fs_force_seg_regime")


for _name in ("redomap", "scanomap", "combine", "argmin_pack", "argmin_unpack", "partials_pack", "partials_unpack",
              "copy_2d", "nn_knn", "kmeans_step", "kmeans_finish", "seg_map_reduce", "scan_reduce", "stream_red",
              "seg_reduce", "seg_scan", "transpose_2d"):
    globals()[_name] = _traced(globals()[_name])
