"""Sequential CPU oracle for the libfutseg hot path (numpy in, numpy out).

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this
package.  It shares no code with the CUDA path and never imports it.

Each function is a thin ctypes wrapper over ``oracle/oracle.c``, which is the
plain definition of the SOAC (PAPER.md L125-130 map/reduce/scan; L240-254
fold = reduce . map; Fig 4a L469-471 stream_red counts; footnote 5 L1230-1233
segmented reduce/scan; L1389-1393 transpose).  The readings R1-R5 it takes
where the paper is silent are listed in the C file's header and in DESIGN.md.

Output conventions (match DESIGN.md "Oracle"):
  * f32 ADD results (reduce, scan, vreduce, seg_*, stream_red sums) are f64
    (accumulated in f64, reading R2); everything else keeps the element type.
  * ARGMIN returns ``(values, indices)`` with int64 indices; -1 = empty.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

OPS = {"add": 0, "min": 1, "max": 2, "argmin": 3}
_DT = {np.dtype(np.int32): 0, np.dtype(np.int64): 1, np.dtype(np.float32): 2}
LAYOUTS = {"row": 0, "col": 1}


def build(force: bool = False) -> str:
    """Compile oracle.c with gcc (no fast-math, no FP contraction)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = f"{_LIB}.{os.getpid()}.tmp"  # concurrent builders (spawned test ranks) each replace atomically
        subprocess.check_call([
            "gcc", "-O2", "-ffp-contract=off", "-fno-fast-math", "-std=c11",
            "-shared", "-fPIC", _SRC, "-o", tmp, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def _L():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        P, I, L = ctypes.c_void_p, ctypes.c_int, ctypes.c_int64
        lib.orc_reduce.argtypes = [I, I, P, L, P, P]
        lib.orc_scan.argtypes = [I, I, P, L, P, P]
        lib.orc_nn_dist.argtypes = [P, P, L, ctypes.c_float, ctypes.c_float, P]
        lib.orc_vreduce.argtypes = [I, I, P, L, L, P, P]
        lib.orc_seg_reduce.argtypes = [I, I, P, L, L, I, P, P]
        lib.orc_seg_scan.argtypes = [I, I, P, L, L, I, P, P]
        lib.orc_stream_red.argtypes = [I, P, P, L, L, L, P, P]
        lib.orc_transpose.argtypes = [L, P, L, L, P]
        lib.orc_nn_knn.argtypes = [P, P, L, ctypes.c_float, ctypes.c_float, L, P, P, P, P]
        lib.orc_kmeans_step.argtypes = [P, L, L, P, L, P, P, P, P, P, P]
        lib.orc_seg_map_reduce.argtypes = [I, I, P, L, L, L, ctypes.c_float, P, P, P]
        lib.orc_scan_reduce.argtypes = [I, I, I, P, L, P]
        for f in ("orc_reduce", "orc_scan", "orc_nn_dist", "orc_vreduce", "orc_seg_reduce",
                  "orc_seg_scan", "orc_stream_red", "orc_transpose", "orc_nn_knn", "orc_kmeans_step", "orc_seg_map_reduce", "orc_scan_reduce"):
            getattr(lib, f).restype = I
        _lib = lib
    return _lib


def _p(a):
    return a.ctypes.data_as(ctypes.c_void_p) if a is not None and a.size else None


def _arr(x):
    x = np.ascontiguousarray(x)
    if x.dtype not in _DT:
        raise TypeError(f"oracle: unsupported dtype {x.dtype}")
    return x


def _out_dtype(op, dt):
    return np.float64 if (op == "add" and dt == np.float32) else dt


def _check(rc, what):
    if rc != 0:
        raise ValueError(f"oracle {what}: status {rc}")


def reduce(x, op="add"):
    """reduce (+) 0(+) x  (L128).  Returns a scalar, or (value, index) for argmin."""
    x = _arr(x).reshape(-1)
    out = np.zeros(1, _out_dtype(op, x.dtype))
    idx = np.full(1, -7, np.int64)
    _check(_L().orc_reduce(OPS[op], _DT[x.dtype], _p(x), x.size, _p(out), _p(idx)), "reduce")
    return (out[0], int(idx[0])) if op == "argmin" else out[0]


def scan(x, op="add"):
    """Inclusive scan (+) 0(+) x  (L130)."""
    x = _arr(x).reshape(-1)
    out = np.zeros(x.size, _out_dtype(op, x.dtype))
    idx = np.full(x.size, -7, np.int64)
    _check(_L().orc_scan(OPS[op], _DT[x.dtype], _p(x), x.size, _p(out), _p(idx)), "scan")
    return (out, idx) if op == "argmin" else out


def nn_dist(lat, lng, q0, q1):
    """The NN map f: f32 Euclidean distance to (q0, q1), no FMA contraction (reading R5)."""
    lat = np.ascontiguousarray(lat, np.float32)
    lng = np.ascontiguousarray(lng, np.float32)
    out = np.zeros(lat.size, np.float32)
    _check(_L().orc_nn_dist(_p(lat), _p(lng), lat.size, float(q0), float(q1), _p(out)), "nn_dist")
    return out


def nn_knn(lat, lng, q, kk):
    """NEXT-2: Rodinia NN's kk nearest neighbours as kk rounds of the argmin reduce over
    the distance map, each round excluding its winner (L1653-1655, reading R16).
    Returns (dist[kk] f32, idx[kk] int64); rounds beyond n give (+inf, -1)."""
    lat = np.ascontiguousarray(lat, np.float32)
    lng = np.ascontiguousarray(lng, np.float32)
    n = lat.size
    dist = np.zeros(kk, np.float32)
    idx = np.zeros(kk, np.int64)
    ds = np.zeros(max(n, 1), np.float32)
    ch = np.zeros(max(n, 1), np.uint8)
    _check(_L().orc_nn_knn(_p(lat), _p(lng), n, float(q[0]), float(q[1]), kk, _p(dist), _p(idx), _p(ds), _p(ch)),
           "nn_knn")
    return dist, idx


def kmeans_step(points, centres, prev=None):
    """NEXT-1: one Rodinia K-means iteration (Sec. 2.4; readings R18/R19):
    f32 fma distance argmin (first centre on ties), f64 sums, counts, new centres
    (old centre kept for an empty cluster), delta vs ``prev``.
    Returns (membership[n] i32, sums[k][d] f64, counts[k] i32, new_centres[k][d] f64, delta)."""
    points = np.ascontiguousarray(points, np.float32)
    centres = np.ascontiguousarray(centres, np.float32)
    n, d = points.shape
    k = centres.shape[0]
    assert centres.shape[1] == d
    mem = np.zeros(max(n, 1), np.int32)
    sums = np.zeros((k, d), np.float64)
    counts = np.zeros(k, np.int32)
    newc = np.zeros((k, d), np.float64)
    delta = np.zeros(1, np.int64)
    pv = None if prev is None else np.ascontiguousarray(prev, np.int32)
    _check(_L().orc_kmeans_step(_p(points), n, d, _p(centres), k, _p(pv) if pv is not None else None, _p(mem),
                                _p(sums), _p(counts), _p(newc), _p(delta)), "kmeans_step")
    return mem[:n], sums, counts, newc, int(delta[0])


def redomap(x, op="add", map="id", lng=None, q=(0.0, 0.0)):
    """fold (+,0(+)) f = reduce (+) . map f  (L240-241, L254).  map in {"id", "nn_dist"}."""
    if map == "nn_dist":
        x = nn_dist(x, lng, q[0], q[1])
    return reduce(x, op)


def scanomap(x, op="add", map="id", lng=None, q=(0.0, 0.0)):
    """scan (+) . map f (DESIGN.md reading: "scanomap" by analogy with L254)."""
    if map == "nn_dist":
        x = nn_dist(x, lng, q[0], q[1])
    return scan(x, op)


def vreduce(x, op="add"):
    """reduce (map (+)) (replicate w 0(+)) over a [m][w] array (Fig 4b, G5)."""
    x = _arr(x)
    assert x.ndim == 2
    m, w = x.shape
    out = np.zeros(w, _out_dtype(op, x.dtype))
    idx = np.full(w, -7, np.int64)
    _check(_L().orc_vreduce(OPS[op], _DT[x.dtype], _p(x), m, w, _p(out), _p(idx)), "vreduce")
    return (out, idx) if op == "argmin" else out


def seg_reduce(x, nseg, seglen, op="add", layout="row"):
    """map (reduce (+) 0(+)) over the logical [nseg][seglen] array stored in ``x``."""
    x = _arr(x).reshape(-1)
    assert x.size == nseg * seglen
    out = np.zeros(nseg, _out_dtype(op, x.dtype))
    idx = np.full(nseg, -7, np.int64)
    _check(_L().orc_seg_reduce(OPS[op], _DT[x.dtype], _p(x), nseg, seglen, LAYOUTS[layout],
                               _p(out), _p(idx)), "seg_reduce")
    return (out, idx) if op == "argmin" else out


def seg_map_reduce(x, nseg, seglen, c, op="add"):
    """NEXT-4, L247-252: map (\\row -> (map (+c) row, reduce op row)) over the row-major
    [nseg][seglen] x.  Returns (mapped [nseg*seglen] of x's dtype, reduced [nseg]
    (f64 for f32 add) [, argmin index])."""
    x = _arr(x).reshape(-1)
    assert x.size == nseg * seglen
    mapped = np.zeros(x.size, x.dtype)
    out = np.zeros(nseg, _out_dtype(op, x.dtype))
    idx = np.full(nseg, -7, np.int64)
    ci = int(c) if x.dtype.kind == "i" else 0
    _check(_L().orc_seg_map_reduce(OPS[op], _DT[x.dtype], _p(x), nseg, seglen, ci, float(c), _p(mapped), _p(out),
                                   _p(idx)), "seg_map_reduce")
    return (mapped, out, idx) if op == "argmin" else (mapped, out)


def scan_reduce(x, scan_op="add", red_op="add"):
    """NEXT-3, Fig 10a: reduce red_op (scan scan_op x), the scan materialised (unfused).
    f32 results in f64."""
    x = _arr(x).reshape(-1)
    out = np.zeros(1, np.float64 if x.dtype == np.float32 else x.dtype)
    _check(_L().orc_scan_reduce(OPS[scan_op], OPS[red_op], _DT[x.dtype], _p(x), x.size, _p(out)), "scan_reduce")
    return out[0]


def seg_scan(x, nseg, seglen, op="add", layout="row"):
    """map (scan (+) 0(+)); output has the input's shape and layout (flat)."""
    x = _arr(x).reshape(-1)
    assert x.size == nseg * seglen
    out = np.zeros(x.size, _out_dtype(op, x.dtype))
    idx = np.full(x.size, -7, np.int64)
    _check(_L().orc_seg_scan(OPS[op], _DT[x.dtype], _p(x), nseg, seglen, LAYOUTS[layout],
                             _p(out), _p(idx)), "seg_scan")
    return (out, idx) if op == "argmin" else out


def stream_red(vals, keys, k):
    """K-means centre sums and counts (Fig 4a/4c): returns (sums[k][w], counts[k])."""
    vals = _arr(vals)
    keys = np.ascontiguousarray(keys, np.int32).reshape(-1)
    n = keys.size
    w = vals.shape[1] if vals.ndim == 2 else 0
    assert vals.shape[0] == n
    sums = np.zeros((k, w), _out_dtype("add", vals.dtype))
    counts = np.zeros(k, np.int32)
    _check(_L().orc_stream_red(_DT[vals.dtype], _p(vals), _p(keys), n, w, k, _p(sums), _p(counts)),
           "stream_red")
    return sums, counts


def transpose_2d(x):
    """out[j][i] = in[i][j]  (L1389-1393)."""
    x = np.ascontiguousarray(x)
    r, c = x.shape
    out = np.empty((c, r), x.dtype)
    _check(_L().orc_transpose(x.dtype.itemsize, _p(x), r, c, _p(out)), "transpose")
    return out
