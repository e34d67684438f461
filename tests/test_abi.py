"""C-ABI boundary checks that need no GPU (tier 2).

* the library loads and exports every entry point include/futseg.h declares;
* host-side validation returns the documented status BEFORE any launch
  (null pointers, negative or overflowing sizes, unsupported (op, dtype),
  aliasing outputs, missing / small / misaligned workspace);
* workspace queries and the segment-length regime choice are pure host logic.
No call here reaches a kernel: every argument set is invalid, so the library
must return before touching CUDA.
"""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "futseg.h")


@pytest.fixture(scope="module")
def fs():
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_pldi_henriksenseho17_b200 as m
    return m


def declared_symbols():
    txt = open(HEADER).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"^\s*(?:const\s+)?[\w]+\s*\**\s*(fs_\w+)\s*\(", txt, flags=re.M)))


def test_exports_every_declared_symbol(fs):
    syms = declared_symbols()
    assert len(syms) >= 17, syms
    lib = ctypes.CDLL(fs.library_path())
    missing = [s for s in syms if not hasattr(lib, s)]
    assert not missing, missing


def test_version_and_status_strings(fs):
    assert "sm_100a" in fs.version()
    for s in range(8):
        assert fs.C.fs_status_string(s).decode().startswith("FS_")


OK, NULL, SIZE, UNSUP, ALIAS, WS, CUDA, BOUNDS = range(8)
I32, I64, F32 = 0, 1, 2
FAKE_IN = 0x10000000  # never dereferenced: every call below fails validation
FAKE_OUT = 0x20000000
FAKE_WS = 0x30000000


def op(fs, o, dt, width=1):
    return fs.fs_opdesc(o, dt, width)


def mid(fs, kind=0):
    return fs.fs_mapdesc(kind, 0.0, 0.0, 0)


def P(a):
    return ctypes.c_void_p(a) if a else None


def redomap(fs, o, m, a, b, n, out, idx, ws, wsb):
    return fs.C.fs_redomap(o, m, P(a), P(b), n, P(out), P(idx), P(ws), wsb, None)


def test_redomap_validation(fs):
    big = 1 << 30
    assert redomap(fs, op(fs, 9, I32), mid(fs), FAKE_IN, 0, 10, FAKE_OUT, 0, FAKE_WS, big) == UNSUP
    assert redomap(fs, op(fs, 0, 7), mid(fs), FAKE_IN, 0, 10, FAKE_OUT, 0, FAKE_WS, big) == UNSUP
    assert redomap(fs, op(fs, 0, I32), mid(fs), FAKE_IN, 0, -1, FAKE_OUT, 0, FAKE_WS, big) == SIZE
    assert redomap(fs, op(fs, 0, I32), mid(fs), 0, 0, 10, FAKE_OUT, 0, FAKE_WS, big) == NULL
    assert redomap(fs, op(fs, 0, I32), mid(fs), FAKE_IN, 0, 10, 0, 0, FAKE_WS, big) == NULL
    assert redomap(fs, op(fs, 3, I32), mid(fs), FAKE_IN, 0, 10, FAKE_OUT, 0, FAKE_WS, big) == NULL  # argmin needs idx
    # output inside the input range
    assert redomap(fs, op(fs, 0, I32), mid(fs), FAKE_IN, 0, 10, FAKE_IN + 8, 0, FAKE_WS, big) == ALIAS
    # map NN_DIST requires f32 and two inputs; ID forbids a second input
    assert redomap(fs, op(fs, 0, I32), mid(fs, 1), FAKE_IN, FAKE_IN + 64, 4, FAKE_OUT, 0, FAKE_WS, big) == UNSUP
    assert redomap(fs, op(fs, 0, F32), mid(fs, 1), FAKE_IN, 0, 4, FAKE_OUT, 0, FAKE_WS, big) == NULL
    assert redomap(fs, op(fs, 0, F32), mid(fs), FAKE_IN, FAKE_IN + 64, 4, FAKE_OUT, 0, FAKE_WS, big) == UNSUP
    # workspace missing, too small, misaligned
    assert redomap(fs, op(fs, 0, I32), mid(fs), FAKE_IN, 0, 10, FAKE_OUT, 0, 0, 0) == WS
    assert redomap(fs, op(fs, 0, I32), mid(fs), FAKE_IN, 0, 10, FAKE_OUT, 0, FAKE_WS, 16) == WS
    assert redomap(fs, op(fs, 0, I32), mid(fs), FAKE_IN, 0, 10, FAKE_OUT, 0, FAKE_WS + 4, big) == WS
    # misaligned element pointer
    assert redomap(fs, op(fs, 0, I32), mid(fs), FAKE_IN + 2, 0, 10, FAKE_OUT, 0, FAKE_WS, big) == UNSUP
    # VADD: width must be >= 1 and n*width must not overflow
    assert redomap(fs, op(fs, 4, F32, 0), mid(fs), FAKE_IN, 0, 10, FAKE_OUT, 0, FAKE_WS, big) == SIZE
    assert redomap(fs, op(fs, 4, F32, 1 << 40), mid(fs), FAKE_IN, 0, 1 << 40, FAKE_OUT, 0, FAKE_WS, big) == SIZE


def test_scan_seg_transpose_stream_red_validation(fs):
    big = 1 << 30
    o = op(fs, 0, F32)
    # VADD is not a scan operator
    assert fs.C.fs_scanomap(op(fs, 4, F32, 3), mid(fs), P(FAKE_IN), None, 10, P(FAKE_OUT), None, None, None,
                            P(FAKE_WS), big, None) == UNSUP
    assert fs.C.fs_scanomap(o, mid(fs), P(FAKE_IN), None, 10, P(FAKE_IN + 4), None, None, None, P(FAKE_WS), big,
                            None) == ALIAS
    # argmin carry needs its index
    assert fs.C.fs_scanomap(op(fs, 3, F32), mid(fs), P(FAKE_IN), None, 10, P(FAKE_OUT), P(FAKE_OUT + 4096),
                            P(FAKE_WS + 8192), None, P(FAKE_WS), big, None) == NULL
    # seg: overflow, bad layout, alias, vadd
    assert fs.C.fs_seg_reduce(o, P(FAKE_IN), 1 << 40, 1 << 40, 0, P(FAKE_OUT), None, P(FAKE_WS), big, None) == SIZE
    assert fs.C.fs_seg_reduce(o, P(FAKE_IN), 4, 4, 2, P(FAKE_OUT), None, P(FAKE_WS), big, None) == UNSUP
    assert fs.C.fs_seg_reduce(o, P(FAKE_IN), 4, 4, 0, P(FAKE_IN + 16), None, P(FAKE_WS), big, None) == ALIAS
    assert fs.C.fs_seg_reduce(op(fs, 4, F32, 2), P(FAKE_IN), 4, 4, 0, P(FAKE_OUT), None, P(FAKE_WS), big,
                              None) == UNSUP
    assert fs.C.fs_seg_scan(o, P(FAKE_IN), 4, 4, 1, P(FAKE_IN + 60), None, P(FAKE_WS), big, None) == ALIAS
    assert fs.C.fs_seg_scan(op(fs, 3, I32), P(FAKE_IN), 4, 4, 0, P(FAKE_OUT), None, P(FAKE_WS), big, None) == NULL
    # transpose: in-place is an alias, negative sizes
    assert fs.C.fs_transpose_2d(F32, P(FAKE_IN), 8, 8, P(FAKE_IN), None) == ALIAS
    assert fs.C.fs_transpose_2d(F32, P(FAKE_IN), -1, 8, P(FAKE_OUT), None) == SIZE
    assert fs.C.fs_transpose_2d(9, P(FAKE_IN), 8, 8, P(FAKE_OUT), None) == UNSUP
    assert fs.C.fs_transpose_2d(F32, None, 8, 8, P(FAKE_OUT), None) == NULL
    # stream_red
    assert fs.C.fs_stream_red(F32, P(FAKE_IN), P(FAKE_IN + 4096), 10, 4, 3, P(FAKE_IN + 8), P(FAKE_OUT), P(FAKE_WS),
                              big, None) == ALIAS
    assert fs.C.fs_stream_red(F32, P(FAKE_IN), None, 10, 4, 3, P(FAKE_OUT), P(FAKE_OUT + 4096), P(FAKE_WS), big,
                              None) == NULL
    assert fs.C.fs_stream_red(5, P(FAKE_IN), P(FAKE_IN + 4096), 10, 4, 3, P(FAKE_OUT), None, P(FAKE_WS), big,
                              None) == UNSUP
    assert fs.C.fs_stream_red(F32, P(FAKE_IN), P(FAKE_IN + 4096), 10, 4, 3, P(FAKE_OUT), None, None, 0,
                              None) == WS
    # combine
    assert fs.C.fs_combine(op(fs, 3, F32), P(FAKE_IN), None, 4, P(FAKE_OUT), P(FAKE_OUT + 64), None) == NULL
    assert fs.C.fs_combine(o, P(FAKE_IN), None, 4, P(FAKE_IN), None, None) == ALIAS


def test_nn_knn_validation(fs):
    big = 1 << 30
    f = ctypes.c_float(0.0)
    knn = fs.C.fs_nn_knn
    assert knn(P(FAKE_IN), P(FAKE_IN + 4096), 1000, f, f, 1025, P(FAKE_OUT), P(FAKE_OUT + 8192), P(FAKE_WS), big,
               None) == SIZE                                   # kk > 1024
    assert knn(P(FAKE_IN), P(FAKE_IN + 4096), 1 << 32, f, f, 10, P(FAKE_OUT), P(FAKE_OUT + 8192), P(FAKE_WS), big,
               None) == SIZE                                   # 32-bit record indices
    assert knn(P(FAKE_IN), P(FAKE_IN + 4096), 1000, f, f, -1, P(FAKE_OUT), P(FAKE_OUT + 8192), P(FAKE_WS), big,
               None) == SIZE
    assert knn(P(FAKE_IN), None, 1000, f, f, 10, P(FAKE_OUT), P(FAKE_OUT + 8192), P(FAKE_WS), big, None) == NULL
    assert knn(P(FAKE_IN), P(FAKE_IN + 4096), 1000, f, f, 10, P(FAKE_OUT), None, P(FAKE_WS), big, None) == NULL
    assert knn(P(FAKE_IN), P(FAKE_IN + 4096), 1000, f, f, 10, P(FAKE_IN + 8), P(FAKE_OUT), P(FAKE_WS), big,
               None) == ALIAS                                  # out_dist inside lat
    assert knn(P(FAKE_IN), P(FAKE_IN + 4096), 1000, f, f, 10, P(FAKE_OUT), P(FAKE_OUT + 16), P(FAKE_WS), big,
               None) == ALIAS                                  # out_idx overlaps out_dist
    assert knn(P(FAKE_IN), P(FAKE_IN + 4096), 1000, f, f, 10, P(FAKE_OUT), P(FAKE_OUT + 8192), None, 0,
               None) == WS
    assert knn(None, None, 0, f, f, 0, None, None, None, 0, None) == OK  # kk = 0: nothing to do
    sz = ctypes.c_size_t(0)
    assert fs.C.fs_nn_knn_workspace(855280, 100, ctypes.byref(sz)) == OK and sz.value > 0


def test_kmeans_step_validation(fs):
    big = 1 << 30
    km = fs.C.fs_kmeans_step
    A = lambda o: P(FAKE_OUT + o)
    ok_args = lambda: [P(FAKE_IN), 1000, 34, P(FAKE_IN + (1 << 20)), 32, None, A(0), A(1 << 16), A(1 << 17),
                       A(1 << 18), A(1 << 19), P(FAKE_WS), big, None]
    a = ok_args(); a[4] = 33
    assert km(*a) == UNSUP                                    # k > 32
    a = ok_args(); a[2] = 41
    assert km(*a) == UNSUP                                    # d > 40
    a = ok_args(); a[0] = P(FAKE_IN + 4)
    assert km(*a) == UNSUP                                    # points must be 16-byte aligned (TMA)
    a = ok_args(); a[7] = None
    assert km(*a) == NULL                                     # sums required
    a = ok_args(); a[6] = P(FAKE_IN + 64)
    assert km(*a) == ALIAS                                    # membership inside the points
    a = ok_args(); a[8] = A(1 << 16)
    assert km(*a) == ALIAS                                    # counts on top of sums
    a = ok_args(); a[11] = None; a[12] = 0
    assert km(*a) == WS
    sz = ctypes.c_size_t(0)
    assert fs.C.fs_kmeans_step_workspace(1 << 26, 34, 32, ctypes.byref(sz)) == OK and sz.value > 0
    assert fs.C.fs_kmeans_step_workspace(-1, 34, 32, ctypes.byref(sz)) == SIZE


def test_scan_reduce_validation(fs):
    big = 1 << 30
    sr = fs.C.fs_scan_reduce
    assert sr(1, 0, F32, P(FAKE_IN), 100, P(FAKE_OUT), P(FAKE_WS), big, None) == UNSUP   # scan op must be ADD
    assert sr(0, 3, F32, P(FAKE_IN), 100, P(FAKE_OUT), P(FAKE_WS), big, None) == UNSUP   # no argmin reduce
    assert sr(0, 0, F32, P(FAKE_IN), 100, P(FAKE_IN + 8), P(FAKE_WS), big, None) == ALIAS
    assert sr(0, 0, F32, None, 100, P(FAKE_OUT), P(FAKE_WS), big, None) == NULL
    assert sr(0, 0, F32, P(FAKE_IN), -1, P(FAKE_OUT), P(FAKE_WS), big, None) == SIZE
    assert sr(0, 0, F32, P(FAKE_IN), 100, P(FAKE_OUT), None, 0, None) == WS


def test_workspace_queries_and_regimes(fs):
    sz = ctypes.c_size_t(0)
    assert fs.C.fs_redomap_workspace(op(fs, 0, F32), 1 << 28, ctypes.byref(sz)) == OK and sz.value >= 256
    assert fs.C.fs_scanomap_workspace(op(fs, 3, I64), 1 << 28, ctypes.byref(sz)) == OK
    assert sz.value > (1 << 28) // 2048 * 4  # one status word per tile at least
    assert fs.C.fs_seg_reduce_workspace(op(fs, 0, F32), 4, 1 << 26, 0, ctypes.byref(sz)) == OK
    assert fs.C.fs_stream_red_workspace(F32, 1 << 26, 34, 32, ctypes.byref(sz)) == OK
    assert fs.C.fs_redomap_workspace(op(fs, 0, F32), -5, ctypes.byref(sz)) == SIZE
    assert fs.C.fs_redomap_workspace(op(fs, 0, F32), 5, None) == NULL
    import torch
    r = lambda nseg, L, **kw: fs.seg_regime(nseg, L, **kw)
    assert r(1 << 28, 1) == 0 and r(1 << 22, 64) == 0
    assert r(1 << 20, 256) == 0  # KG0 wide lanes cover powers of two up to 256 (f32)
    assert r(1 << 20, 512) == 1 and r(1 << 20, 1000) == 1 and r(1 << 15, 8192) == 1
    assert r(1 << 13, 1 << 15) == 2
    assert r(4, 1 << 26) == 3 and r(1, 1 << 28) == 3
    assert r(64, 64, layout="col") == 4
    assert r(64, 64, scan=True) == 7 and r(1 << 20, 1024, scan=True) == 7 and r(64, 63, scan=True) == 11
    assert r(1 << 20, 3, scan=True) == 11 and r(1 << 20, 33, scan=True) == 11 and r(64, 7, scan=True, op="argmin") == 5
    assert r(1 << 12, 16384, scan=True) == 9 and r(64, 16384, scan=True) == 5 and r(64, 4092, scan=True) == 11 and r(64, 4100, scan=True) == 5  # KS2: >= 1.7 x SMs rows; the ring above 4096
    assert r(64, 16384, scan=True, op="argmin") == 5 and r(64, 16385, scan=True) == 5
    assert r(1 << 12, 2048, scan=True) == 10 and r(1 << 12, 2048, scan=True, dtype=torch.int64) == 10
    assert r(1 << 12, 8192, scan=True) == 10 and r(1 << 12, 16384, scan=True, dtype=torch.int64) == 9
    assert r(1 << 20, 512, scan=True, dtype=torch.int64) == 7 and r(1 << 20, 1024, scan=True, dtype=torch.int64) == 10
    assert r(1, 1 << 28, scan=True) == 12 and r(2, 1 << 27, scan=True) == 5 and r(1, 5, scan=True) == 12
    assert r(4096, 1000, scan=True, op="argmin") == 5 and r(1 << 21, 128, scan=True, op="argmin") == 7
    assert r(0, 64) == 6 and r(64, 0) == 6
    assert r(64, 64, dtype=torch.int64, op="argmin") == 0
    fs.force_seg_regime(2)
    try:
        assert r(1 << 20, 16) == 2
    finally:
        fs.force_seg_regime(-1)
    assert r(1 << 20, 16) == 0
    for forced, shape, want in ((5, (1 << 20, 1024), 5), (12, (1 << 10, 1024), 12), (11, (1 << 10, 1024), 11),
                                (12, (1 << 20, 3), 11), (8, (1 << 20, 3), 8), (11, (64, 63), 11), (9, (1 << 12, 2048), 10)):
        fs.force_seg_regime(forced)
        try:
            assert r(*shape, scan=True) == want, (forced, shape)
        finally:
            fs.force_seg_regime(-1)
    fs.force_seg_regime(5)
    try:
        assert r(64, 63, scan=True, op="argmin") == 5
    finally:
        fs.force_seg_regime(-1)
    for bad in (-2, 4, 6, 13):
        with pytest.raises(fs.FutsegError):
            fs.force_seg_regime(bad)
    assert fs.last_seg_regime() == -1  # no segmented call has run in this (CPU-only) process


def test_python_layer_refuses_cpu_tensors(fs):
    import torch
    with pytest.raises(ValueError, match="CUDA"):
        fs.redomap(torch.ones(10), "add")
    with pytest.raises(ValueError, match="CUDA"):
        fs.transpose_2d(torch.ones(3, 3))
