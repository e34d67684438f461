#!/usr/bin/env python
"""bench.py -- libfutseg hot-path benchmark (one JSON line on rank 0).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
    python -m torch.distributed.run --nproc-per-node N --master-addr 127.0.0.1 bench.py --gpus N

A STEP is one pass of the whole hot path over one
batch of synthetic input resident in HBM.  At N GPUs the same global problem is
sharded over the ranks (strong scaling, BASELINE.json configs[4]: "k-means
n=2^26 ... sharded by points"; --weak gives every rank a whole problem):

  redomap      f32 add over 2^28 (C4-shaped, 1 GiB)                       A1
  nn_argmin    Rodinia NN argmin redomap, 855,280 (lat,lng) f32 (C2)      A1
  scanomap     f32 add inclusive scan over 2^28                            A2
  stream_red   k-means centre sums+counts, n=2^26, d=34, k=32 (C5)         A3
  seg_reduce   f32 add, 2^28 elements, seglen 32 / 1024 / 65536 / 2^20
               (regimes KG1 / KG2 / KG3 / KG4) and column-major seglen 1024 A4
  seg_scan     f32 add, 2^28 elements, seglen 1024, row-major             A5
  transpose_2d f32 2^14 x 2^14 (C5)                                        A6
  combine      at N > 1: ONE collective per exchange (dist.py): all_reduce
               of the redomap partial, of the packed NN argmin key and of the
               packed k-means sums + counts; all_gather of the scan totals
               for the carries (NCCL over NVLink)                          A7

value = algorithmic bytes of all ranks' steps / max-over-ranks device time
(GB/s, SURVEY.md 8(d) byte counts).  Every input is larger than L2 except
the 6.8 MB NN input, which the ~21 GB the rest of the step streams evicts
between iterations.  See DESIGN.md "Measurement".
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "GB/s and elements/s per primitive (fraction of B200 HBM peak) at 1/2/4/8 GPUs"
GB = 1e9


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


# ------------------------------------------------------------------ clocks
class ClockSampler:
    """Samples SM clock and throttle reasons with NVML while the timed region runs."""

    REASONS = {
        0x0000000000000001: "gpu_idle", 0x0000000000000002: "applications_clocks_setting",
        0x0000000000000004: "sw_power_cap", 0x0000000000000008: "hw_slowdown",
        0x0000000000000020: "sw_thermal_slowdown", 0x0000000000000040: "hw_thermal_slowdown",
        0x0000000000000080: "hw_power_brake_slowdown", 0x0000000000000100: "display_clocks_setting",
    }

    def __init__(self, index: int):
        self.samples, self.reasons, self.max_mhz = [], set(), None
        self._stop = threading.Event()
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:  # noqa: BLE001
            self.nv = None

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                mask = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for bit, name in self.REASONS.items():
                    if mask & bit and name != "gpu_idle":
                        self.reasons.add(name)
            except Exception:  # noqa: BLE001
                pass
            self._stop.wait(0.01)

    def __enter__(self):
        if self.nv:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self.nv:
            self.t.join()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": ["nvml unavailable"]}
        return {"sm_mhz": statistics.median(self.samples), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


# ------------------------------------------------------------------ workload
def build_workload(fs, dev, rank, world, quick, weak=False):
    """The step's inputs on this rank.  Strong scaling (default, BASELINE.json configs[4]: the
    single-GPU problem sharded over the N GPUs): rank r holds shard_range of every global array
    -- its slice of the 2^28 C4 array (= nseg/N whole rows of every seglen), its records of the
    855,280 NN records, its points of the 2^26 k-means points, its [2^14/N][2^14] row block of
    the transpose.  --weak: every rank holds a whole single-GPU problem (seeds offset by rank)."""
    import torch
    import workloads as wl
    from paper_conf_pldi_henriksenseho17_b200.dist import shard_range
    sh = 4 if quick else 0  # --quick: 16x smaller inputs (for harness checks only)
    P, r = (1, 0) if weak else (world, rank)
    ng = (1 << 28) >> sh
    lo, hi = shard_range(ng, r, P)
    n = hi - lo
    W = {}
    W["x"] = wl.device_uniform(n, 5 + 1000 * rank, dev)
    lat, lng, q = wl.c2_nn(seed=2 + (rank if weak else 0))
    nlo, nhi = shard_range(lat.size, r, P)
    W["lat"], W["lng"], W["q"] = torch.from_numpy(lat[nlo:nhi].copy()).to(dev), torch.from_numpy(lng[nlo:nhi].copy()).to(dev), q
    kg = (1 << 26) >> sh
    klo, khi = shard_range(kg, r, P)
    W["pts"], W["mem"] = wl.c5_kmeans_shard(rank, dev, n=khi - klo)
    t = (1 << 14) >> (sh // 2)
    tlo, thi = shard_range(t, r, P)
    W["tmat"] = wl.device_uniform((thi - tlo, t), 6 + 1000 * rank, dev)
    # preallocated outputs (no allocation inside the timed region)
    f32 = dict(dtype=torch.float32, device=dev)
    W["o_red"] = torch.empty((), **f32)
    W["o_nn"] = (torch.empty((), **f32), torch.empty((), dtype=torch.int64, device=dev))
    W["o_scan"] = torch.empty(n, **f32)
    W["o_sums"] = torch.empty((32, 34), **f32)
    W["o_cnt"] = torch.empty(32, dtype=torch.int32, device=dev)
    W["o_segscan"] = torch.empty(n, **f32)
    W["o_tr"] = torch.empty((t, thi - tlo), **f32)
    W["seglens"] = [32, 1024, 65536, 1 << 20]
    W["o_seg"] = {L: torch.empty(n // L, **f32) for L in W["seglens"]}
    W["o_segcol"] = torch.empty(n // 1024, **f32)
    W["n"], W["t"], W["t_rows"] = n, t, thi - tlo
    W["ibase_x"], W["ibase_nn"] = lo, nlo
    W["global"] = {"n": ng, "nn": lat.size, "k": kg, "t": t}
    return W


def make_step(fs, W, world):
    """[(name, fn, algorithmic bytes per rank, elements per rank)] for one step.  At N > 1 the
    combines are the multi-GPU layer's single collectives (dist.py)."""
    from paper_conf_pldi_henriksenseho17_b200 import dist as fdist
    n, t, tr = W["n"], W["t"], W["t_rows"]
    nn = W["lat"].numel()
    kn = W["pts"].shape[0]
    multi = world > 1
    st = []

    def red():
        if multi:
            fdist.redomap(W["x"], "add")  # local fold + ONE all_reduce
        else:
            fs.redomap(W["x"], "add", out=W["o_red"])

    def nn_argmin():
        if multi:  # local argmin + packed key + ONE all_reduce MIN
            fdist.redomap(W["lat"], "argmin", ibase=W["ibase_nn"], map="nn_dist", lng=W["lng"], query=W["q"])
        else:
            fs.redomap(W["lat"], "argmin", map="nn_dist", lng=W["lng"], query=W["q"], out=W["o_nn"][0],
                       out_idx=W["o_nn"][1])

    def scan():
        if multi:
            fdist.scanomap(W["x"], "add")  # local total + ONE all_gather + carry-in scan
        else:
            fs.scanomap(W["x"], "add", out=W["o_scan"])

    def kmeans():
        if multi:
            fdist.stream_red(W["pts"], W["mem"], 32)  # packed sums + counts, ONE all_reduce
        else:
            fs.stream_red(W["pts"], W["mem"], 32, sums=W["o_sums"], counts=W["o_cnt"])

    st.append(("redomap_f32_add", red, 4 * n, n))
    st.append(("nn_argmin_redomap", nn_argmin, 8 * nn, nn))
    st.append(("scanomap_f32_add", scan, 8 * n, n))
    st.append(("stream_red_kmeans_k32_d34", kmeans, (4 * 34 + 4) * kn, kn))
    for L in W["seglens"]:
        st.append((f"seg_reduce_row_L{L}",
                   (lambda L=L: fs.seg_reduce(W["x"], n // L, L, "add", out=W["o_seg"][L])),
                   4 * n + 4 * (n // L), n))
    st.append(("seg_reduce_col_L1024", lambda: fs.seg_reduce(W["x"], n // 1024, 1024, "add", layout="col",
                                                             out=W["o_segcol"]), 4 * n + 4 * (n // 1024), n))
    st.append(("seg_scan_row_L1024", lambda: fs.seg_scan(W["x"], n // 1024, 1024, "add", out=W["o_segscan"]),
               8 * n, n))
    st.append(("transpose_2d_f32", lambda: fs.transpose_2d(W["tmat"], out=W["o_tr"]), 8 * t * tr, t * tr))
    return st


# ------------------------------------------------------------------ SURVEY 8(f) "next" rows
def time_next_rows(fs, W, dev, K, peak):
    """Each NEXT row timed on its own (one warm-up call, then CUDA events over K reps, L2
    flushed before every rep by READING a 1 GB buffer outside the events -- a write flush
    would leave ~126 MB of dirty lines for the timed kernel to write back; median and min).
    Not part of the step value (8(a) rows only)."""
    import torch
    flush = torch.ones(1 << 28, dtype=torch.float32, device=dev)  # 1 GB: ~160 us of reads, the host stays ahead
    rows = {}

    def timed(fn, reps=K):
        fn()  # warm-up: workspace growth, function attributes
        ms = []
        for _ in range(reps):
            torch.amax(flush)  # evict by READING 1 GB: no dirty lines left to write back
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            fn()
            b.record()
            b.synchronize()
            ms.append(a.elapsed_time(b))
        return statistics.median(ms), min(ms)

    # NEXT-2: NN's 100 argmin rounds (L1653-1655) as one selection launch
    nn, kk = W["lat"].numel(), 100
    od = torch.empty(kk, dtype=torch.float32, device=dev)
    oi = torch.empty(kk, dtype=torch.int64, device=dev)
    l0 = fs.launch_count()
    avg, mn = timed(lambda: fs.nn_knn(W["lat"], W["lng"], W["q"], kk, out_dist=od, out_idx=oi))
    launches = (fs.launch_count() - l0) // K
    # the paper's structure for reference: kk argmin-redomap launches back to back (the
    # exclusion step between rounds not even counted) -- what "dominated by frequent
    # launches of short kernels" (L1655-1656) costs on this GPU
    o1, o2 = W["o_nn"]
    avg_r, _ = timed(lambda: [fs.redomap(W["lat"], "argmin", map="nn_dist", lng=W["lng"], query=W["q"],
                                         out=o1, out_idx=o2) for _ in range(kk)], reps=max(3, K // 4))
    b = 8 * nn
    rows["nn_knn_k100_c2"] = {"ms": round(avg, 4), "ms_min": round(mn, 4), "GB_s": round(b / (avg * 1e-3) / GB, 1),
                              "elements_per_s": float(f"{nn / (avg * 1e-3):.4g}"), "bytes": b,
                              "frac_of_peak": round(b / (avg * 1e-3) / GB / peak, 4), "launches": launches,
                              "vs_100_argmin_launches_ms": round(avg_r, 4),
                              "note": "C2 records (L2-flushed, cold); bit-exact vs 100 oracle argmin rounds"}
    # NEXT-1: one fused K-means iteration at C5 (n = 2^26, d = 34, k = 32): assignment on the
    # tensor cores (TF32, certified exact) + stream_red centre update + new centres + delta
    pts = W["pts"]
    kn, d = pts.shape
    g = torch.Generator(device=dev).manual_seed(77)
    cen = pts[torch.randint(0, kn, (32,), device=dev, generator=g)].clone()
    prev = W["mem"]
    mem = torch.empty(kn, dtype=torch.int32, device=dev)
    sums = torch.empty((32, d), dtype=torch.float32, device=dev)
    cnt = torch.empty(32, dtype=torch.int32, device=dev)
    newc = torch.empty((32, d), dtype=torch.float32, device=dev)
    dl = torch.empty(1, dtype=torch.int64, device=dev)
    avg, mn = timed(lambda: fs.kmeans_step(pts, cen, prev=prev, membership=mem, sums=sums, counts=cnt,
                                           new_centres=newc, delta=dl))
    b = kn * (4 * d + 4 + 4)  # points + prev membership in, new membership out
    flops = 2.0 * kn * 32 * d  # the x.c contraction (what the tensor cores do)
    rows["kmeans_step_c5_k32_d34"] = {"ms": round(avg, 4), "ms_min": round(mn, 4),
                                      "GB_s": round(b / (avg * 1e-3) / GB, 1),
                                      "elements_per_s": float(f"{kn / (avg * 1e-3):.4g}"), "bytes": b,
                                      "frac_of_peak": round(b / (avg * 1e-3) / GB / peak, 4),
                                      "tflops_tf32": round(flops / (avg * 1e-3) / 1e12, 1),
                                      "note": "fused assignment (mma.sync TF32 + exact near-tie re-evaluation) + "
                                              "stream_red + new centres + delta; membership bit-exact vs f32 oracle"}
    # NEXT-3: Fig 10c's fused stream_seq, reduce (scan x) in one read (2^28 f32, C4), vs
    # the unfused program (scanomap materialised, then redomap)
    x, n = W["x"], W["n"]
    o1 = torch.empty((), dtype=torch.float32, device=dev)
    for red in ("add", "max"):
        avg, mn = timed(lambda: fs.scan_reduce(x, red, out=o1))
        avg_u, _ = timed(lambda: fs.redomap(fs.scanomap(x, "add", out=W["o_scan"]), red, out=o1))
        b = 4 * n
        rows[f"scan_reduce_{red}_2^28"] = {"ms": round(avg, 4), "ms_min": round(mn, 4),
                                          "GB_s": round(b / (avg * 1e-3) / GB, 1),
                                          "elements_per_s": float(f"{n / (avg * 1e-3):.4g}"), "bytes": b,
                                          "frac_of_peak": round(b / (avg * 1e-3) / GB / peak, 4),
                                          "vs_unfused_scan_then_reduce_ms": round(avg_u, 4)}
    # NEXT-4: the L247-252 row nest (map (+1.0) row, reduce (+) row) over the C5 matrix
    # [2^14][2^14] f32 and over C4 rows [2^18][1024]: one read, two outputs
    for name, xm, nseg, L in (("seg_map_reduce_2^14x2^14", W["tmat"], W["t"], W["t"]),
                              ("seg_map_reduce_2^18x1024", W["x"], W["n"] // 1024, 1024)):
        om = torch.empty_like(xm)
        orow = torch.empty(nseg, dtype=torch.float32, device=dev)
        avg, mn = timed(lambda: fs.seg_map_reduce(xm, nseg, L, 1.0, "add", out_map=om, out=orow))
        b = 8 * nseg * L + 4 * nseg
        rows[name] = {"ms": round(avg, 4), "ms_min": round(mn, 4), "GB_s": round(b / (avg * 1e-3) / GB, 1),
                      "elements_per_s": float(f"{nseg * L / (avg * 1e-3):.4g}"), "bytes": b,
                      "frac_of_peak": round(b / (avg * 1e-3) / GB / peak, 4),
                      "note": "x read once; x + 1.0 written and every row summed"}
        del om
    # BASELINE configs[0] (C1): i32 sum over 2^20 full-range values (wraps) and the 1024 x 1024
    # seg_reduce; configs[2] (C3): the kdd_cup shape n = 494,019, d = 34, k = 5, stream_red and the
    # fused kmeans_step -- small inputs (L2-resident), so cold (L2 flushed by reading 1 GB) and warm
    # (inputs just read, in L2) are both reported; latency-bound, elements/s is the useful figure
    import numpy as np
    import workloads as wl
    x1 = torch.from_numpy(wl.c1()).to(dev)
    o1 = torch.empty((), dtype=torch.int32, device=dev)
    oseg = torch.empty(1024, dtype=torch.int32, device=dev)
    pts3, mem3 = wl.c3_kmeans(keys="clustered")
    P3, M3 = torch.from_numpy(pts3).to(dev), torch.from_numpy(mem3).to(dev)
    cen3 = P3[:5].clone()
    sums3 = torch.empty((5, 34), dtype=torch.float32, device=dev)
    cnt3 = torch.empty(5, dtype=torch.int32, device=dev)
    km3 = [torch.empty(P3.shape[0], dtype=torch.int32, device=dev), torch.empty((5, 34), dtype=torch.float32, device=dev),
           torch.empty(5, dtype=torch.int32, device=dev), torch.empty((5, 34), dtype=torch.float32, device=dev),
           torch.empty(1, dtype=torch.int64, device=dev)]

    def warm_timed(fn, reps=max(K, 5), inner=20):
        """Warm: the inputs stay in L2 and the calls are enqueued back to back (inner per event
        pair), so the host's per-call overhead is hidden behind the GPU work as in a pipeline."""
        fn()
        ms = []
        for _ in range(reps):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            for _ in range(inner):
                fn()
            b.record()
            b.synchronize()
            ms.append(a.elapsed_time(b) / inner)
        return statistics.median(ms), min(ms)

    nk = P3.shape[0]
    for name, fn, b, el in (
            ("c1_redomap_i32_add_2^20", lambda: fs.redomap(x1, "add", out=o1), 4 << 20, 1 << 20),
            ("c1_seg_reduce_i32_add_1024x1024", lambda: fs.seg_reduce(x1, 1024, 1024, "add", out=oseg),
             (4 << 20) + 4096, 1 << 20),
            ("c3_stream_red_kdd_k5_d34", lambda: fs.stream_red(P3, M3, 5, sums=sums3, counts=cnt3), nk * 140, nk),
            ("c3_kmeans_step_kdd_k5_d34", lambda: fs.kmeans_step(P3, cen3, prev=M3, membership=km3[0], sums=km3[1],
                                                                  counts=km3[2], new_centres=km3[3], delta=km3[4]),
             nk * 144, nk)):
        cold, cmin = timed(fn)
        warm, wmin = warm_timed(fn)
        rows[name] = {"ms_cold": round(cold, 4), "ms_warm": round(warm, 4), "ms_min_warm": round(wmin, 4),
                      "elements_per_s_cold": float(f"{el / (cold * 1e-3):.4g}"),
                      "elements_per_s_warm": float(f"{el / (warm * 1e-3):.4g}"), "bytes": b,
                      "GB_s_cold": round(b / (cold * 1e-3) / GB, 1), "GB_s_warm": round(b / (warm * 1e-3) / GB, 1),
                      "note": "BASELINE configs[0]/[2]: small, L2-resident -> latency-bound; bit-exact integers"}
    return rows


# ------------------------------------------------------------------ cpu baseline (oracle)
def oracle_sample(W, scale_shift):
    """Host copies of a bounded sample of every primitive's input (same data as the GPU run)."""
    s = {}
    m = min(W["n"], (1 << 26) >> scale_shift)
    s["x"] = W["x"][:m].cpu().numpy()
    s["lat"], s["lng"] = W["lat"].cpu().numpy(), W["lng"].cpu().numpy()
    kr = min(W["pts"].shape[0], (1 << 22) >> scale_shift)
    s["pts"], s["mem"] = W["pts"][:kr].cpu().numpy(), W["mem"][:kr].cpu().numpy()
    tt = min(W["t"], 4096 >> (scale_shift // 2))
    s["tmat"] = W["tmat"][:tt, :tt].cpu().numpy()
    return s


def oracle_step(s, q):
    """One pass of the oracle over the sample; returns (algorithmic bytes, seconds)."""
    import oracle
    x = s["x"]
    m = x.size
    t0 = time.perf_counter()
    oracle.reduce(x, "add")
    oracle.redomap(s["lat"], "argmin", "nn_dist", s["lng"], q)
    oracle.scan(x, "add")
    oracle.stream_red(s["pts"], s["mem"], 32)
    for L in (32, 1024, 65536):
        oracle.seg_reduce(x, m // L, L, "add")
    oracle.seg_reduce(x, m // 1024, 1024, "add", "col")
    oracle.seg_scan(x, m // 1024, 1024, "add")
    oracle.transpose_2d(s["tmat"])
    dt = time.perf_counter() - t0
    kr = s["mem"].size
    tt = s["tmat"].shape[0]
    nbytes = (4 * m + 8 * s["lat"].size + 8 * m + 140 * kr + 3 * (4 * m) + sum(4 * (m // L) for L in (32, 1024, 65536))
              + 4 * m + 4 * (m // 1024) + 8 * m + 8 * tt * tt)
    return nbytes, dt, f"{m} f32 (redomap, scan, seg ops L=32/1024/65536/col, seg_scan), NN {s['lat'].size} " \
                       f"records, k-means {kr}x34 k=32, transpose {tt}x{tt}"


def host_cpu():
    """The host's CPU model and core count (recorded beside the oracle baseline)."""
    model = "unknown"
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    model = line.split(":", 1)[1].strip()
                    break
    except OSError:
        pass
    return model, os.cpu_count() or 1


def oracle_step_allcores(s, q, threads):
    """The same bounded sample as oracle_step, split over ``threads`` host threads: every
    primitive's independent units (array chunks, rows, points, records, row blocks) are divided
    into contiguous pieces and each piece runs the unmodified oracle concurrently (the ctypes
    calls release the GIL) -- stream_red semantics with s = #cores; the few-element
    combine of the pieces' results is not timed work of note.  Returns (bytes, seconds)."""
    import concurrent.futures as cf
    import oracle
    x = s["x"]
    m = x.size
    tt = s["tmat"].shape[0]

    def pieces(n, unit=1):
        k = max(1, min(threads, n // max(unit, 1)))
        step = -(-n // k)
        step = -(-step // unit) * unit
        return [(a, min(n, a + step)) for a in range(0, n, step)]

    jobs = []
    for a, b in pieces(m):
        jobs.append(lambda a=a, b=b: oracle.reduce(x[a:b], "add"))
        jobs.append(lambda a=a, b=b: oracle.scan(x[a:b], "add"))
    for a, b in pieces(s["lat"].size):
        jobs.append(lambda a=a, b=b: oracle.redomap(s["lat"][a:b], "argmin", "nn_dist", s["lng"][a:b], q))
    for a, b in pieces(s["mem"].size):
        jobs.append(lambda a=a, b=b: oracle.stream_red(s["pts"][a:b], s["mem"][a:b], 32))
    for L in (32, 1024, 65536):
        for a, b in pieces(m, L):
            jobs.append(lambda a=a, b=b, L=L: oracle.seg_reduce(x[a:b], (b - a) // L, L, "add"))
    for a, b in pieces(m, 1024):
        jobs.append(lambda a=a, b=b: oracle.seg_reduce(x[a:b], (b - a) // 1024, 1024, "add", "col"))
        jobs.append(lambda a=a, b=b: oracle.seg_scan(x[a:b], (b - a) // 1024, 1024, "add"))
    for a, b in pieces(tt):
        jobs.append(lambda a=a, b=b: oracle.transpose_2d(s["tmat"][a:b]))
    t0 = time.perf_counter()
    with cf.ThreadPoolExecutor(max_workers=threads) as ex:
        list(ex.map(lambda f: f(), jobs))
    dt = time.perf_counter() - t0
    kr = s["mem"].size
    nbytes = (4 * m + 8 * s["lat"].size + 8 * m + 140 * kr + 3 * (4 * m) + sum(4 * (m // L) for L in (32, 1024, 65536))
              + 4 * m + 4 * (m // 1024) + 8 * m + 8 * tt * tt)
    return nbytes, dt


def run_reference(args):
    """--impl reference: the oracle (the only reference this tier has), timed on host cores."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import numpy as np
    import torch
    import workloads as wl
    dev = "cuda" if torch.cuda.is_available() else "cpu"
    W = {"x": wl.device_uniform(1 << 23, 5, dev), "lat": None}
    lat, lng, q = wl.c2_nn(seed=2)
    W["lat"], W["lng"] = torch.from_numpy(lat), torch.from_numpy(lng)
    W["pts"], W["mem"] = wl.c5_kmeans_shard(0, dev, n=1 << 19)
    W["tmat"] = wl.device_uniform((2048, 2048), 6, dev)
    W["n"], W["t"] = 1 << 23, 2048
    s = oracle_sample(W, 0)
    model, ncpu = host_cpu()
    _, _, desc = oracle_step(s, q)  # (also the single-core warm-up)
    for _ in range(args.warmup):
        oracle_step_allcores(s, q, ncpu)
    tot_b, tot_t = 0, 0.0
    for _ in range(args.steps):
        b, dt = oracle_step_allcores(s, q, ncpu)
        tot_b += b
        tot_t += dt
    val = tot_b / tot_t / GB
    b1, dt1, _ = oracle_step(s, q)
    line = {"impl": "reference", "metric": METRIC, "value": round(val, 4), "unit": "GB/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(1e3 * tot_t / args.steps, 3),
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64-accumulated (f32 in)",
            "data": "synthetic",
            "config": {"workload": "libfutseg hot-path suite (bounded oracle sample per step)", "sample": desc},
            "cpu_baseline": {"value": round(val, 4), "unit": "GB/s", "cores": ncpu, "cpu_model": model,
                             "kind": "oracle, chunked over the host cores (stream_red semantics, s = #cores)",
                             "sample": desc, "single_core": {"value": round(b1 / dt1 / GB, 4), "cores": 1}},
            "e2e": {"value": round(val, 4), "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------ main
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--quick", action="store_true", help="16x smaller inputs (harness check; not a bench value)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=4)
    ap.add_argument("--only", default="", help="comma-separated primitive names (profiling aid)")
    ap.add_argument("--no-next", action="store_true", help="skip the SURVEY 8(f) next-row measurements")
    ap.add_argument("--weak", action="store_true", help="N > 1: every rank runs a whole single-GPU problem")
    args = ap.parse_args()
    if args.warmup < 3 and not args.quick and not args.only:
        print("bench.py: --warmup must be >= 3", file=sys.stderr)
        args.warmup = 3
    if args.impl == "reference":
        return run_reference(args)

    import torch
    import torch.distributed as tdist
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        print(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world}; launch N>1 with torch.distributed.run",
              file=sys.stderr)
        sys.exit(2)
    # FUTSEG_BENCH_DEVICE0=1 + FUTSEG_BENCH_BACKEND=gloo: every rank on cuda:0 over gloo -- a
    # functional check of the N > 1 path on a one-GPU box (not a performance number)
    if os.environ.get("FUTSEG_BENCH_DEVICE0") == "1":
        local = 0
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        backend = os.environ.get("FUTSEG_BENCH_BACKEND", "nccl")
        if backend == "nccl":
            tdist.init_process_group("nccl", device_id=dev)
        else:
            tdist.init_process_group(backend)
    import paper_conf_pldi_henriksenseho17_b200 as fs

    W = build_workload(fs, dev, rank, world, args.quick, weak=args.weak)
    steps = make_step(fs, W, world)
    if args.only:
        keep = set(args.only.split(","))
        steps = [s for s in steps if s[0] in keep]
    names = [s[0] for s in steps]

    def barrier():
        if world > 1:
            tdist.barrier()
        torch.cuda.synchronize()

    for _ in range(args.warmup):
        for _, fn, _, _ in steps:
            fn()
    barrier()

    K = args.steps
    ev = [[(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in steps]
          for _ in range(K)]
    start, end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    l0 = fs.launch_count()
    with ClockSampler(local) as clk:
        barrier()
        start.record()
        for s in range(K):
            for p, (_, fn, _, _) in enumerate(steps):
                ev[s][p][0].record()
                fn()
                ev[s][p][1].record()
        end.record()
        barrier()
    launches = fs.launch_count() - l0
    total_ms = start.elapsed_time(end)
    tmax = torch.tensor([total_ms], device=dev, dtype=torch.float64)
    if world > 1:
        tdist.all_reduce(tmax, op=tdist.ReduceOp.MAX)
    total_ms = float(tmax.item())
    per = {}
    for p, (name, _, nbytes, nel) in enumerate(steps):
        ms = [ev[s][p][0].elapsed_time(ev[s][p][1]) for s in range(K)]
        avg = sum(ms) / K
        per[name] = {"ms": round(avg, 4), "ms_min": round(min(ms), 4), "GB_s": round(nbytes / (avg * 1e-3) / GB, 1),
                     "elements_per_s": float(f"{nel / (avg * 1e-3):.4g}"), "bytes": nbytes}
    step_bytes = sum(s[2] for s in steps)
    step_elems = sum(s[3] for s in steps)
    tot = torch.tensor([step_bytes, step_elems], device=dev, dtype=torch.float64)
    if world > 1:
        tdist.all_reduce(tot)  # the whole job's bytes (strong: the global problem; weak: N problems)
    job_bytes, job_elems = float(tot[0].item()), float(tot[1].item())
    value = job_bytes * K / (total_ms * 1e-3) / GB
    peak, peak_src = peaks()
    for name in per:
        per[name]["frac_of_peak"] = round(per[name]["GB_s"] / peak, 4)
    dom = max(per, key=lambda k: per[k]["ms"])
    traffic = None
    tf = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(tf):
        with open(tf) as f:
            t = json.load(f).get(dom)
        traffic = t.get("traffic_bytes_per_launch") if isinstance(t, dict) else t

    # ---------------- e2e: host buffers, H2D + compute + D2H inside the timed region
    e2e = None
    if not args.no_e2e and not args.only:
        host_in = {k: W[k].cpu().pin_memory() for k in ("x", "lat", "lng", "pts", "mem", "tmat")}
        outs = [W["o_red"], W["o_nn"][0], W["o_nn"][1], W["o_scan"], W["o_sums"], W["o_cnt"], W["o_segscan"],
                W["o_tr"], W["o_segcol"]] + list(W["o_seg"].values())
        host_out = [torch.empty(o.shape, dtype=o.dtype, pin_memory=True) for o in outs]
        h2d = sum(v.numel() * v.element_size() for v in host_in.values())
        d2h = sum(o.numel() * o.element_size() for o in outs)
        KE = max(1, args.e2e_steps)
        # Pipelined through three streams, as a user of the API would run it: H2D copies (in the
        # order the step consumes them), the primitives (each waits for its own inputs), D2H
        # copies (each output as soon as its primitive is done).  PCIe is full duplex, so the
        # outputs leave while the next inputs arrive.  Buffers are reused across steps: an input
        # copy waits for the previous step's last reader, a step's compute for the previous
        # step's output copies.
        comp = torch.cuda.current_stream(dev)
        s_in, s_out = torch.cuda.Stream(dev), torch.cuda.Stream(dev)
        by_name = {name: fn for name, fn, _, _ in steps}
        needs = {"nn_argmin_redomap": ("lat", "lng"), "stream_red_kmeans_k32_d34": ("pts", "mem"),
                 "transpose_2d_f32": ("tmat",)}
        produces = {"redomap_f32_add": [W["o_red"]], "nn_argmin_redomap": list(W["o_nn"]),
                    "scanomap_f32_add": [W["o_scan"]], "stream_red_kmeans_k32_d34": [W["o_sums"], W["o_cnt"]],
                    "seg_reduce_col_L1024": [W["o_segcol"]], "seg_scan_row_L1024": [W["o_segscan"]],
                    "transpose_2d_f32": [W["o_tr"]]}
        for L in W["seglens"]:
            produces[f"seg_reduce_row_L{L}"] = [W["o_seg"][L]]
        h_of = {id(o): h for o, h in zip(outs, host_out)}
        order_in = ["lat", "lng", "x", "pts", "mem", "tmat"]
        order_run = ["nn_argmin_redomap"] + [nm for nm in by_name if nm not in needs] + \
                    ["stream_red_kmeans_k32_d34", "transpose_2d_f32"]
        barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(comp)
        s_in.wait_stream(comp)
        s_out.wait_stream(comp)
        last_read = {}
        out_done = None
        for _ in range(KE):
            arrived = {}
            with torch.cuda.stream(s_in):
                for k in order_in:
                    if k in last_read:
                        s_in.wait_event(last_read[k])
                    W[k].copy_(host_in[k], non_blocking=True)
                    arrived[k] = torch.cuda.Event()
                    arrived[k].record(s_in)
            if out_done is not None:
                comp.wait_event(out_done)
            for nm in order_run:
                for k in needs.get(nm, ("x",)):
                    comp.wait_event(arrived[k])
                by_name[nm]()
                ev = torch.cuda.Event()
                ev.record(comp)
                for k in needs.get(nm, ("x",)):
                    last_read[k] = ev
                s_out.wait_event(ev)
                with torch.cuda.stream(s_out):
                    for o in produces[nm]:
                        h_of[id(o)].copy_(o, non_blocking=True)
            out_done = torch.cuda.Event()
            out_done.record(s_out)
        comp.wait_stream(s_out)
        comp.wait_stream(s_in)
        e1.record(comp)
        barrier()
        ems = torch.tensor([e0.elapsed_time(e1)], device=dev, dtype=torch.float64)
        if world > 1:
            tdist.all_reduce(ems, op=tdist.ReduceOp.MAX)
        e2e = {"value": round(job_bytes * KE / (float(ems.item()) * 1e-3) / GB, 2), "unit": "GB/s",
               "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h, "steps": KE,
               "note": "same algorithmic bytes; pinned host inputs copied in and all outputs copied out every step, "
                       "H2D / compute / D2H on three streams (each primitive waits for its own inputs, each output "
                       "leaves as soon as it is ready)"}

    # ---------------- SURVEY 8(f) next rows (single GPU, own timing; not in the step value)
    nxt = None
    if rank == 0 and world == 1 and not args.no_next and not args.only and not args.quick:
        nxt = time_next_rows(fs, W, dev, max(K, 5), peak)

    # ---------------- cpu baseline: the oracle on a bounded sample, rank 0, N = 1
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline and not args.only:
        s = oracle_sample(W, 4 if args.quick else 0)
        b, dt, desc = oracle_step(s, W["q"])
        model, ncpu = host_cpu()
        b2, dt2 = oracle_step_allcores(s, W["q"], ncpu)
        cpu = {"value": round(b / dt / GB, 4), "unit": "GB/s", "cores": 1, "kind": "oracle",
               "sample": desc, "seconds": round(dt, 2), "cpu_model": model, "nproc": ncpu,
               "all_cores": {"value": round(b2 / dt2 / GB, 4), "unit": "GB/s", "cores": ncpu,
                             "kind": "oracle, chunked over the host cores (stream_red semantics, s = #cores)",
                             "seconds": round(dt2, 2)}}

    if rank == 0:
        line = {
            "metric": METRIC, "value": round(value, 2), "unit": "GB/s", "n_gpus": world, "steps": K,
            "warmup": args.warmup, "ms_per_step": round(total_ms / K, 4), "higher_is_better": True,
            "scaling": "weak" if (args.weak and world > 1) else "strong", "vs_baseline": None, "dtype": "f32",
            "data": "synthetic",
            "config": {"workload": "libfutseg hot-path suite: redomap 2^28 f32, NN argmin 855,280 (C2), scanomap 2^28, "
                                   "k-means stream_red 2^26x34 k=32 (C5), seg_reduce 2^28 L=32/1024/65536/2^20 row + "
                                   "L=1024 col, seg_scan 2^28 L=1024, transpose 2^14^2 f32 (C5)" +
                                   (" [QUICK 1/16 sizes]" if args.quick else ""),
                       "per_rank_bytes_per_step": step_bytes, "per_rank_elements_per_step": step_elems,
                       "l2": "inputs > L2 (126 MB) except NN (6.8 MB), evicted by the ~21 GB rest of each step",
                       "parallelism": (f"dp{world} (weak: a whole single-GPU problem per GPU)" if args.weak else
                                       f"dp{world} (strong: the single-GPU problem sharded over {world} GPU(s), "
                                       "BASELINE configs[4])"),
                       "elements_per_s": float(f"{job_elems * K / (total_ms * 1e-3):.4g}")},
            "roofline": {"bound": "hbm", "kernel": dom, "achieved": per[dom]["GB_s"], "peak": peak, "unit": "GB/s",
                         "frac": round(per[dom]["GB_s"] / peak, 4), "traffic": traffic, "peak_source": peak_src,
                         "bytes_per_launch": per[dom]["bytes"]},
            "per_primitive": per,
            "next_rows": nxt,
            "clocks": clk.summary(),
            "gpu_launches": launches,
            "e2e": e2e,
            "cpu_baseline": cpu,
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        tdist.destroy_process_group()


if __name__ == "__main__":
    main()
