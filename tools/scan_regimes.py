#!/usr/bin/env python
"""Row-major seg_scan f32 add over 2^28 elements: auto regime vs the look-back ring scan (5),
KS2 (9) and the flat scan per row (12) forced, for the long-row seglens where they compete.
Device time (CUDA events, median of reps, 1 GB L2 flush before each rep); fraction of the
measured HBM peak."""
import json
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_pldi_henriksenseho17_b200 as fs  # noqa: E402

PEAK = 6546.9


def main():
    n = 1 << 28
    x = torch.rand(n, device="cuda")
    y = torch.empty_like(x)
    flush = torch.empty(1 << 28, device="cuda")
    out = []
    seglens = [int(v) for v in sys.argv[1].split(",")] if len(sys.argv) > 1 else \
        [1 << 17, 1 << 18, 1 << 19, 1 << 20, 1 << 21, 1 << 22, 1 << 24, 1 << 26, 1 << 27]
    for L in seglens:
        nseg = n // L
        rec = {"seglen": L, "nseg": nseg}
        for reg in (-1, 5, 9, 12):
            fs.force_seg_regime(reg)
            try:
                fn = lambda: fs.seg_scan(x[: nseg * L], nseg, L, "add", out=y[: nseg * L])
                fn()
                launched = fs.last_seg_regime()
                ts = []
                for _ in range(5):
                    flush.sum()
                    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    a.record()
                    fn()
                    b.record()
                    b.synchronize()
                    ts.append(a.elapsed_time(b))
                ms = statistics.median(ts)
                rec[f"r{reg}"] = {"launched": launched, "frac": round(8 * nseg * L / ms / 1e6 / PEAK, 4)}
            finally:
                fs.force_seg_regime(-1)
        out.append(rec)
        print(json.dumps(rec), flush=True)


if __name__ == "__main__":
    main()
