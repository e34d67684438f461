"""Profiling driver: seg_map_reduce over the same 2^28 f32 as [2^14][2^14] and [2^18][1024]."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import workloads  # noqa: E402
import paper_conf_pldi_henriksenseho17_b200 as fs  # noqa: E402

x = workloads.device_uniform(1 << 28, 5, torch.device("cuda:0"))
om = torch.empty_like(x)
for nseg, L in ((1 << 14, 1 << 14), (1 << 18, 1024), (1 << 14, 1 << 14)):
    for _ in range(2):
        fs.seg_map_reduce(x, nseg, L, 1.0, "add", out_map=om)
torch.cuda.synchronize()
