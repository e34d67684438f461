"""Profiling driver: fused scan_reduce over 2^28 f32 on cuda:0."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import workloads  # noqa: E402
import paper_conf_pldi_henriksenseho17_b200 as fs  # noqa: E402

x = workloads.device_uniform(1 << 28, 5, torch.device("cuda:0"))
for _ in range(3):
    fs.scan_reduce(x, os.environ.get("RED", "add"))
torch.cuda.synchronize()
