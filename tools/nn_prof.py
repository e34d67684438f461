"""Profiling driver: NN argmin redomap (C2 and a tiny input) on cuda:0."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import workloads  # noqa: E402
import paper_conf_pldi_henriksenseho17_b200 as fs  # noqa: E402

lat, lng, q = workloads.c2_nn()
L, G = torch.from_numpy(lat).cuda(), torch.from_numpy(lng).cuda()
for n in (1000, 100_000, lat.size):
    for _ in range(3):
        fs.redomap(L[:n], "argmin", map="nn_dist", lng=G[:n], query=q)
torch.cuda.synchronize()
