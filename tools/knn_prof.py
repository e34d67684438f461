import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, workloads, paper_conf_pldi_henriksenseho17_b200 as fs
lat, lng, q = workloads.c2_nn()
L, G = torch.from_numpy(lat).cuda(), torch.from_numpy(lng).cuda()
for _ in range(3):
    d, i = fs.nn_knn(L, G, q, 100)
torch.cuda.synchronize()
