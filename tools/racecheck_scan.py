import os, sys
sys.path.insert(0, os.getcwd())
import numpy as np, torch, workloads, paper_conf_pldi_henriksenseho17_b200 as fs
x = torch.from_numpy(workloads.mixed(300_001, 1, np.float32)).cuda()
fs.scanomap(x, "add"); fs.seg_scan(x[:300*1000], 300, 1000, "add"); torch.cuda.synchronize(); print("ok")
