import numpy as np, torch, sys
sys.path.insert(0, '.')
import paper_conf_pldi_henriksenseho17_b200 as fs, workloads, oracle
fs.force_seg_regime(11)
for nseg, L in [(200, 33), (64, 64), (100, 100), (50, 1000), (64, 2048), (9, 4097), (16, 8192), (150, 12_288), (160, 16_384)]:
    for dt, op in ((np.float32, "add"), (np.int32, "add"), (np.int64, "add"), (np.int64, "min"), (np.int32, "max")):
        x = workloads.mixed(nseg * L, 3, dt)
        try:
            g = fs.seg_scan(torch.from_numpy(x).cuda(), nseg, L, op); torch.cuda.synchronize()
            print("ok", nseg, L, np.dtype(dt).name, op, fs.last_seg_regime(), flush=True)
        except Exception as e:
            print("FAIL", nseg, L, np.dtype(dt).name, op, fs.last_seg_regime(), e, flush=True)
            sys.exit(1)
