"""One fused-permutation quantise launch (M=4096, K from argv, calibrated perm) for ncu."""
import os, sys
import numpy as np
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_asplos_liu0rxpwl0w25_b200 as cb  # noqa: E402
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth  # noqa: E402
K = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
up = synth.make_unpermuted_problem(4096, K, 128, seed=2, m_calib=64)
perm, tags, _ = cb.calibrate_perm(np.abs(up.x_calib.astype(np.float32)).max(0))
x = torch.from_numpy(up.x).cuda()
pm = torch.from_numpy(perm).cuda()
for _ in range(2):
    cb.quantize_act(x, tags, perm=pm)
torch.cuda.synchronize()
