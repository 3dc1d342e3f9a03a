"""One KV4 quantise + dequantise launch (T=32768, C=1024, G=128) for ncu."""
import os, sys
import numpy as np
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_asplos_liu0rxpwl0w25_b200 as cb  # noqa: E402
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth  # noqa: E402
x = torch.from_numpy(synth.make_kv(32768, 1024, np.random.default_rng(0))).cuda()
for _ in range(2):
    c, s, m = cb.kv4_quantize(x, 128)
    y = cb.kv4_dequantize(c, s, m, 128)
torch.cuda.synchronize()
