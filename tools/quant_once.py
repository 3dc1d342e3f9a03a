"""One comet_quantize_act launch (after one warm-up) at M x K, for ncu captures of kernel 1.
Usage: python tools/quant_once.py M K"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_asplos_liu0rxpwl0w25_b200 as cb  # noqa: E402
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth  # noqa: E402

M, K = int(sys.argv[1]), int(sys.argv[2])
tags = synth.make_tags(K, 0.05, np.random.default_rng(1))
x = bench.dev_activations(torch, M, K, tags, 3, torch.device("cuda", 0))
act, sc = cb.quantize_act(x, tags)
cb.quantize_act(x, tags, out=(act, sc))
torch.cuda.synchronize()
print("ok")
