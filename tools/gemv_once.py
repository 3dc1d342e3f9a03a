"""A few orientation-4 launches of the LLaMA-3-70B gate/up GEMM at M = 1 (ncu target).
Usage: python tools/gemv_once.py"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_asplos_liu0rxpwl0w25_b200 as cb  # noqa: E402
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth  # noqa: E402

dev = torch.device("cuda", 0)
K, N, M = 8192, 28672, 1
tags = synth.make_tags(K, bench.FRAC, np.random.default_rng(7))
wp, swd, _ = bench.dev_weights(cb, torch, N, K, 71, dev)
x = bench.dev_activations(torch, M, K, tags, 701, dev)
act, sc = cb.quantize_act(x, tags)
plan = cb.Plan(M, N, K, tags, orientation=4)
y = torch.empty((M, N), dtype=torch.float16, device=dev)
for _ in range(3):
    cb.w4ax_gemm(plan, act, sc, wp, swd, out=y)
torch.cuda.synchronize()
print("ok")
