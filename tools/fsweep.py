"""Prefill GEMM TOPS vs INT8-block fraction (LLaMA-3-8B up, M = 8192, auto plan), back-to-back
launches.  Usage: python tools/fsweep.py"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_asplos_liu0rxpwl0w25_b200 as cb  # noqa: E402
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth  # noqa: E402

dev = torch.device("cuda", 0)
M, K, N = 8192, 4096, 14336
wp, sw, _ = bench.dev_weights(cb, torch, N, K, 1, dev)
res = []
for f in (0.0, 0.05, 0.25, 1.0):
    tags = synth.make_tags(K, f, np.random.default_rng(2))
    x = bench.dev_activations(torch, M, K, tags, 3, dev)
    act, sc = cb.quantize_act(x, tags)
    plan = cb.Plan(M, N, K, tags)
    y = torch.empty((M, N), dtype=torch.float16, device=dev)
    us = bench.us_rotating(torch, [lambda: cb.w4ax_gemm(plan, act, sc, wp, sw, out=y)], rounds=20)
    res.append(f"f={f:.2f} {2.0 * M * N * K / us / 1e6:7.1f} TOPS")
print(" | ".join(res))
