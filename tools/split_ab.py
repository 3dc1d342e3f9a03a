"""Prefill GEMM per scheduling mode (LLaMA-3-70B layers at M = 4096, f = 5 %): whole-tile
remapping (0) vs hybrid stream-K (1) vs auto, each layer timed alone (events, L2 flushed by the
bench Timer).  Usage (GPU box): python tools/split_ab.py"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_asplos_liu0rxpwl0w25_b200 as cb  # noqa: E402
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth  # noqa: E402

dev = torch.device("cuda", 0)
timer = bench.Timer(torch, dev)
M = 4096
for name, K, N in (("gate_up", 8192, 28672), ("down", 28672, 8192), ("qkv", 8192, 10240)):
    tags = synth.make_tags(K, 0.05, np.random.default_rng(1))
    wp, sw, _ = bench.dev_weights(cb, torch, N, K, 2, dev)
    x = bench.dev_activations(torch, M, K, tags, 3, dev)
    act, sc = cb.quantize_act(x, tags)
    y = torch.empty((M, N), dtype=torch.float16, device=dev)
    row = []
    for mode in (-1, 0, 1):
        plan = cb.Plan(M, N, K, tags, split_mode=mode)
        us = timer.us(lambda: cb.w4ax_gemm(plan, act, sc, wp, sw, out=y), iters=10)
        row.append(f"mode {mode:2d}: {us:7.1f} us {2.0 * M * N * K / us / 1e6:7.1f} TOPS (max/mean {plan.info()['max_cta_cost'] / plan.info()['mean_cta_cost']:.3f})")
    print(name, " | ".join(row), flush=True)
