"""Prefill pair-kernel tile widths on the LLaMA-3-70B layers at M = 4096 (events, L2 cleaned by
the bench Timer): tile_w 256 (production) / 192 / 160 / 128.  Usage (GPU box): python tools/tilew_ab.py"""
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
    for tw in (256, 192, 160, 128):
        plan = cb.Plan(M, N, K, tags, orientation=3, tile_w=tw)
        us = timer.us(lambda: cb.w4ax_gemm(plan, act, sc, wp, sw, out=y), iters=10)
        row.append(f"tile_w {tw}: {us:7.1f} us {2.0 * M * N * K / us / 1e6:7.1f} TOPS")
    print(name, " | ".join(row), flush=True)
