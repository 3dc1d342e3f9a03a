"""NEXT-3: group-wise vs per-channel weight scales on the prefill pair kernel (LLaMA-3-70B
layers, M = 4096), back-to-back launches.  Usage: python tools/grouped_time.py"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_asplos_liu0rxpwl0w25_b200 as cb  # noqa: E402
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth  # noqa: E402

dev = torch.device("cuda", 0)
M = 4096
for name, K, N in (("gate_up", 8192, 28672), ("down", 28672, 8192), ("qkv", 8192, 10240)):
    tags = synth.make_tags(K, 0.05, np.random.default_rng(0))
    wp, sw, _ = bench.dev_weights(cb, torch, N, K, 1, dev)
    swg = (sw[None, :] * (0.5 + torch.rand(K // 128, N, device=dev))).contiguous()
    x = bench.dev_activations(torch, M, K, tags, 2, dev)
    act, sc = cb.quantize_act(x, tags)
    plan = cb.Plan(M, N, K, tags, **({"orientation": 1} if M < 128 else {}))
    y = torch.empty((M, N), dtype=torch.float16, device=dev)
    us_c = bench.us_rotating(torch, [lambda: cb.w4ax_gemm(plan, act, sc, wp, sw, out=y)], rounds=10)
    us_g = bench.us_rotating(torch, [lambda: cb.w4ax_gemm_grouped(plan, act, sc, wp, swg, out=y)], rounds=10)
    ops = 2.0 * M * N * K
    print(f"{name:8s} per-channel {us_c:8.1f} us {ops / us_c / 1e6:7.1f} TOPS | grouped {us_g:8.1f} us {ops / us_g / 1e6:7.1f} TOPS")
