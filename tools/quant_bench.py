"""Kernel 1 (comet_quantize_act) throughput on the bench's layer inputs (M = 4096; K = 8192 and
28672) and decode sizes: mean per launch over back-to-back launches cycling through input
copies totalling > 2 x L2 (every launch reads HBM).  GB/s on the SURVEY §8(d) algorithmic bytes
(16-bit input + codes at their packed width + FP32 scales) and on the bytes the layout moves.
Usage: python tools/quant_bench.py"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_asplos_liu0rxpwl0w25_b200 as cb  # noqa: E402
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth  # noqa: E402

dev = torch.device("cuda", 0)
peaks, _ = bench.load_peaks()
for M, K in [(4096, 8192), (4096, 28672), (8192, 14336), (4096, 11008), (256, 4096), (256, 11008), (1, 8192), (32, 28672)]:
    tags = synth.make_tags(K, 0.05, np.random.default_rng(1))
    x = bench.dev_activations(torch, M, K, tags, 3, dev)
    ncopy = max(2, -(-300 * (1 << 20) // (M * K * 2)))
    xs = [x] + [x.clone() for _ in range(min(ncopy, 64) - 1)]
    act, sc = cb.quantize_act(x, tags)
    us = bench.us_rotating(torch, [lambda x_=x_: cb.quantize_act(x_, tags, out=(act, sc)) for x_ in xs])
    f = tags.mean()
    alg = M * K * 2 + M * K * (0.5 * (1 - f) + f) + 4 * M * (K // 128)
    moved = M * K * 2 + M * K + (K // 128) * M * 6 + M * 4
    print(f"M={M:5d} K={K:6d} {us:8.2f} us  {alg / us / 1e3:7.1f} GB/s alg ({alg / us / 1e3 / peaks['hbm_gbs']:.3f})"
          f"  {moved / us / 1e3:7.1f} GB/s moved")
