"""Diagnostic: fixed-cost anatomy of the decode GEMM (event-timed, L2 clean before every launch):
an empty torch kernel, tiny GEMMs (one tile; one tile per CTA) and the LLaMA-2-7B q/k/v/o layer
under each scheduler mode.  Usage: python tools/dec_overhead.py"""
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
z = torch.zeros(1, device=dev)
print("empty torch kernel      ", round(timer.us(lambda: z.add_(1.0)), 2), "us")
for (M, N, K, mode) in ((1, 128, 128, -1), (1, 128 * 148, 512, 0), (1, 128 * 148, 4096, 0), (1, 128 * 148, 4096, 1),
                        (1, 4096, 4096, 0), (1, 4096, 4096, 1), (1, 4096, 4096, 2), (16, 4096, 4096, 1),
                        (1, 10240, 8192, 1), (1, 28672, 8192, 1)):
    tags = synth.make_tags(K, 0.05, np.random.default_rng(0))
    wp, sw, _ = bench.dev_weights(cb, torch, N, K, 1, dev)
    x = bench.dev_activations(torch, M, K, tags, 2, dev)
    act, sc = cb.quantize_act(x, tags)
    plan = cb.Plan(M, N, K, tags, split_mode=mode)
    y = torch.empty((M, N), dtype=torch.float16, device=dev)
    us = timer.us(lambda: cb.w4ax_gemm(plan, act, sc, wp, sw, out=y))
    us_nf = timer.us(lambda: cb.w4ax_gemm(plan, act, sc, wp, sw, out=y), flush=False)
    i = plan.info()
    print(f"M={M:3d} N={N:6d} K={K:5d} mode={i['split_mode']} tiles={i['n_tiles']:5d} split={i['n_split_tiles']:4d} "
          f"items={i['n_items']:4d}  {us:7.2f} us (L2 warm {us_nf:7.2f})  {N * K / 2 / us / 1e3:7.1f} GB/s")
