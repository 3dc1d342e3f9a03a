"""Diagnostic (needs a COMET_DIAG=1 build): time the LLaMA-3-70B gate/up GEMM (M=4096) with
parts of the pipeline switched off through COMET_ABLATE bits -- 4 skip widening stores,
8 skip MMAs, 16 skip promotion work -- to see which role bounds the K-block period.
Usage: python tools/ablate_time.py [orientation] [bits ...]"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_asplos_liu0rxpwl0w25_b200 as cb  # noqa: E402
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth  # noqa: E402

orient = int(sys.argv[1]) if len(sys.argv) > 1 else 0
bits = [int(b) for b in sys.argv[2:]] or [0, 16, 4, 8, 20, 24, 12, 28]
M, K, N = 4096, 8192, 28672
rng = np.random.default_rng(0)
tags = synth.make_tags(K, 0.05, rng)
x = torch.randn(M, K, device="cuda", dtype=torch.float16)
w = torch.randint(-8, 8, (N, K), device="cuda", dtype=torch.int8)
sw = torch.rand(N, device="cuda", dtype=torch.float32)
act, sc = cb.quantize_act(x, tags)
wp = cb.pack_weight(w)
plan = cb.Plan(M, N, K, tags, orientation=orient)
y = cb.w4ax_gemm(plan, act, sc, wp, sw)
flops = 2.0 * M * N * K
for b in bits:
    os.environ["COMET_ABLATE"] = str(b)
    for _ in range(3):
        cb.w4ax_gemm(plan, act, sc, wp, sw, out=y)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record()
    for _ in range(10):
        cb.w4ax_gemm(plan, act, sc, wp, sw, out=y)
    e1.record()
    torch.cuda.synchronize()
    us = e0.elapsed_time(e1) * 100.0
    print(f"ablate {b:2d}: {us:8.1f} us  {flops / us / 1e6:7.1f} TOPS", flush=True)
