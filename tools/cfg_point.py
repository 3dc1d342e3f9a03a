"""Run one GEMM point of config 2 or 3 (for an ncu capture).  Usage:
  python tools/cfg_point.py c2 <M> <layer: qkvo|gate_up|down>     (LLaMA-2-7B shapes)
  python tools/cfg_point.py c3 <f percent> <layer: up|down>      (LLaMA-3-8B MLP, M = 8192)"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_asplos_liu0rxpwl0w25_b200 as cb  # noqa: E402
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth  # noqa: E402

cfg = sys.argv[1]
dev = torch.device("cuda", 0)
if cfg == "c2":
    M, layer = int(sys.argv[2]), sys.argv[3]
    K, N = dict((n, (k, nn)) for n, k, nn in bench.LLAMA2_7B)[layer]
    f = 0.05
else:
    M, f, layer = 8192, float(sys.argv[2]) / 100.0, sys.argv[3]
    K, N = dict((n, (k, nn)) for n, k, nn in bench.LLAMA3_8B)[layer]
tags = synth.make_tags(K, f, np.random.default_rng(1))
wp, sw, _ = bench.dev_weights(cb, torch, N, K, 2, dev)
x = bench.dev_activations(torch, M, K, tags, 3, dev)
act, sc = cb.quantize_act(x, tags)
plan = cb.Plan(M, N, K, tags)
y = torch.empty((M, N), dtype=torch.float16, device=dev)
for _ in range(3):
    cb.w4ax_gemm(plan, act, sc, wp, sw, out=y)
torch.cuda.synchronize()
print(cfg, M, K, N, f, plan.info())
