"""Decode GEMM A/B: plan orientation 1 (tcgen05, TMEM-widened weights) against orientation 4
(gemm_v.cu, mma.sync with register-streamed weights) on the config-5 layers at M = 1, 4, 8.
Same timing as bench.py's decode sweep: back-to-back launches over weight copies > 2 x L2.
Usage: python tools/gemv_ab.py [orientations, default 1,4] [c2: LLaMA-2-7B shapes]"""
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
orients = [int(o) for o in (sys.argv[1] if len(sys.argv) > 1 else "1,4").split(",")]
layers = bench.LAYERS
if len(sys.argv) > 2 and sys.argv[2] == "c2":   # LLaMA-2-7B (config 2) shapes
    layers = [("qkvo", 4096, 4096, "col"), ("gate_up", 4096, 11008, "col"), ("down", 11008, 4096, "row")]
for li, (name, K, N, kind) in enumerate(layers):
    tags = synth.make_tags(K, bench.FRAC, np.random.default_rng(7))
    wp, swd, _ = bench.dev_weights(cb, torch, N, K, 70 + li, dev)
    ncopy = max(2, -(-300 * (1 << 20) // (N * K // 2)))
    wps = [wp] + [wp.clone() for _ in range(ncopy - 1)]
    for M in (1, 4, 8):
        x = bench.dev_activations(torch, M, K, tags, 700 + M, dev)
        act, sc = cb.quantize_act(x, tags)
        y = torch.empty((M, N), dtype=torch.float16, device=dev)
        nbytes = N * K // 2 + N * 4 + act.numel() + sc.numel() * 4 + M * N * 2
        line = f"{name:8s} M={M}"
        for o in orients:
            plan = cb.Plan(M, N, K, tags, orientation=o)
            us = bench.us_rotating(torch, [lambda w_=w_: cb.w4ax_gemm(plan, act, sc, w_, swd, out=y) for w_ in wps])
            st = bench.us_rotating(torch, [lambda w_=w_: (cb.quantize_act(x, tags, out=(act, sc)),
                                                          cb.w4ax_gemm(plan, act, sc, w_, swd, out=y)) for w_ in wps])
            gbs = nbytes / us / 1e3
            line += f" | o{o} {us:6.2f} us {gbs:7.1f} GB/s {gbs / peaks['hbm_gbs']:.3f} step {st:6.2f}"
        print(line, flush=True)
    del wps, wp
