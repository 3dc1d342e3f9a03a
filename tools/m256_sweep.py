"""Config-2 M=256 (LLaMA-2-7B shapes): every orientation / tile / scheduler mode, back-to-back
rotating-weight timing.  Usage: python tools/m256_sweep.py [M]"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_asplos_liu0rxpwl0w25_b200 as cb  # noqa: E402
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth  # noqa: E402

M = int(sys.argv[1]) if len(sys.argv) > 1 else 256
dev = torch.device("cuda", 0)
for name, K, N in (("qkvo", 4096, 4096), ("gate_up", 4096, 11008), ("down", 11008, 4096)):
    tags = synth.make_tags(K, 0.05, np.random.default_rng(0))
    wp, sw, _ = bench.dev_weights(cb, torch, N, K, 1, dev)
    wps = [wp] + [wp.clone() for _ in range(max(1, -(-300 * (1 << 20) // (N * K // 2))) - 1)]
    x = bench.dev_activations(torch, M, K, tags, 2, dev)
    act, sc = cb.quantize_act(x, tags)
    y = torch.empty((M, N), dtype=torch.float16, device=dev)
    res = []
    for kw in (dict(), dict(orientation=3, split_mode=0), dict(orientation=3, split_mode=1), dict(orientation=2, tile_w=128),
               dict(orientation=2, tile_w=192), dict(orientation=2, tile_w=128, split_mode=1), dict(orientation=1, tile_n=128),
               dict(orientation=1, tile_n=64), dict(orientation=1, tile_n=128, split_mode=0), dict(orientation=3, tile_w=128)):
        try:
            plan = cb.Plan(M, N, K, tags, **kw)
        except cb.CometError as e:
            res.append((kw, str(e)[:40]))
            continue
        us = bench.us_rotating(torch, [lambda w_=w_: cb.w4ax_gemm(plan, act, sc, w_, sw, out=y) for w_ in wps])
        res.append((kw, f"{us:7.2f} us {2.0 * M * N * K / us / 1e6:7.1f} TOPS split={plan.info()['n_split_tiles']}"))
    for kw, r in res:
        print(f"{name:8s} {str(kw):48s} {r}")
