"""Time comet_quantize_act on the bench's layer inputs (M=4096) and the decode sizes."""
import os, sys, statistics
import numpy as np
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_asplos_liu0rxpwl0w25_b200 as cb  # noqa: E402
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth  # noqa: E402
for M, K in [(4096, 8192), (4096, 28672), (1, 8192), (32, 28672)]:
    rng = np.random.default_rng(1)
    tags = synth.make_tags(K, 0.05, rng)
    x = torch.from_numpy(synth.make_activations(M, K, tags, rng)).cuda()
    act, sc = cb.quantize_act(x, tags)
    torch.cuda.synchronize()
    ev = []
    for i in range(23):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); cb.quantize_act(x, tags, out=(act, sc)); b.record(); ev.append((a, b))
    torch.cuda.synchronize()
    us = statistics.median(a.elapsed_time(b) for a, b in ev[3:]) * 1e3
    nbytes = M * K * 2 + M * K + (K // 128) * M * 6
    print(f"M={M:5d} K={K:6d} {us:8.2f} us {nbytes / us / 1e3:8.1f} GB/s")
