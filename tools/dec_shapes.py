"""Diagnostic: decode GEMM (M=1) on shapes that divide evenly over the 148 SMs (no split tiles,
no fix-up kernel) against the LLaMA-3-70B gate/up layer (stream-K + fix-up); event-timed, L2
clean before every launch, mean of the middle 80 % of 60 launches (the event clock ticks in
~1 us steps, the mean dithers through them)."""
import os
import statistics
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_asplos_liu0rxpwl0w25_b200 as cb  # noqa: E402
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth  # noqa: E402

dev = torch.device("cuda", 0)
timer = bench.Timer(torch, dev)


def tmean(fn, iters=60):
    torch.cuda.synchronize()
    ws = []
    torch.cuda._sleep(int(4e7))
    for i in range(iters):
        timer.flush.fill_(i & 0xFF)
        timer.flush_rd.sum()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); fn(); b.record()
        ws.append((a, b))
    torch.cuda.synchronize()
    v = sorted(a.elapsed_time(b) * 1e3 for a, b in ws)
    k = len(v) // 10
    return statistics.mean(v[k:len(v) - k])


z = torch.zeros(1, device=dev)
print("empty kernel", round(tmean(lambda: z.add_(1.0)), 2))
for (M, N, K, mode) in ((1, 148 * 128 * 2, 8192, 0), (1, 148 * 128, 8192 * 2, 0), (1, 28672, 8192, 1),
                        (1, 28672, 8192, 0), (1, 148 * 128 * 4, 4096, 0), (8, 28672, 8192, 1), (32, 28672, 8192, 1)):
    tags = synth.make_tags(K, 0.05, np.random.default_rng(0))
    wp, sw, _ = bench.dev_weights(cb, torch, N, K, 1, dev)
    x = bench.dev_activations(torch, M, K, tags, 2, dev)
    act, sc = cb.quantize_act(x, tags)
    plan = cb.Plan(M, N, K, tags, split_mode=mode)
    y = torch.empty((M, N), dtype=torch.float16, device=dev)
    us = tmean(lambda: cb.w4ax_gemm(plan, act, sc, wp, sw, out=y))
    i = plan.info()
    print(f"M={M:3d} N={N:6d} K={K:6d} mode={i['split_mode']} tiles={i['n_tiles']:5d} split={i['n_split_tiles']:4d} "
          f"{us:7.2f} us  {N * K / 2 / us / 1e3:7.1f} GB/s")
