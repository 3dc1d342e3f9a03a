"""Time comet_quantize_act (identity and fused-permutation paths) on the bench's layer inputs
(M=4096) and the decode sizes.  L2 is left full of clean unrelated lines (256 MiB write + 256 MiB read) before every timed launch."""
import os, sys, statistics
import numpy as np
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_asplos_liu0rxpwl0w25_b200 as cb  # noqa: E402
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth  # noqa: E402
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
flush_rd = torch.ones(64 << 20, dtype=torch.float32, device="cuda")
for M, K in [(4096, 8192), (4096, 28672), (1, 8192), (32, 28672)]:
    rng = np.random.default_rng(1)
    tags = synth.make_tags(K, 0.05, rng)
    x = torch.from_numpy(synth.make_activations(M, K, tags, rng)).cuda()
    perm = torch.from_numpy(rng.permutation(K).astype(np.int32)).cuda()
    up = synth.make_unpermuted_problem(4, K, 128, seed=2)
    cperm, _, _ = cb.calibrate_perm(np.abs(up.x_calib.astype(np.float32)).max(0))
    cperm = torch.from_numpy(cperm).cuda()
    for name, pm in (("identity", None), ("randperm", perm), ("calperm", cperm)):
        act, sc = cb.quantize_act(x, tags, perm=pm)
        torch.cuda.synchronize()
        ev = []
        for i in range(23):
            flush.fill_(i & 0xFF); flush_rd.sum()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(); cb.quantize_act(x, tags, perm=pm, out=(act, sc)); b.record(); ev.append((a, b))
        torch.cuda.synchronize()
        us = statistics.median(a.elapsed_time(b) for a, b in ev[3:]) * 1e3
        nbytes = M * K * 2 + M * K + (K // 128) * M * 6
        print(f"{name:8s} M={M:5d} K={K:6d} {us:8.2f} us {nbytes / us / 1e3:8.1f} GB/s")
