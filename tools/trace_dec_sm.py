"""Diagnostic (COMET_TRACE=1 build): decode GEMM CTA end times against the SM each CTA ran on
(%smid) and its bytes, to see whether the bandwidth-share tail follows the SM (e.g. the die).
Usage: python tools/trace_dec_sm.py [M] [layer]"""
import ctypes
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_asplos_liu0rxpwl0w25_b200 as cb  # noqa: E402
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth  # noqa: E402

M = int(sys.argv[1]) if len(sys.argv) > 1 else 1
K, N = 8192, 28672
tags = synth.make_tags(K, 0.05, np.random.default_rng(0))
x = torch.randn(M, K, device="cuda", dtype=torch.float16)
w = torch.randint(-8, 8, (N, K), device="cuda", dtype=torch.int8)
sw = torch.rand(N, device="cuda", dtype=torch.float32)
act, sc = cb.quantize_act(x, tags)
wp = cb.pack_weight(w)
for mode in (1, 0):
    plan = cb.Plan(M, N, K, tags, split_mode=mode)
    y = cb.w4ax_gemm(plan, act, sc, wp, sw)
    buf = torch.zeros(32768 + 4 * 1024, dtype=torch.int64, device="cuda")
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    L = cb.lib()
    L.comet_debug_set_trace.argtypes = [ctypes.c_void_p]
    ends = []
    for rep in range(5):
        L.comet_debug_set_trace(ctypes.c_void_p(buf.data_ptr()))
        flush.fill_(rep)
        torch.cuda.synchronize()
        buf.zero_()
        cb.w4ax_gemm(plan, act, sc, wp, sw, out=y)
        torch.cuda.synchronize()
        L.comet_debug_set_trace(None)
        g = buf[32768:32768 + 4 * plan.info()["num_ctas"]].view(-1, 4).cpu().numpy()
        t0 = g[:, 0].min()
        ends.append((g[:, 3], (g[:, 2] - t0) / 1e3))
    items = plan.describe()
    work = np.zeros(plan.info()["num_ctas"])
    for cta, tile, k0, k1 in items:
        work[cta] += k1 - k0
    sm = ends[0][0]
    e = np.mean([dict(zip(s_, t_)).__getitem__ for s_, t_ in ends][:1] and [np.array([dict(zip(s_, t_))[x] for x in sm]) for s_, t_ in ends], axis=0)
    print(f"mode {mode}: end (us) by smid, mean of 5 launches; work = K-blocks per CTA")
    order = np.argsort(sm)
    for lo in range(0, len(order), 16):
        idx = order[lo:lo + 16]
        print("  sm", f"{int(sm[idx[0]]):3d}-{int(sm[idx[-1]]):3d}", " ".join(f"{v:5.1f}" for v in e[idx]))
    print("  end by work: ", {int(k): round(float(e[work == k].mean()), 2) for k in np.unique(work)})
    # do CTAs with the same smid across launches end at a similar relative time?
    ranks = []
    for s_, t_ in ends:
        d = dict(zip(s_, t_))
        ranks.append(np.array([d[x] for x in sm]))
    ranks = np.array(ranks)
    c = np.corrcoef(ranks)
    print("  launch-to-launch correlation of per-SM end times:", np.round(c[0, 1:], 2))
