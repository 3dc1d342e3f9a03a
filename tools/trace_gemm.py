"""Diagnostic: clock64 timeline of the first two CTAs of one W4Ax GEMM launch (LLaMA-3-70B
gate/up, M=4096).  Events per K-block: 0 producer issued loads, 1 MMA loop top, 2 MMA after
acc_empty wait, 3 MMA after b_full wait, 4 widen done (b_full arrive), 5 widen start (after
full wait), 6 promotion after acc_full wait, 7 promotion done.  Usage (on the GPU box):
  COMET_ABLATE=<bits> python tools/trace_gemm.py [orientation] > gpurun_out/trace.json"""
import ctypes
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_asplos_liu0rxpwl0w25_b200 as cb  # noqa: E402
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth  # noqa: E402

orient = int(sys.argv[1]) if len(sys.argv) > 1 else 0
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
buf = torch.zeros(2 * 16 * 1024, dtype=torch.int64, device="cuda")
L = cb.lib()
L.comet_debug_set_trace.argtypes = [ctypes.c_void_p]
L.comet_debug_set_trace(ctypes.c_void_p(buf.data_ptr()))
for _ in range(2):
    cb.w4ax_gemm(plan, act, sc, wp, sw, out=y)
torch.cuda.synchronize()
L.comet_debug_set_trace(None)
t = buf.view(2, 16, 1024).cpu().numpy()
print(json.dumps({"info": plan.info(), "trace": t.tolist()}))
