"""Diagnostic: per-CTA end-time spread of the decode GEMM (needs a COMET_TRACE=1 build)."""
import ctypes, os, sys
import numpy as np
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_asplos_liu0rxpwl0w25_b200 as cb  # noqa: E402
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth  # noqa: E402
M = int(sys.argv[1]) if len(sys.argv) > 1 else 1
layer = sys.argv[2] if len(sys.argv) > 2 else "gate_up"
K, N = {"gate_up": (8192, 28672), "down": (28672, 8192), "qkv": (8192, 10240)}[layer]
tags = synth.make_tags(K, 0.05, np.random.default_rng(0))
x = torch.randn(M, K, device="cuda", dtype=torch.float16)
w = torch.randint(-8, 8, (N, K), device="cuda", dtype=torch.int8)
sw = torch.rand(N, device="cuda", dtype=torch.float32)
act, sc = cb.quantize_act(x, tags)
wp = cb.pack_weight(w)
plan = cb.Plan(M, N, K, tags)
y = cb.w4ax_gemm(plan, act, sc, wp, sw)
buf = torch.zeros(32768 + 4 * 1024, dtype=torch.int64, device="cuda")
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
flush_rd = torch.ones(64 << 20, dtype=torch.float32, device="cuda")
L = cb.lib()
L.comet_debug_set_trace.argtypes = [ctypes.c_void_p]
L.comet_debug_set_trace(ctypes.c_void_p(buf.data_ptr()))
ends = []
for i in range(5):
    flush.fill_(i); flush_rd.sum()
    torch.cuda.synchronize()
    buf.zero_()
    cb.w4ax_gemm(plan, act, sc, wp, sw, out=y)
    torch.cuda.synchronize()
    b = buf.cpu().numpy()
    n = plan.info()["num_ctas"]
    g = b[32768:32768 + 4 * n].reshape(-1, 4)
    t0 = g[:, 0].min()
    ends.append((g[:, 2] - t0) / 1e3)
L.comet_debug_set_trace(None)
items = plan.describe()
units = np.zeros(n)
for r in items:
    units[r[0]] += r[2] - r[1]
e = np.mean(ends, axis=0)
print("K-blocks per CTA min/med/max", units.min(), np.median(units), units.max())
print("CTA end us deciles", np.round(np.percentile(e, [0, 10, 25, 50, 75, 90, 100]), 2).tolist())
print("corr(units, end)", np.round(np.corrcoef(units, e)[0, 1], 3))
order = np.argsort(e)
print("earliest 8 CTAs", order[:8].tolist(), np.round(e[order[:8]], 1).tolist())
print("latest 8 CTAs", order[-8:].tolist(), np.round(e[order[-8:]], 1).tolist())
print("run-to-run std of per-CTA end (us) median", np.round(np.median(np.std(ends, axis=0)), 2))
