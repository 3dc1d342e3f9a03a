"""Diagnostic: timeline of the decode GEMM (orientation 1) on LLaMA-3-70B gate/up at small M.
Needs a COMET_TRACE=1 (or COMET_DIAG=1) build.  Prints per-CTA start/end spread (globaltimer)
and, for CTA 0, the clock64 timeline of every role:
  0 producer issued stage s | 1/2 MMA after full / after a_full wait (stage) |
  3/5 widen group 0 after full wait / after a_full arrive (stage seq) | 4/6 same, group 1 |
  7/8/9 promotion after s_full / after acc_full / done (K-block) | 10/11/12 epilogue of item i:
  start / partials ready (owner of a split tile) / done.
Usage: python tools/trace_dec.py [M] [layer]"""
import ctypes
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_asplos_liu0rxpwl0w25_b200 as cb  # noqa: E402
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth  # noqa: E402

M = int(sys.argv[1]) if len(sys.argv) > 1 else 1
layer = sys.argv[2] if len(sys.argv) > 2 else "gate_up"
K, N = {"gate_up": (8192, 28672), "down": (28672, 8192), "qkv": (8192, 10240),
        "l2_qkvo": (4096, 4096), "l2_gate_up": (4096, 11008), "l2_down": (11008, 4096)}[layer]
rng = np.random.default_rng(0)
tags = synth.make_tags(K, 0.05, rng)
x = torch.randn(M, K, device="cuda", dtype=torch.float16)
w = torch.randint(-8, 8, (N, K), device="cuda", dtype=torch.int8)
sw = torch.rand(N, device="cuda", dtype=torch.float32)
act, sc = cb.quantize_act(x, tags)
wp = cb.pack_weight(w)
plan = cb.Plan(M, N, K, tags)
y = cb.w4ax_gemm(plan, act, sc, wp, sw)
buf = torch.zeros(32768 + 4 * 1024, dtype=torch.int64, device="cuda")
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
L = cb.lib()
L.comet_debug_set_trace.argtypes = [ctypes.c_void_p]
L.comet_debug_set_trace(ctypes.c_void_p(buf.data_ptr()))
for i in range(3):
    flush.fill_(i)
    torch.cuda.synchronize()
    buf.zero_()
    cb.w4ax_gemm(plan, act, sc, wp, sw, out=y)
    torch.cuda.synchronize()
L.comet_debug_set_trace(None)
b = buf.cpu().numpy()
info = plan.info()
print("plan", {k: info[k] for k in ("tile_n", "num_ctas", "split_mode", "n_tiles", "n_items", "n_split_tiles")})
g = b[32768:32768 + 4 * info["num_ctas"]].reshape(-1, 4)
t0 = g[:, 0].min()
ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
flush.fill_(9)
ev0.record()
cb.w4ax_gemm(plan, act, sc, wp, sw, out=y)
ev1.record()
torch.cuda.synchronize()
print("event time (us, trace build)", round(ev0.elapsed_time(ev1) * 1e3, 2))
print("CTA start  (us) min/med/max", *(np.round(np.percentile(g[:, 0] - t0, [0, 50, 100]) / 1e3, 2)))
print("CTA setup  (us) min/med/max", *(np.round(np.percentile(g[:, 1] - t0, [0, 50, 100]) / 1e3, 2)))
print("CTA end    (us) min/med/max", *(np.round(np.percentile(g[:, 2] - t0, [0, 50, 100]) / 1e3, 2)))
print("slowest CTAs", np.argsort(g[:, 2])[-5:].tolist(), np.round((np.sort(g[:, 2])[-5:] - t0) / 1e3, 2).tolist())
items = plan.describe()
for cta in (0, 1):
    t = b[:32768].reshape(2, 16, 1024)[cta]
    base = t[0][0]
    n_st = int((t[0] > 0).sum())
    n_kb = int((t[8] > 0).sum())
    print(f"--- CTA {cta}: {n_st} stages, {n_kb} K-blocks promoted, items",
          [tuple(r[1:]) for r in items if r[0] == cta])

    def rel(e, n):
        return (t[e][:n] - base).astype(np.int64)

    prod = rel(0, n_st)
    n_m = (n_st + 1) // 2                      # MMA events: issuer 0 = even stages only
    m_go, m_done = rel(1, n_m), rel(2, n_m)
    wg = [rel(3, n_st), rel(4, n_st), rel(5, n_st), rel(6, n_st)]
    idx = np.arange(n_st)
    wstart = np.minimum(wg[0], wg[1])          # v4: both widen halves take every stage
    wdone = np.maximum(wg[2], wg[3])
    p_go, p_done = rel(7, n_st), rel(8, n_st)
    print("producer issue   first 10:", prod[:10].tolist())
    print("widen start      first 10:", wstart[:10].tolist())
    print("widen done       first 10:", wdone[:10].tolist())
    print("MMA(even) go     first 5 :", m_go[:5].tolist())
    print("MMA(even) done   first 5 :", m_done[:5].tolist())
    print("promo go         first 10:", p_go[:10].tolist())
    print("promo done       first 10:", p_done[:10].tolist())
    if n_st > 8:
        e = np.arange(3, n_st - 1)
        em = np.arange(2, n_m - 1)
        print("per-stage period medians: producer", np.median(np.diff(prod[3:])), "widen", np.median(np.diff(wdone[3:])),
              "promo", np.median(np.diff(p_done[3:])), "MMA (2 stages)", np.median(np.diff(m_done[2:])))
        print("latencies: producer->widen start", np.median(wstart[e] - prod[e]), "widen dur", np.median(wdone[e] - wstart[e]),
              "widen done->MMA go", np.median(m_go[em] - wdone[2 * em]), "MMA issue dur", np.median(m_done[em] - m_go[em]),
              "MMA done->promo go", np.median(p_go[2 * em] - m_done[em]), "promo dur", np.median(p_done[e] - p_go[e]))
    if n_st > 8:
        e13, e14, e15 = rel(13, n_st), rel(14, n_st), rel(15, n_st)
        print("widen g0 phases (median clk): LDS+release+a_empty wait", np.median(e14[e] - wg[0][e]),
              "convert+tmem st issue", np.median(e13[e] - e14[e]), "wait::st", np.median(e15[e] - e13[e]),
              "fence+arrive", np.median(wg[2][e] - e15[e]))
    ep = [(t[10][i] - base, t[11][i] - base if t[11][i] else -1, t[12][i] - base) for i in range(8) if t[10][i]]
    print("epilogues (start, partials ready, done):", ep)
    print("end of last promotion", p_done[-1] if n_st else None)

# detailed timeline of CTA 1 around its item boundaries: per stage, each role's timestamps
t = b[:32768].reshape(2, 16, 1024)[1]
base = t[0][0]
n_st = int((t[0] > 0).sum())
print("stage | W-issued widenStart widenDone MMAgo MMAdone promoGo promoDone")
for i in range(n_st):
    def g(e, k):
        return int(t[e][k] - base) if t[e][k] else -1
    print(f"{i:3d} | {g(0, i):7d} {min(g(3, i), g(4, i)):7d} {max(g(5, i), g(6, i)):7d} {g(1, i):7d} {g(2, i):7d} {g(7, i):7d} {g(8, i):7d}")
print("epilogue start/last/done per item:", [(int(t[10][i] - base), int(t[11][i] - base) if t[11][i] else -1, int(t[12][i] - base)) for i in range(6) if t[10][i]])
