"""Time the KV4 kernels (NEXT-4) on a LLaMA-3-70B-shaped KV cache: C = 8 KV heads x 128 =
1024 channels, T = 32768 tokens (e.g. 8 sequences x 4096), group 128.  L2 is left full of clean
unrelated lines before every timed launch.  Prints GB/s against the algorithmic bytes."""
import json, os, statistics, sys
import numpy as np
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_asplos_liu0rxpwl0w25_b200 as cb  # noqa: E402
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth  # noqa: E402
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
flush_rd = torch.ones(64 << 20, dtype=torch.float32, device="cuda")
hbm = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "MEASURED_PEAKS.json")))["hbm_gbs"] \
    if os.path.exists(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "MEASURED_PEAKS.json")) else 6550.0
res = {}
for T, C, G in [(32768, 1024, 128), (131072, 1024, 128), (4096, 8192, 128)]:
    x = torch.from_numpy(synth.make_kv(T, C, np.random.default_rng(0))).cuda()
    codes, scales, mins = cb.kv4_quantize(x, G)
    y = cb.kv4_dequantize(codes, scales, mins, G)
    ng = (T + G - 1) // G
    for name, fn, nbytes in (("quantize", lambda: cb.kv4_quantize(x, G, out=(codes, scales, mins)), T * C * 2 + T * C // 2 + ng * C * 8),
                             ("dequantize", lambda: cb.kv4_dequantize(codes, scales, mins, G, out=y), T * C * 2 + T * C // 2 + ng * C * 8)):
        torch.cuda.synchronize()
        ev = []
        for i in range(23):
            flush.fill_(i & 0xFF); flush_rd.sum()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(); fn(); b.record(); ev.append((a, b))
        torch.cuda.synchronize()
        us = statistics.median(a.elapsed_time(b) for a, b in ev[3:]) * 1e3
        gbs = nbytes / us / 1e3
        res[f"{name}_T{T}_C{C}"] = {"us": round(us, 2), "GB/s": round(gbs, 1), "frac_hbm": round(gbs / hbm, 3), "bytes": nbytes}
        print(f"{name:10s} T={T:6d} C={C:5d} G={G} {us:8.2f} us {gbs:8.1f} GB/s  {gbs / hbm:.3f} of {hbm}")
print(json.dumps(res))
