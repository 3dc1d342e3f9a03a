"""Run bench.py's config-5 decode sweep alone (GPU box).  Usage: python tools/decode_bench.py"""
import json, os, sys
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_asplos_liu0rxpwl0w25_b200 as cb  # noqa: E402
dev = torch.device("cuda", 0)
peaks, _ = bench.load_peaks()
d = bench.decode_sweep(cb, torch, dev, peaks, bench.Timer(torch, dev))
for k, v in d["layers"].items():
    print(f"{k:12s} {v['us']:7.2f} us {v['GB/s']:7.1f} GB/s {v['frac_hbm']:.3f}  isolated {v['isolated_us']:6.2f}  step {v['step_us']:6.2f}"
          f"  fused {v.get('fused_step_us', float('nan')):6.2f}")
