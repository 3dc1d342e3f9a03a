"""Time the decode-regime GEMM (BASELINE config 5) alone: LLaMA-3-70B layers at small M, L2
flushed before every launch.  Prints one line per (layer, M) and a JSON summary on the last line.

  python tools/decode_time.py [--Ms 1,4,8,32] [--tile-n 0] [--split-mode -1] [--orientation 0] [--iters 20]
"""
import argparse
import json
import os
import statistics
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_asplos_liu0rxpwl0w25_b200 as cb  # noqa: E402
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth  # noqa: E402

LAYERS = [("gate_up", 8192, 28672), ("down", 28672, 8192), ("qkv", 8192, 10240)]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--Ms", default="1,4,8,32")
    ap.add_argument("--tile-n", type=int, default=0)
    ap.add_argument("--split-mode", type=int, default=-1)
    ap.add_argument("--orientation", type=int, default=0, help="0 = auto, 1 = TMEM decode kernel, 4 = warp-level")
    ap.add_argument("--iters", type=int, default=20)
    ap.add_argument("--layers", default="gate_up,down,qkv")
    ap.add_argument("--flush", type=int, default=1, help="1 = write + read 256 MiB before every launch")
    ap.add_argument("--sleep-cycles", type=float, default=4e7)
    a = ap.parse_args()
    dev = torch.device("cuda", 0)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    flush_rd = torch.ones(64 << 20, dtype=torch.float32, device=dev)   # 256 MiB, read to leave L2 clean
    hbm = 6448.4
    p = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "MEASURED_PEAKS.json")
    if os.path.exists(p):
        hbm = json.load(open(p))["hbm_gbs"]
    res = {}
    for name, K, N in LAYERS:
        if name not in a.layers.split(","):
            continue
        rng = np.random.default_rng(7)
        tags = synth.make_tags(K, 0.05, rng)
        w, s_w = synth.make_weights(N, K, rng)
        wp = cb.pack_weight(torch.from_numpy(w).to(dev))
        swd = torch.from_numpy(s_w).to(dev)
        for M in [int(m) for m in a.Ms.split(",")]:
            x = torch.from_numpy(synth.make_activations(M, K, tags, rng)).to(dev)
            plan = cb.Plan(M, N, K, tags, tile_n=a.tile_n, split_mode=a.split_mode, orientation=a.orientation)
            act, sc = cb.quantize_act(x, tags)
            y = torch.empty((M, N), dtype=torch.float16, device=dev)
            evs = []
            cb.w4ax_gemm(plan, act, sc, wp, swd, out=y)
            torch.cuda.synchronize()
            # queue every launch behind a GPU sleep so host-side launch latency never shows up
            # as GPU idle time inside the events
            torch.cuda._sleep(int(a.sleep_cycles))
            for i in range(a.iters + 3):
                if a.flush:
                    flush.fill_(i & 0xFF)
                    flush_rd.sum()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                cb.w4ax_gemm(plan, act, sc, wp, swd, out=y)
                e1.record()
                evs.append((e0, e1))
            torch.cuda.synchronize()
            us = statistics.median(e0.elapsed_time(e1) for e0, e1 in evs[3:]) * 1e3
            nbytes = N * K // 2 + N * 4 + act.numel() + sc.numel() * 4 + M * N * 2
            gbs = nbytes / (us * 1e-6) / 1e9
            info = plan.info()
            res[f"{name}_M{M}"] = {"us": round(us, 2), "GB/s": round(gbs, 1), "frac": round(gbs / hbm, 3)}
            print(f"{name:8s} M={M:3d} tile_n={info['tile_n']:3d} split={info['split_mode']} "
                  f"{us:8.2f} us {gbs:8.1f} GB/s {gbs / hbm:.3f}", flush=True)
        del wp
    print(json.dumps(res))


if __name__ == "__main__":
    main()
