"""Stress: repeat the orientation-2 stream-K parity case many times in one process; report the
first failing iteration (a sticky CUDA error stops the loop)."""
import sys, os
import numpy as np
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_asplos_liu0rxpwl0w25_b200 as cb  # noqa: E402
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth  # noqa: E402
import oracle  # noqa: E402
which = sys.argv[2] if len(sys.argv) > 2 else "all"
cases = []
if which in ("all", "prefill"):
    cases += [(300, 1152, 1, 2, 23), (230, 2048, 1, 2, 23), (129, 256, 1, 2, 23), (1000, 384, 1, 2, 23),
              (300, 1152, 0, 2, 23), (512, 1024, 1, 3, 46)]
if which in ("all", "pair"):
    cases += [(512, 1280, 1, 3, 46, 160), (300, 1152, 1, 3, 30, 192), (700, 1024, 1, 3, 40, 128),
              (256, 2048, 0, 3, 20, 256), (600, 768, 1, 3, 14, 256)]
if which in ("all", "decode"):
    cases += [(1, 2048, 1, 1, 37), (16, 1024, 1, 1, 23), (32, 2048, 1, 1, 148), (100, 1152, 1, 1, 37),
              (7, 4096, -1, 1, 0), (64, 512, 2, 1, 13)]
n_iter = int(sys.argv[1]) if len(sys.argv) > 1 else 50
refs = {}
for it in range(n_iter):
    for case in cases:
        M, N, sm, ori, nsm = case[:5]
        tw = case[5] if len(case) > 5 else 0
        key = (M, N)
        if key not in refs:
            p = synth.make_problem(M, 1024, N, frac=0.25, seed=M + N)
            refs[key] = (p, oracle.w4ax(p.x, p.tags, p.w, p.s_w)[0])
        p, yref = refs[key]
        act, sc = cb.quantize_act(torch.from_numpy(p.x).cuda(), p.tags)
        wp = cb.pack_weight(torch.from_numpy(p.w).cuda())
        plan = cb.Plan(M, N, 1024, p.tags, split_mode=sm, num_sms=nsm, orientation=ori, tile_w=tw)
        y = cb.w4ax_gemm(plan, act, sc, wp, torch.from_numpy(p.s_w).cuda(), out_dtype=torch.float32)
        try:
            torch.cuda.synchronize()
        except Exception as e:
            print("FAIL iter", it, "case", case, repr(e)[:200])
            sys.exit(1)
        if not np.allclose(y.cpu().numpy(), yref, rtol=1e-3, atol=1e-2):
            print("WRONG iter", it, "case", case)
            sys.exit(1)
print("ok", n_iter)
