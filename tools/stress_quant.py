"""Stress: repeat kernel 1 in all its forms (identity, cluster-split for small M, fused
permutation staged / gathered) and the KV4 kernels; every result is compared bit-exactly with
the first iteration's, which is checked against the oracle."""
import os, sys
import numpy as np
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_asplos_liu0rxpwl0w25_b200 as cb  # noqa: E402
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth  # noqa: E402
import oracle  # noqa: E402
from oracle import calibrate as ocal  # noqa: E402
n_iter = int(sys.argv[1]) if len(sys.argv) > 1 else 50
cases = [(1, 28672, False), (32, 28672, True), (300, 8192, False), (5, 8192, True), (1000, 2048, False)]
base = {}
for it in range(n_iter):
    for (M, K, use_perm) in cases:
        key = (M, K, use_perm)
        if key not in base:
            p = synth.make_problem(M, K, 128, frac=0.1, seed=M + K)
            perm = np.random.default_rng(K).permutation(K).astype(np.int32) if use_perm else None
            base[key] = [p, perm, None]
        p, perm, ref = base[key]
        pd = torch.from_numpy(perm).cuda() if perm is not None else None
        act, sc = cb.quantize_act(torch.from_numpy(p.x).cuda(), p.tags, perm=pd)
        try:
            torch.cuda.synchronize()
        except Exception as e:
            print("FAIL iter", it, key, repr(e)[:200]); sys.exit(1)
        a = act.cpu().numpy()[: M * K].copy()
        if ref is None:
            xp = ocal.permute_channels(p.x, perm) if perm is not None else p.x
            codes, _ = oracle.quantize(xp, p.tags)
            base[key][2] = a
        elif not np.array_equal(a, ref):
            print("WRONG iter", it, key); sys.exit(1)
    kv = torch.from_numpy(synth.make_kv(4096, 1024, np.random.default_rng(1))).cuda()
    c, s, m = cb.kv4_quantize(kv, 128)
    torch.cuda.synchronize()
print("ok", n_iter)
