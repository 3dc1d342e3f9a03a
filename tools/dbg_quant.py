"""Diagnostic: first quantisation mismatches against the oracle for one seeded problem."""
import os, sys
import numpy as np
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import paper_conf_asplos_liu0rxpwl0w25_b200 as cb
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth
import oracle
from _layout import decode_act
M, K = int(sys.argv[1]), int(sys.argv[2])
p = synth.make_problem(M, K, 128, frac=0.05, seed=M + K)
act, sc = cb.quantize_act(torch.from_numpy(p.x).cuda(), p.tags)
codes, scales, qsum, corr = decode_act(act.cpu().numpy(), sc.cpu().numpy(), p.M, p.K, p.tags)
rc, rs = oracle.quantize(p.x, p.tags)
bad = np.argwhere(codes != rc)
print("tags int8 blocks", np.nonzero(p.tags)[0].tolist(), "mismatches", len(bad))
for m, k in bad[:12]:
    b = k // 128
    print(f"m {m} k {k} block {b} tag {p.tags[b]} x {float(p.x[m,k]):.6g} gpu {codes[m,k]} ref {rc[m,k]} s_gpu {scales[m,b]:.6g} s_ref {rs[m,b]:.6g}")
print("scales equal", np.array_equal(scales[:M].view(np.uint32), rs.view(np.uint32)))
