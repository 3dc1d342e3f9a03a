"""Distribution of the pair kernel's MMA issue period over a whole launch (tools/trace_gemm.py
output of a build with COMET_TRACE=1 COMET_TRACE_MASK=0x0808: MMA issue events only, the
least perturbing trace).  Separates the steady-state period from the long gaps (tile
boundaries, fix-ups).  Usage: python tools/trace_period.py trace.json [cta]"""
import json
import sys

import numpy as np

d = json.load(open(sys.argv[1]))
cta = int(sys.argv[2]) if len(sys.argv) > 2 else 0
t = np.array(d["trace"][cta], dtype=np.int64)
ev, od = t[3], t[11]
n = int((ev > 0).sum()) + int((od > 0).sum())
iss = np.zeros(n, dtype=np.int64)
iss[0::2] = ev[: (n + 1) // 2]
iss[1::2] = od[: n // 2]
iss = iss[iss > 0]
dd = np.diff(iss)
tot = iss[-1] - iss[0]
print(f"CTA {cta}: {len(iss)} K-blocks, {tot} clk, mean period {tot / (len(iss) - 1):.0f}")
for p in (10, 25, 50, 75, 90, 99):
    print(f"  p{p:<3d} {np.percentile(dd, p):8.0f}")
big = dd[dd > 2000]
print(f"  gaps > 2000 clk: {len(big)}, {big.sum()} clk = {100 * big.sum() / tot:.1f} % of the span; "
      f"period excluding them {(tot - big.sum()) / (len(dd) - len(big)):.0f}")
print("  largest gaps at K-block index:", [(int(i), int(dd[i])) for i in np.argsort(-dd)[:12]])
