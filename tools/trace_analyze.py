"""Summarise a tools/trace_gemm.py timeline of the pair kernel (orientation 3; build with
COMET_TRACE=1, or COMET_DIAG=1 which adds the ablation hooks).

Event rows (per CTA, clock64), K-block j of the CTA's sequence:
  14/0  producer before its slot_free wait / after issuing the loads of j
  1/3   MMA issuer of even j (index j/2) before / after its mma_ready wait (= MMA issue)
  13/11 the same for odd j
  5/2/4 widen group 0 (even j, index j/2): after full wait / stores done / arrive
  12/6  promotion warp 0 before / after its acc_full wait for j
  8/9   its first TMEM load issued / landed; 10 accumulator released (batched mode); 7 done
Prints medians of the steady-state intervals.
Usage: python tools/trace_analyze.py trace.json [cta]"""
import json
import sys

import numpy as np

d = json.load(open(sys.argv[1]))
cta = int(sys.argv[2]) if len(sys.argv) > 2 else 0
t = np.array(d["trace"][cta], dtype=np.int64)          # [16][1024]
n_even = int((t[3] > 0).sum())
lo, hi = max(4, n_even // 8), min(n_even, 500) - 4


def med(v):
    v = np.asarray(v)
    return f"median {np.median(v):7.0f}  p10 {np.percentile(v, 10):7.0f}  p90 {np.percentile(v, 90):7.0f}"


def issue(j):           # MMA issue time of K-block j
    return t[3][j // 2] if j % 2 == 0 else t[11][j // 2]


js = [j for j in range(2 * lo, 2 * hi) if t[6][j + 2] > 0 and issue(j + 2) > 0]
print(f"CTA {cta}: {len(js)} steady-state K-blocks")
per = np.diff([issue(j) for j in js])
print("  MMA issue period                 ", med(per))
print("  producer issue(j) -> MMA issue(j)", med([issue(j) - t[0][j] for j in js]))
print("  producer wait for slot_free      ", med([t[0][j] - t[14][j] for j in js]))
ev = [j for j in js if j % 2 == 0]
print("  TMA issue -> widen start (even j)", med([t[5][j // 2] - t[0][j] for j in ev]))
print("  widen start -> done              ", med([t[2][j // 2] - t[5][j // 2] for j in ev]))
print("  widen arrive -> MMA issue        ", med([issue(j) - t[4][j // 2] for j in ev]))
print("  MMA wait (even issuer)           ", med([t[3][j // 2] - t[1][j // 2] for j in ev]))
print("  MMA issue(j) -> promo wake(j)    ", med([t[6][j] - issue(j) for j in js]))
print("  promo wait for acc_full          ", med([t[6][j] - t[12][j] for j in js]))
print("  promo wake -> first load landed  ", med([t[9][j] - t[6][j] for j in js]))
if (t[10] > 0).any():
    print("  promo wake -> released           ", med([t[10][j] - t[6][j] for j in js]))
print("  promo wake -> done               ", med([t[7][j] - t[6][j] for j in js]))
if (t[10] > 0).any():
    print("  released(j) -> MMA issue(j+2)    ", med([issue(j + 2) - t[10][j] for j in js]))
    print("  released(j) -> promo wait(j+1)   ", med([t[12][j + 1] - t[10][j] for j in js]))
print("  promo done(j) -> MMA issue(j+2)  ", med([issue(j + 2) - t[7][j] for j in js]))
print("  MMA issue(j) -> MMA issue(j+2)   ", med([issue(j + 2) - issue(j) for j in js]))
# tile boundaries (whole 64-K-block tiles, gate_up): promotion gap done(j) -> next wait(j+1) and
# the MMA issue spacing across the boundary, against the interior
nkb = int(sys.argv[3]) if len(sys.argv) > 3 else 64
bj = [j for j in range(8, min(n_even * 2, 1000) - 2) if (j + 1) % nkb == 0 and t[7][j] > 0 and t[12][j + 1] > 0]
ij = [j for j in range(8, min(n_even * 2, 1000) - 2) if (j + 1) % nkb != 0 and t[7][j] > 0 and t[12][j + 1] > 0]
if bj:
    print(f"  tile boundaries: {len(bj)}")
    print("  promo done(j) -> next wait, boundary", med([t[12][j + 1] - t[7][j] for j in bj]))
    print("  promo done(j) -> next wait, interior", med([t[12][j + 1] - t[7][j] for j in ij]))
    print("  MMA issue(j) -> issue(j+1), boundary", med([issue(j + 1) - issue(j) for j in bj if issue(j + 1) > 0]))
    print("  MMA issue(j) -> issue(j+1), interior", med([issue(j + 1) - issue(j) for j in ij if issue(j + 1) > 0]))
    print("  promo wake(j+1) - promo done(j), boundary", med([t[6][j + 1] - t[7][j] for j in bj]))
# epilogue phases (event 15 at 4 i + {0: before the WG-group barrier, 1: after it, 2: after chunk
# 1's store, 3: after the last chunk}) against the tile's last promotion done
if bj:
    e15 = t[15]
    rows = []
    for k, j in enumerate(bj):
        i = (j + 1) // nkb - 1
        if e15[4 * i + 3] > 0:
            rows.append((e15[4 * i] - t[7][j], e15[4 * i + 1] - e15[4 * i], e15[4 * i + 2] - e15[4 * i + 1],
                         e15[4 * i + 3] - e15[4 * i + 2], t[12][j + 1] - e15[4 * i + 3]))
    if rows:
        r = np.array(rows)
        print("  epilogue: done->start, group barrier, chunks 0-1, chunks 2-3, ->next wait (medians)",
              np.median(r, axis=0).astype(int).tolist())
