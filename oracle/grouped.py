"""Oracle for NEXT-3: group-wise weight scales -- TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

Reading R18: the paper's QoQ comparison uses group-wise weight scales "with a
group size of 128"; with the FMPQ block as the group, every (128-channel block b,
output channel n) has its own scale s_w[b, n], and dequantisation becomes

    y[m, n] = sum_b s_a[m, b] * s_w[b, n] * acc_b[m, n]        (binary64, b ascending)

with acc_b the exact per-block integer accumulators of oracle.gemm_blocks.

Parity status: pinned (equal block scales reduce to the per-channel oracle.dequant; an exact
rational evaluation on config 1; the quantisation error bound against the unquantised product).
"""
from __future__ import annotations

import numpy as np


def dequant_grouped(acc: np.ndarray, s_a: np.ndarray, s_wg: np.ndarray) -> np.ndarray:
    """acc [nb, M, N] int64, s_a [M, nb] float32, s_wg [nb, N] float32 -> y [M, N] float64."""
    nb, M, N = acc.shape
    y = np.zeros((M, N), dtype=np.float64)
    for b in range(nb):
        y += (s_a[:, b].astype(np.float64)[:, None] * s_wg[b].astype(np.float64)[None, :]) * acc[b].astype(np.float64)
    return y
