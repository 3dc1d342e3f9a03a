"""Oracle for the FMPQ channel permutation -- TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

Written from P:L138-144 / Fig. 4(d): "we utilize sampled activations from the calibration dataset
to locate outlier channels and apply permutation to group these channels into a single block.
To further maintain computational equivalence, the corresponding positions in the weight matrix
also need to be permuted."  Reading R16: an outlier channel is one whose
calibration max-abs exceeds `ratio` (10, the "tenfold" of P:L126) times the median channel
max-abs; the permutation lists the outlier channels first (ascending), then the rest
(ascending); the ceil(n_outliers / 128) blocks that then hold outliers are the INT8 blocks.

Parity status: pinned (planted outliers recovered; permutation validity and order by brute
force; the median against Python's statistics.median; computational equivalence X'W'^T = XW^T
within the quantisation bound; the paper's "< 20 % of blocks INT8" on Fig. 3-like inputs).
"""
from __future__ import annotations

import numpy as np

BLOCK = 128


def channel_amax(x: np.ndarray) -> np.ndarray:
    """amax[k] = max over calibration rows of |x[m, k]| (float16 input -> float32, exact)."""
    return np.abs(x.astype(np.float32)).max(axis=0)


def median(amax: np.ndarray) -> float:
    """Median in binary64: the central order statistic, or the mean of the two central ones."""
    v = np.sort(np.asarray(amax, dtype=np.float64))
    K = v.shape[0]
    if K % 2 == 1:
        return float(v[K // 2])
    return float((v[K // 2 - 1] + v[K // 2]) / 2.0)


def calibrate_perm(amax: np.ndarray, ratio: float = 10.0):
    """-> (perm int32 [K], tags uint8 [K/128], n_outliers)."""
    a = np.asarray(amax, dtype=np.float32)
    K = a.shape[0]
    thr = float(ratio) * median(a)
    is_out = a.astype(np.float64) > thr
    outl = [k for k in range(K) if is_out[k]]
    rest = [k for k in range(K) if not is_out[k]]
    perm = np.array(outl + rest, dtype=np.int32)
    n8 = (len(outl) + BLOCK - 1) // BLOCK
    tags = np.array([1 if b < n8 else 0 for b in range(K // BLOCK)], dtype=np.uint8)
    return perm, tags, len(outl)


def permute_channels(x: np.ndarray, perm: np.ndarray) -> np.ndarray:
    """x'[:, k] = x[:, perm[k]] (the same map applied to activations and weights)."""
    return np.ascontiguousarray(x[:, np.asarray(perm, dtype=np.int64)])
