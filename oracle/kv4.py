"""Oracle for NEXT-4: KV-cache INT4 quantisation -- TEST INFRASTRUCTURE ONLY (see
oracle/__init__.py).

Written from P:L146 ("we use a channel-wise 4-bit quantization strategy for the KV cache") and
P:L242 ("channel-wise asymmetric INT4 group quantization for the KV cache"), with reading R17
(DESIGN.md §3): a K or V cache tensor X[T tokens][C channels] (C = KV heads x head_dim) is cut
into groups of G consecutive tokens; every (group g, channel c) gets its own asymmetric
min-max quantiser (min as the offset, 15 steps), in IEEE binary32 with no contraction:

    mn = min_t x[t,c],  mx = max_t x[t,c]          (t in group g)
    d = mx - mn;  s = d / 15;  r = 15 / d          (d == 0: s = 0, r = 0)
    q = clamp(rint_half_even((x - mn) * r), 0, 15)
    x_hat = mn + q * s                             (two binary32 roundings), then -> f16/bf16 (RN)

Every step is numpy binary32 arithmetic (each operation correctly rounded, never fused).

Parity status: pinned (pure-Python brute force over exact rationals on small cases; the
round-trip bound |x - x_hat| <= s/2 (1 + 2^-20) + 2^-22 (|mn| + |x|); min -> code 0 and
max -> code 15; constant groups reproduced exactly; ragged last group).
"""
from __future__ import annotations

import numpy as np


def quantize(x: np.ndarray, group: int = 128):
    """x: [T, C] float32 values (exact f16/bf16).  Returns (q uint8 [T, C] in 0..15,
    s float32 [ng, C], mn float32 [ng, C]) with ng = ceil(T / group)."""
    x = np.asarray(x, dtype=np.float32)
    T, C = x.shape
    ng = (T + group - 1) // group
    q = np.zeros((T, C), dtype=np.uint8)
    s = np.zeros((ng, C), dtype=np.float32)
    mn = np.zeros((ng, C), dtype=np.float32)
    for g in range(ng):
        xs = x[g * group: min(T, (g + 1) * group)]
        lo = xs.min(axis=0)
        hi = xs.max(axis=0)
        d = (hi - lo).astype(np.float32)
        with np.errstate(divide="ignore", invalid="ignore"):
            sg = np.where(d == 0, np.float32(0), d / np.float32(15)).astype(np.float32)
            rg = np.where(d == 0, np.float32(0), np.float32(15) / d).astype(np.float32)
        t = ((xs - lo[None, :]).astype(np.float32) * rg[None, :]).astype(np.float32)
        q[g * group: min(T, (g + 1) * group)] = np.clip(np.rint(t), 0, 15).astype(np.uint8)
        s[g] = sg
        mn[g] = lo
    return q, s, mn


def dequantize(q: np.ndarray, s: np.ndarray, mn: np.ndarray, group: int = 128) -> np.ndarray:
    """x_hat[t, c] = mn[g, c] + q[t, c] * s[g, c] in binary32 (g = t // group)."""
    T, C = q.shape
    g = np.arange(T) // group
    prod = (q.astype(np.float32) * s[g]).astype(np.float32)
    return (mn[g] + prod).astype(np.float32)


def pack(q: np.ndarray) -> np.ndarray:
    """Packed codes [T, C/2]: byte j = q[:, 2j] | q[:, 2j+1] << 4 (include/comet.h)."""
    return (q[:, 0::2] | (q[:, 1::2] << 4)).astype(np.uint8)


def unpack(p: np.ndarray) -> np.ndarray:
    T, H = p.shape
    q = np.empty((T, 2 * H), dtype=np.uint8)
    q[:, 0::2] = p & 0xF
    q[:, 1::2] = p >> 4
    return q
