"""NEXT-4: INT4 KV-cache quantisation (reading R17).

CPU pins of the oracle (oracle/kv4.py) against things other than itself: a pure-Python
brute force over exact rationals (Fraction) with explicit binary32 rounding, the round-trip
error bound, the min/max codes, constant groups and ragged last groups; plus ABI validation
of the two C entry points without a GPU."""
import ctypes
from fractions import Fraction

import numpy as np
import pytest

from oracle import kv4 as okv
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth
from test_oracle_pins import f32_round


def f32(v: Fraction) -> Fraction:
    """Round an exact rational to the nearest binary32 (ties to even), exactly."""
    return f32_round(v)


def brute(x: np.ndarray, G: int):
    T, C = x.shape
    q = np.zeros((T, C), np.int64)
    for c in range(C):
        for g0 in range(0, T, G):
            col = [Fraction(float(v)) for v in x[g0:g0 + G, c]]
            lo, hi = min(col), max(col)
            d = f32(hi - lo)
            r = Fraction(0) if d == 0 else f32(Fraction(15) / d)
            for i, v in enumerate(col):
                t = f32(f32(v - lo) * r)
                fl = t.numerator // t.denominator
                rem = t - fl
                n = fl + (1 if rem > Fraction(1, 2) or (rem == Fraction(1, 2) and fl % 2 == 1) else 0)
                q[g0 + i, c] = min(max(n, 0), 15)
    return q


@pytest.mark.parametrize("T,C,G", [(40, 8, 32), (64, 4, 64), (7, 3, 32)])
def test_kv4_quantize_brute_force(T, C, G):
    rng = np.random.default_rng(T * C)
    x = synth.make_kv(T, C, rng, outlier_channels=1).astype(np.float32)
    q, s, mn = okv.quantize(x, G)
    assert np.array_equal(q.astype(np.int64), brute(x, G))
    ng = (T + G - 1) // G
    for g in range(ng):
        xs = x[g * G:(g + 1) * G]
        assert np.array_equal(mn[g], xs.min(0))
        d = (xs.max(0) - xs.min(0)).astype(np.float32)
        assert np.array_equal(s[g], np.where(d == 0, 0, d / np.float32(15)).astype(np.float32))


@pytest.mark.parametrize("G", [32, 128])
def test_kv4_roundtrip_bound_and_extremes(G):
    rng = np.random.default_rng(G)
    x = synth.make_kv(300, 64, rng).astype(np.float32)     # ragged last group (300 % G != 0)
    q, s, mn = okv.quantize(x, G)
    xh = okv.dequantize(q, s, mn, G)
    g = np.arange(300) // G
    bound = s[g] / 2 * (1 + 2.0 ** -20) + 2.0 ** -22 * (np.abs(mn[g]) + np.abs(x))
    assert np.all(np.abs(xh - x) <= bound)
    for gi in range(g.max() + 1):
        xs, qs = x[g == gi], q[g == gi]
        assert np.all(qs[np.argmin(xs, 0), np.arange(64)] == 0)
        assert np.all(qs[np.argmax(xs, 0), np.arange(64)] == 15)


def test_kv4_constant_group_exact_and_pack_roundtrip():
    x = np.full((64, 8), 3.25, np.float32)
    x[:, 1] = -7.0
    q, s, mn = okv.quantize(x, 32)
    assert np.all(q == 0) and np.all(s == 0)
    assert np.array_equal(okv.dequantize(q, s, mn, 32), x)
    rng = np.random.default_rng(1)
    qq = rng.integers(0, 16, size=(5, 16), dtype=np.uint8)
    p = okv.pack(qq)
    assert p[0, 0] == (qq[0, 0] | (qq[0, 1] << 4))
    assert np.array_equal(okv.unpack(p), qq)


def test_kv4_abi_validation_without_gpu():
    cb = pytest.importorskip("paper_conf_asplos_liu0rxpwl0w25_b200")
    L = cb.lib()
    v = ctypes.c_void_p(256)
    assert L.comet_kv4_quantize(v, 0, 10, 100, 100, 128, v, v, v, None) == 2     # C % 64
    assert L.comet_kv4_quantize(v, 0, 10, 128, 128, 100, v, v, v, None) == 2     # group
    assert L.comet_kv4_quantize(v, 0, 10, 128, 120, 128, v, v, v, None) == 3     # ld < C
    assert L.comet_kv4_dequantize(v, v, v, 10, 128, 128, v, 2, 128, None) == 1   # f32 output
    assert L.comet_kv4_quantize(None, 0, 10, 128, 128, 128, v, v, v, None) == 1
