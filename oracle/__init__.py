"""CPU oracle for the COMET W4Ax hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its ``cpu_baseline`` leg and
``--impl reference``) may import this package.  The product path
(``paper_conf_asplos_liu0rxpwl0w25_b200``) never imports it and shares no code with it.

The arithmetic lives in ``comet_oracle.c`` (plain C, binary32 quantisation exactly as
written in the paper's FMPQ description, int64 GEMM, binary64 dequantisation); this module
only compiles it with gcc and marshals numpy arrays.  ``planner.py`` holds the schedule
oracle (makespan of a tile->SM assignment, P:L212-228 / Fig. 8).

Parity status per function:
  quantize        pinned (brute force, invariants I2/I3/I5/I6, odd symmetry, paper bound)
  gemm_blocks     pinned (python big-int brute force, numpy int64 matmul I8, I1)
  dequant         pinned (closed form I4, exact Fraction check)
  w4ax_rows       pinned (equals the three functions above, which are pinned)
  planner.*       pinned (Fig. 8 worked example)
  calibrate.*     pinned (NEXT-1: planted outliers, brute-force order, statistics.median, P:L140
                  equivalence bound, "< 20 %" claim) -- oracle/calibrate.py
  kv4.*           pinned (NEXT-4: exact-rational brute force, round-trip bound) -- oracle/kv4.py
  grouped.*       pinned (NEXT-3: per-channel reduction, exact Fraction, error bound) -- oracle/grouped.py
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "comet_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

BLOCK = 128  # k = 128 channels per FMPQ block


def build(force: bool = False) -> str:
    """Compile comet_oracle.c -> liboracle.so (gcc, strict IEEE binary32)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        cmd = ["gcc", "-O2", "-fno-fast-math", "-ffp-contract=off", "-fopenmp", "-shared",
               "-fPIC", "-o", _LIB + ".tmp", _SRC, "-lm"]
        subprocess.check_call(cmd)
        os.replace(_LIB + ".tmp", _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        P = ctypes.c_void_p
        I64 = ctypes.c_int64
        lib.oracle_quantize.argtypes = [P, ctypes.c_int, I64, I64, P, P, P]
        lib.oracle_gemm_blocks.argtypes = [P, P, I64, I64, I64, P, I64, P]
        lib.oracle_dequant.argtypes = [P, P, P, I64, I64, P, I64, P]
        lib.oracle_w4ax_rows.argtypes = [P, ctypes.c_int, I64, I64, P, P, P, I64, P, I64,
                                         P, P, P, P]
        for f in (lib.oracle_quantize, lib.oracle_gemm_blocks, lib.oracle_dequant,
                  lib.oracle_w4ax_rows, lib.oracle_num_threads):
            f.restype = ctypes.c_int
        _lib = lib
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def _as_u16(x: np.ndarray) -> tuple[np.ndarray, int]:
    """Accept float16 arrays or uint16 bit patterns tagged by dtype name."""
    if x.dtype == np.float16:
        return np.ascontiguousarray(x).view(np.uint16), 0
    raise TypeError("use quantize(..., bf16_bits=...) for bfloat16 input")


def num_threads() -> int:
    return int(_load().oracle_num_threads())


def quantize(x: np.ndarray, tags: np.ndarray, *, bf16_bits: bool = False):
    """FMPQ block quantisation.

    x: [M, K] float16, or uint16 bfloat16 bit patterns with ``bf16_bits=True``.
    tags: [K/128] uint8, 1 = INT8 (outlier) block, 0 = INT4 block.
    Returns (codes int8 [M, K], scales float32 [M, K/128]).
    """
    if bf16_bits:
        assert x.dtype == np.uint16
        xb, is_bf16 = np.ascontiguousarray(x), 1
    else:
        xb, is_bf16 = _as_u16(x)
    M, K = xb.shape
    tags = np.ascontiguousarray(tags, dtype=np.uint8)
    assert tags.shape == (K // BLOCK,)
    codes = np.empty((M, K), dtype=np.int8)
    scales = np.empty((M, K // BLOCK), dtype=np.float32)
    rc = _load().oracle_quantize(_ptr(xb), is_bf16, M, K, _ptr(tags), _ptr(codes), _ptr(scales))
    if rc != 0:
        raise ValueError(f"oracle_quantize rc={rc}")
    return codes, scales


def gemm_blocks(q: np.ndarray, w: np.ndarray, rows=None) -> np.ndarray:
    """acc[b, i, n] = sum_{k in block b} q[rows[i], k] * w[n, k] (exact int64)."""
    q = np.ascontiguousarray(q, dtype=np.int8)
    w = np.ascontiguousarray(w, dtype=np.int8)
    M, K = q.shape
    N = w.shape[0]
    rows = np.arange(M, dtype=np.int64) if rows is None else np.ascontiguousarray(rows, np.int64)
    acc = np.empty((K // BLOCK, rows.shape[0], N), dtype=np.int64)
    rc = _load().oracle_gemm_blocks(_ptr(q), _ptr(w), M, N, K, _ptr(rows), rows.shape[0], _ptr(acc))
    if rc == -2:
        raise OverflowError("a per-block accumulator does not fit int32")
    if rc != 0:
        raise ValueError(f"oracle_gemm_blocks rc={rc}")
    return acc


def dequant(acc: np.ndarray, s_a: np.ndarray, s_w: np.ndarray, rows=None) -> np.ndarray:
    """y[i, n] = s_w[n] * sum_b s_a[rows[i], b] * acc[b, i, n] in binary64."""
    acc = np.ascontiguousarray(acc, dtype=np.int64)
    s_a = np.ascontiguousarray(s_a, dtype=np.float32)
    s_w = np.ascontiguousarray(s_w, dtype=np.float32)
    nb, nrows, N = acc.shape
    rows = np.arange(nrows, dtype=np.int64) if rows is None else np.ascontiguousarray(rows, np.int64)
    y = np.empty((nrows, N), dtype=np.float64)
    _load().oracle_dequant(_ptr(acc), _ptr(s_a), _ptr(s_w), N, nb, _ptr(rows), nrows, _ptr(y))
    return y


def w4ax(x: np.ndarray, tags: np.ndarray, w: np.ndarray, s_w: np.ndarray, *,
         bf16_bits: bool = False):
    """Whole path on all rows: returns (y float64 [M,N], acc_blocks int64 [nb,M,N], codes, scales)."""
    codes, scales = quantize(x, tags, bf16_bits=bf16_bits)
    acc = gemm_blocks(codes, w)
    y = dequant(acc, scales, s_w)
    return y, acc, codes, scales


def w4ax_rows(x: np.ndarray, tags: np.ndarray, w: np.ndarray, s_w: np.ndarray, rows,
              *, bf16_bits: bool = False):
    """Whole path for a sample of token rows (bounded memory at BASELINE sizes).

    Returns (y float64 [nrows, N], acc_sum int64 [nrows, N], codes int8 [nrows, K],
    scales float32 [nrows, nb]).
    """
    if bf16_bits:
        xb, is_bf16 = np.ascontiguousarray(x), 1
    else:
        xb, is_bf16 = _as_u16(x)
    M, K = xb.shape
    w = np.ascontiguousarray(w, dtype=np.int8)
    N = w.shape[0]
    s_w = np.ascontiguousarray(s_w, dtype=np.float32)
    tags = np.ascontiguousarray(tags, dtype=np.uint8)
    rows = np.ascontiguousarray(rows, dtype=np.int64)
    n = rows.shape[0]
    y = np.empty((n, N), np.float64)
    acc_sum = np.empty((n, N), np.int64)
    codes = np.empty((n, K), np.int8)
    scales = np.empty((n, K // BLOCK), np.float32)
    rc = _load().oracle_w4ax_rows(_ptr(xb), is_bf16, M, K, _ptr(tags), _ptr(w), _ptr(s_w), N,
                                  _ptr(rows), n, _ptr(y), _ptr(acc_sum), _ptr(codes), _ptr(scales))
    if rc == -2:
        raise OverflowError("a per-block accumulator does not fit int32")
    if rc != 0:
        raise ValueError(f"oracle_w4ax_rows rc={rc}")
    return y, acc_sum, codes, scales
