"""Seeded synthetic workloads (numpy only).  Shared by tests, bench and smoke.

Holds none of the method's arithmetic: it only draws inputs with the shapes and value
structure of the paper's workloads (DESIGN.md §4 "input recipe"):

* X: N(0, 1) activations, cast to float16 (bfloat16 bit patterns on request).
* tags: n8 = round(f * nb) INT8 ("outlier") blocks (at least 1 if f > 0) at seeded random
  block positions -- after COMET's channel permutation the outlier channels sit in a few
  128-channel blocks; FMPQ leaves < 20 % of blocks INT8, ~16 % on
  average and 8 % on LLaMA-1-30B.
* outliers: in every INT8 block, 4 seeded channels are scaled by U(20, 100): outliers are
  "< 1 %" of features with magnitudes "tenfold or even a hundredfold" the rest,
  concentrated in specific channels (Fig. 3).
* W: 4-bit weight codes uniform in [-8, 7] (stand-in for OmniQuant W4) and
  per-output-channel scales s_w = U(0.5, 1.5) / (8 sqrt(K)) so outputs are O(1).
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

BLOCK = 128


@dataclass(frozen=True)
class Layer:
    name: str
    K: int   # input channels
    N: int   # output channels


# LLaMA linear-layer shapes named in BASELINE.json configs.
LLAMA2_7B = (Layer("qkvo", 4096, 4096), Layer("gate_up", 4096, 11008), Layer("down", 11008, 4096))
LLAMA3_8B = (Layer("up", 4096, 14336), Layer("down", 14336, 4096))
LLAMA3_70B = (Layer("gate_up", 8192, 28672), Layer("down", 28672, 8192), Layer("qkv", 8192, 10240))


def bf16_bits_from_f32(a: np.ndarray) -> np.ndarray:
    """Round float32 -> bfloat16 (round-half-even) and return the uint16 bit patterns."""
    u = np.ascontiguousarray(a, dtype=np.float32).view(np.uint32).astype(np.uint64)
    lsb = (u >> 16) & 1
    r = ((u + 0x7FFF + lsb) >> 16).astype(np.uint16)
    return r


def bf16_bits_to_f32(b: np.ndarray) -> np.ndarray:
    return (np.ascontiguousarray(b, dtype=np.uint16).astype(np.uint32) << 16).view(np.float32)


def make_tags(K: int, frac: float, rng: np.random.Generator, n8: int | None = None) -> np.ndarray:
    nb = K // BLOCK
    if n8 is None:
        n8 = int(round(frac * nb))
        if frac > 0 and n8 == 0:
            n8 = 1
    tags = np.zeros(nb, dtype=np.uint8)
    if n8 > 0:
        tags[rng.choice(nb, size=n8, replace=False)] = 1
    return tags


def make_activations(M: int, K: int, tags: np.ndarray, rng: np.random.Generator,
                     *, bf16: bool = False, outliers_per_block: int = 4,
                     lo: float = 20.0, hi: float = 100.0):
    """X[M, K] ~ N(0,1) with `outliers_per_block` boosted channels in every INT8 block.
    Returns float16 array, or uint16 bf16 bit patterns when bf16=True."""
    x = rng.standard_normal((M, K), dtype=np.float32)
    for b in np.nonzero(tags)[0]:
        ch = b * BLOCK + rng.choice(BLOCK, size=outliers_per_block, replace=False)
        x[:, ch] *= rng.uniform(lo, hi, size=outliers_per_block).astype(np.float32)
    if bf16:
        return bf16_bits_from_f32(x)
    return x.astype(np.float16)


def make_weights(N: int, K: int, rng: np.random.Generator):
    """INT4 codes in [-8, 7] and per-output-channel scales."""
    w = rng.integers(-8, 8, size=(N, K), dtype=np.int8)
    s_w = (rng.uniform(0.5, 1.5, size=N) / (8.0 * np.sqrt(K))).astype(np.float32)
    return w, s_w


@dataclass
class Problem:
    x: np.ndarray        # [M,K] float16 (or uint16 bf16 bits if bf16)
    tags: np.ndarray     # [K/128] uint8
    w: np.ndarray        # [N,K] int8 codes in [-8,7]
    s_w: np.ndarray      # [N] float32
    bf16: bool = False

    @property
    def M(self): return self.x.shape[0]

    @property
    def K(self): return self.x.shape[1]

    @property
    def N(self): return self.w.shape[0]


def make_problem(M: int, K: int, N: int, *, frac: float = 0.05, seed: int = 0,
                 bf16: bool = False, n8: int | None = None) -> Problem:
    rng = np.random.default_rng(seed)
    tags = make_tags(K, frac, rng, n8=n8)
    x = make_activations(M, K, tags, rng, bf16=bf16)
    w, s_w = make_weights(N, K, rng)
    return Problem(x=x, tags=tags, w=w, s_w=s_w, bf16=bf16)


@dataclass
class ExactProblem(Problem):
    """A Problem whose inputs are built from chosen integer codes (see make_exact_problem)."""
    q: np.ndarray = None      # [M, K] int16: the codes every block is built from
    e: np.ndarray = None      # [M, nb] int: x[m, block b] = q * 2^e[m, b]
    f: np.ndarray = None      # [N] int: s_w[n] = 2^f[n]


EXACT_SPECIAL_ROWS = ("zero", "all_pos", "alternating", "all_neg")


def make_exact_problem(M: int, K: int, N: int, *, frac: float = 0.05, seed: int = 0,
                       bf16: bool = False, n8: int | None = None,
                       special_rows: dict | None = None) -> ExactProblem:
    """Inputs on which the whole W4Ax path is EXACT in binary32, so a GEMM's FP32 output can be
    compared bit for bit (VERDICT r01 "integer exactness of the production kernels").

    Every (token m, block b) is built from integer codes q in [-qmax_b, qmax_b] (qmax 7 for
    INT4 blocks, 127 for INT8 blocks) with at least one element equal to +-qmax_b, as
    x = q * 2^e[m, b]; so amax = qmax_b 2^e, s_a = 2^e exactly and the quantised codes are q.
    Weight scales are powers of two, s_w[n] = 2^f[n].  Then y[m, n] = sum_b 2^(e[m,b]+f[n])
    acc_b[m, n] is a sum of integers times powers of two, and the exponents are limited so
    that sum_b 2^(e_b - min e) * c_b * sum_k |q| < 2^24 per row (c_b = 15 INT4, 8 INT8): every partial sum of every
    accumulation order (the INT4 blocks' offset-binary operand u = w + 8 included) is exact in
    binary32.  A single wrong accumulator code unit changes y by >= 2^(min e + f).

    special_rows maps a row index to one of EXACT_SPECIAL_ROWS: "zero" (an all-zero row, s_a =
    0), "all_pos" / "all_neg" (every code +-qmax: the largest |sum q w| of a block, e.g. 7 * 15
    * 128 = 13,440 against an all-7 weight row's offset-binary u = 15), "alternating" (codes
    +-qmax alternating: maximal cancellation).  Weight rows 0, 1, 2 and N-1 are all-7, all -8,
    alternating 7/-8 and all-7 (their u = 15, 0, 15/0).  Only input values are drawn here --
    none of the method's arithmetic."""
    rng = np.random.default_rng(seed)
    tags = make_tags(K, frac, rng, n8=n8)
    nb = K // BLOCK
    qmax = np.where(tags != 0, 127, 7).astype(np.int16)                 # [nb]
    qm = np.repeat(qmax, BLOCK)                                          # [K]
    q = (rng.integers(-(1 << 15), 1 << 15, size=(M, K)) % (2 * qm + 1) - qm).astype(np.int16)
    pos = rng.integers(0, BLOCK, size=(M, nb))
    sgn = rng.choice(np.array([-1, 1], np.int16), size=(M, nb))
    rows_i = np.repeat(np.arange(M), nb)
    cols_i = (np.tile(np.arange(nb), M) * BLOCK + pos.reshape(-1))
    q[rows_i, cols_i] = (sgn * qmax[None, :]).reshape(-1)
    special_rows = special_rows or {}
    for r, kind in special_rows.items():
        if not 0 <= r < M:
            continue
        if kind == "zero":
            q[r] = 0
        elif kind == "all_pos":
            q[r] = qm
        elif kind == "all_neg":
            q[r] = -qm
        elif kind == "alternating":
            q[r] = qm * np.where(np.arange(K) % 2 == 0, 1, -1).astype(np.int16)
        else:
            raise ValueError(kind)
    # block exponents: random in [e0, e0 + 3], flattened to e0 for rows that would not be exact
    # (|operand| <= 15 = max u for INT4 blocks, <= 8 = max |w| for INT8 blocks; a binary32 sum
    # of integers whose magnitudes total < 2^24 is exact in every order)
    e0 = -2
    e = rng.integers(e0, e0 + 4, size=(M, nb))
    absq = np.abs(q.astype(np.int64)).reshape(M, nb, BLOCK).sum(2) * np.where(tags != 0, 8, 15)[None, :]
    bound = (absq * (2.0 ** (e - e0))).sum(1)
    e[bound >= 2.0 ** 24] = e0
    assert np.all(absq.sum(1) < 2 ** 24), "row too large for an exact binary32 sum"
    xf = q.astype(np.float32) * np.repeat(np.exp2(e).astype(np.float32), BLOCK, axis=1)
    x = bf16_bits_from_f32(xf) if bf16 else xf.astype(np.float16)
    w = rng.integers(-8, 8, size=(N, K), dtype=np.int8)
    w[0] = 7
    if N > 1:
        w[1] = -8
    if N > 2:
        w[2] = np.where(np.arange(K) % 2 == 0, 7, -8)
    w[N - 1] = 7
    f = rng.integers(-9, -6, size=N)
    s_w = np.exp2(f).astype(np.float32)
    return ExactProblem(x=x, tags=tags, w=w, s_w=s_w, bf16=bf16, q=q, e=e, f=f)


def config1(seed: int = 1) -> Problem:
    """BASELINE config 1: single linear M=16 K=256 N=256, 2 blocks, 1 INT8 outlier block."""
    return make_problem(16, 256, 256, seed=seed, n8=1)


@dataclass
class UnpermutedProblem:
    """Activations BEFORE COMET's channel permutation: outliers in a few scattered channels
    (Fig. 3), plus an independent calibration sample with the same outlier channels
    ("sampled activations from the calibration dataset")."""
    x: np.ndarray          # [M, K] float16 (or uint16 bf16 bits)
    x_calib: np.ndarray    # [M_calib, K], same dtype
    w: np.ndarray          # [N, K] int8 codes
    s_w: np.ndarray        # [N] float32
    outlier_channels: np.ndarray   # sorted int64
    bf16: bool = False


def make_unpermuted_problem(M: int, K: int, N: int, *, n_outlier_channels: int | None = None,
                            channel_frac: float = 0.005, seed: int = 0, m_calib: int = 512,
                            bf16: bool = False, lo: float = 20.0, hi: float = 100.0) -> UnpermutedProblem:
    """N(0,1) activations with `n_outlier_channels` (default: channel_frac of K, at least 1)
    seeded channels scaled by U(lo, hi) -- "< 1 %" of features, 10x-100x."""
    rng = np.random.default_rng(seed)
    n = n_outlier_channels if n_outlier_channels is not None else max(1, int(round(channel_frac * K)))
    ch = np.sort(rng.choice(K, size=n, replace=False)).astype(np.int64)
    mag = rng.uniform(lo, hi, size=n).astype(np.float32)

    def draw(rows):
        x = rng.standard_normal((rows, K), dtype=np.float32)
        x[:, ch] *= mag
        return bf16_bits_from_f32(x) if bf16 else x.astype(np.float16)

    x = draw(M)
    xc = draw(m_calib)
    w, s_w = make_weights(N, K, rng)
    return UnpermutedProblem(x=x, x_calib=xc, w=w, s_w=s_w, outlier_channels=ch, bf16=bf16)


def make_kv(T: int, C: int, rng: np.random.Generator, *, bf16: bool = False,
            outlier_channels: int = 4, lo: float = 5.0, hi: float = 20.0):
    """KV-cache tensor [T tokens, C = heads x head_dim channels]: N(0,1) with a per-channel
    offset U(-1, 1) and `outlier_channels` channels scaled by U(lo, hi) -- K caches carry
    channel-wise outliers, V caches few.  float16, or uint16 bf16 bit patterns."""
    x = rng.standard_normal((T, C), dtype=np.float32)
    x += rng.uniform(-1.0, 1.0, size=C).astype(np.float32)[None, :]
    if outlier_channels:
        ch = rng.choice(C, size=outlier_channels, replace=False)
        x[:, ch] *= rng.uniform(lo, hi, size=outlier_channels).astype(np.float32)
    if bf16:
        return bf16_bits_from_f32(x)
    return x.astype(np.float16)


def sample_rows(M: int, n: int, x: np.ndarray, seed: int = 7) -> np.ndarray:
    """Seeded sample of token rows that always contains the row holding max |x|."""
    rng = np.random.default_rng(seed)
    xf = x.astype(np.float32) if x.dtype == np.float16 else bf16_bits_to_f32(x)
    top = int(np.unravel_index(np.argmax(np.abs(xf)), xf.shape)[0])
    rows = set([top, 0, M - 1])
    while len(rows) < min(n, M):
        rows.add(int(rng.integers(0, M)))
    return np.array(sorted(rows), dtype=np.int64)
