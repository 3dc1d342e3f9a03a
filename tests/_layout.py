"""numpy decoders of the packed layouts, written from the spec in include/comet.h (they do not
call library code).  Used by the parity tests to compare the CUDA path with the oracle."""
from __future__ import annotations

import numpy as np

BLOCK = 128
PAD = 16

# E4M3 encodings of the integers -7..7 as spelled out in include/comet.h
_E4M3_POS = {0: 0x00, 1: 0x38, 2: 0x40, 3: 0x44, 4: 0x48, 5: 0x4A, 6: 0x4C, 7: 0x4E}
E4M3_DECODE = np.full(256, -128, dtype=np.int16)   # -128 marks an invalid byte
for v, b in _E4M3_POS.items():
    E4M3_DECODE[b] = v
    if v:
        E4M3_DECODE[0x80 | b] = -v


def layout(M: int, K: int) -> dict:
    nb = K // BLOCK
    Mp = (M + PAD - 1) // PAD * PAD
    ru = lambda a: (a + 255) // 256 * 256
    qsum_off = ru(M * K)
    corr_off = ru(qsum_off + nb * Mp * 2)
    total = ru(corr_off + Mp * 4)
    return dict(nb=nb, Mp=Mp, qsum_off=qsum_off, corr_off=corr_off, total=total)


def decode_act(buf: np.ndarray, scales: np.ndarray, M: int, K: int, tags: np.ndarray):
    """-> codes int8 [M,K], scales f32 [M,nb], qsum int16 [nb,Mp], corr f32 [Mp]."""
    L = layout(M, K)
    nb, Mp = L["nb"], L["Mp"]
    raw = buf[: M * K].reshape(M, K)
    codes = np.empty((M, K), dtype=np.int16)
    for b in range(nb):
        sl = slice(b * BLOCK, (b + 1) * BLOCK)
        if tags[b]:
            codes[:, sl] = raw[:, sl].view(np.int8)
        else:
            codes[:, sl] = E4M3_DECODE[raw[:, sl]]
    assert np.all(codes != -128), "invalid E4M3 byte in an INT4 block"
    qsum = buf[L["qsum_off"]: L["qsum_off"] + nb * Mp * 2].view(np.int16).reshape(nb, Mp)
    corr = buf[L["corr_off"]: L["corr_off"] + Mp * 4].view(np.float32)
    sc = scales.reshape(nb, Mp)[:, :M].T.copy()
    return codes.astype(np.int8), sc, qsum, corr


def unpack_words(wp: np.ndarray, N: int, K: int) -> np.ndarray:
    """Row-major packed words [N][K/2] -> codes int8 [N][K]: word g byte i = u[8g+i] | u[8g+i+4] << 4,
    u = w + 8 (the word format of include/comet.h)."""
    words = wp.reshape(N, K // 8, 4)
    lo = (words & 0x0F).astype(np.int16) - 8      # u[8g + i]
    hi = (words >> 4).astype(np.int16) - 8        # u[8g + 4 + i]
    out = np.concatenate([lo, hi], axis=2).reshape(N, K)
    return out.astype(np.int8)


def untile_weight(wp: np.ndarray, N: int, K: int) -> np.ndarray:
    """The row-tiled w_packed of include/comet.h -- 1 KB tiles [N/16][K/128][16 rows][64 B] --
    back to row-major [N][K/2] bytes."""
    nb = K // BLOCK
    t = np.asarray(wp).reshape(N // 16, nb, 16, 64)
    return np.ascontiguousarray(t.transpose(0, 2, 1, 3)).reshape(N, K // 2)


def unpack_weight(wp: np.ndarray, N: int, K: int) -> np.ndarray:
    """w_packed (row-tiled, include/comet.h) -> codes int8 [N][K]."""
    return unpack_words(untile_weight(wp, N, K), N, K)
