"""NEXT-1: the FMPQ channel permutation (Fig. 4(d)), CPU side.

Pins for the calibration/permutation oracle (oracle/calibrate.py) against things other than
itself -- planted outlier channels, brute-force order checks, Python's statistics.median, the
computational-equivalence identity of P:L140 within the quantiser's error bound and the
paper's "< 20 % of blocks" claim -- and the library's host calibration
(comet_calibrate_perm) against the oracle, bit-exactly (no GPU needed)."""
import statistics

import numpy as np
import pytest

import oracle
from oracle import calibrate as ocal
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth

BLOCK = 128


def _amax_f32(x):
    return np.abs(x.astype(np.float32)).max(axis=0)


@pytest.mark.parametrize("K", [128, 256, 1024])
def test_median_matches_statistics(K):
    rng = np.random.default_rng(K)
    a = rng.random(K).astype(np.float32)
    assert ocal.median(a) == statistics.median([float(v) for v in a])
    a_odd = a[:-1]
    assert ocal.median(a_odd) == statistics.median([float(v) for v in a_odd])


@pytest.mark.parametrize("K,n_out,seed", [(4096, 20, 1), (8192, 41, 2), (1024, 1, 3), (28672, 143, 4)])
def test_calibration_recovers_planted_outliers(K, n_out, seed):
    p = synth.make_unpermuted_problem(4, K, 128, n_outlier_channels=n_out, seed=seed)
    perm, tags, n = ocal.calibrate_perm(ocal.channel_amax(p.x_calib), 10.0)
    assert n == n_out
    assert np.array_equal(np.sort(perm[:n]), p.outlier_channels)
    # a permutation; each group ascending
    assert np.array_equal(np.sort(perm), np.arange(K))
    assert np.all(np.diff(perm[:n]) > 0) and np.all(np.diff(perm[n:]) > 0)
    assert int(tags.sum()) == -(-n_out // BLOCK) and np.all(tags[: int(tags.sum())] == 1)


def test_permutation_reduces_int8_blocks_below_20_percent():
    """after the permutation "only a small portion of blocks (less than 20%) need 8-bit
    quantization"; without it every block holding an outlier channel is INT8 (Fig. 4(c))."""
    p = synth.make_unpermuted_problem(4, 4096, 128, channel_frac=0.005, seed=5)
    amax = ocal.channel_amax(p.x_calib)
    _, tags, n = ocal.calibrate_perm(amax, 10.0)
    blocks_without = len(set((p.outlier_channels // BLOCK).tolist()))
    assert tags.mean() < 0.20
    assert blocks_without > 5 * int(tags.sum())


def test_ratio_extremes():
    a = np.arange(1, 257, dtype=np.float32)
    perm, tags, n = ocal.calibrate_perm(a, 1e9)
    assert n == 0 and np.array_equal(perm, np.arange(256)) and tags.sum() == 0
    perm, tags, n = ocal.calibrate_perm(a, 1e-9)
    assert n == 256 and tags.sum() == 2


def test_within_block_permutation_permutes_codes_and_keeps_scales():
    """Block max-abs is invariant under a permutation inside each block, so quantising x[:, perm]
    gives codes[:, perm] and the same scales: pins the composition permute -> quantise."""
    p = synth.make_problem(9, 512, 128, frac=0.25, seed=21)
    rng = np.random.default_rng(3)
    perm = np.concatenate([b * BLOCK + rng.permutation(BLOCK) for b in range(4)]).astype(np.int32)
    c0, s0 = oracle.quantize(p.x, p.tags)
    c1, s1 = oracle.quantize(ocal.permute_channels(p.x, perm), p.tags)
    assert np.array_equal(c1, c0[:, perm]) and np.array_equal(s1, s0)


def test_permuted_path_is_computationally_equivalent():
    """permuting the weight columns with the activation channels keeps X W^T; the
    permuted, calibrated W4Ax result is within the quantiser's bound of the unpermuted product
    (the inverse permutation on the weights misses by an order of magnitude more)."""
    p = synth.make_unpermuted_problem(12, 1024, 64, n_outlier_channels=6, seed=8)
    perm, tags, _ = ocal.calibrate_perm(ocal.channel_amax(p.x_calib), 10.0)
    xp = ocal.permute_channels(p.x, perm)
    wpm = ocal.permute_channels(p.w, perm)
    y, acc, codes, scales = oracle.w4ax(xp, tags, wpm, p.s_w)
    wd = p.w.astype(np.float64) * p.s_w.astype(np.float64)[:, None]
    exact = p.x.astype(np.float64) @ wd.T
    half = np.repeat(scales.astype(np.float64), BLOCK, axis=1) / 2 * (1 + 2.0 ** -20)
    bound = half @ np.abs(ocal.permute_channels(wd, perm)).T
    assert np.all(np.abs(y - exact) <= bound + 1e-12)
    # the wrong (inverse) permutation on the weights breaks the equivalence
    inv = np.argsort(perm).astype(np.int32)
    y_bad, *_ = oracle.w4ax(xp, tags, ocal.permute_channels(p.w, inv), p.s_w)
    assert np.mean(np.abs(y_bad - exact)) > 10 * np.mean(np.abs(y - exact))


# --------------------------------------------------------------- library host calibration

cb = pytest.importorskip("paper_conf_asplos_liu0rxpwl0w25_b200")


@pytest.mark.parametrize("K,n_out,seed,ratio", [(4096, 20, 1, 10.0), (8192, 300, 2, 10.0),
                                                (256, 0, 3, 10.0), (1024, 5, 4, 3.0), (28672, 143, 6, 10.0)])
def test_library_calibration_matches_oracle(K, n_out, seed, ratio):
    if n_out:
        p = synth.make_unpermuted_problem(2, K, 128, n_outlier_channels=n_out, seed=seed)
        a = ocal.channel_amax(p.x_calib)
    else:
        a = np.random.default_rng(seed).random(K).astype(np.float32)
    perm, tags, n = cb.calibrate_perm(a, ratio)
    rp, rt, rn = ocal.calibrate_perm(a, ratio)
    assert n == rn and np.array_equal(perm, rp) and np.array_equal(tags, rt)


def test_library_calibration_ties_and_errors():
    a = np.full(256, 2.0, np.float32)        # median 2, nothing above 20
    perm, tags, n = cb.calibrate_perm(a, 10.0)
    assert n == 0 and np.array_equal(perm, np.arange(256))
    a[[7, 200]] = 20.0                        # == ratio * median: not an outlier (strict >)
    a[100] = 20.5
    perm, tags, n = cb.calibrate_perm(a, 10.0)
    assert n == 1 and perm[0] == 100 and tags[0] == 1 and tags[1] == 0
    with pytest.raises(cb.CometError):
        cb.calibrate_perm(np.ones(200, np.float32))          # K % 128
    with pytest.raises(cb.CometError):
        cb.calibrate_perm(np.ones(256, np.float32), -1.0)    # ratio
    bad = np.ones(256, np.float32)
    bad[3] = np.nan
    with pytest.raises(cb.CometError):
        cb.calibrate_perm(bad)
