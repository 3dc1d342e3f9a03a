"""GPU parity of NEXT-1, the fused channel permutation (Fig. 4(d)), through the C
ABI: comet_quantize_act with perm_dev against the oracle quantising x[:, perm] (bit-exact codes,
scales, qsum), comet_pack_weight_perm against packing w[:, perm] (bit-exact), comet_channel_amax
against numpy (exact), and the calibrated end-to-end layer against the oracle (exact INT32
accumulators, rtol 1e-3 / atol 1e-2) and against the unpermuted product (P:L140 equivalence)."""
import numpy as np
import pytest

import oracle
from oracle import calibrate as ocal
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth
from _layout import decode_act, unpack_weight

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

import paper_conf_asplos_liu0rxpwl0w25_b200 as cb   # noqa: E402

DEV = "cuda:0"


def _dev16(x, bf16):
    if bf16:
        return torch.from_numpy(x.view(np.int16)).to(DEV).view(torch.bfloat16)
    return torch.from_numpy(x).to(DEV)


def _check_codes(x, tags, perm, bf16, rows=None):
    M, K = x.shape
    act, sc = cb.quantize_act(_dev16(x, bf16), tags, perm=torch.from_numpy(perm).to(DEV))
    torch.cuda.synchronize()
    codes, scales, qsum, corr = decode_act(act.cpu().numpy(), sc.cpu().numpy(), M, K, tags)
    xp = ocal.permute_channels(x, perm)
    if rows is None:
        rc, rs = oracle.quantize(xp, tags, bf16_bits=bf16)
        rows = np.arange(M)
    else:
        xp = xp[rows]
        rc, rs = oracle.quantize(xp, tags, bf16_bits=bf16)
    assert np.array_equal(codes[rows], rc), "codes differ"
    assert np.array_equal(scales[rows].view(np.uint32), rs.view(np.uint32)), "scales differ"
    nb = K // 128
    rq = rc.reshape(len(rows), nb, 128).astype(np.int64).sum(2)
    assert np.array_equal(qsum[:, rows].T.astype(np.int64), rq)
    Mp = qsum.shape[1]
    assert np.all(qsum[:, M:] == 0) and np.all(sc.cpu().numpy().reshape(nb, Mp)[:, M:] == 0)
    terms = 8.0 * rs.astype(np.float64) * rq * (tags == 0)[None, :]
    bound = np.abs(terms).sum(1) * nb * 2.0 ** -23 + 1e-30
    assert np.all(np.abs(corr[rows] - terms.sum(1)) <= bound)


@pytest.mark.parametrize("M,K,bf16,kind", [
    (1, 256, False, "random"), (16, 256, False, "calib"), (37, 1024, True, "random"),
    (300, 4096, False, "calib"), (5, 8192, True, "calib"), (129, 2048, False, "identity"),
])
def test_quantize_perm_parity(M, K, bf16, kind):
    p = synth.make_unpermuted_problem(M, K, 128, seed=M + K, bf16=bf16)
    if kind == "random":
        perm = np.random.default_rng(K).permutation(K).astype(np.int32)
        tags = synth.make_tags(K, 0.25, np.random.default_rng(M))
    elif kind == "identity":
        perm = np.arange(K, dtype=np.int32)
        tags = synth.make_tags(K, 0.25, np.random.default_rng(M))
    else:
        xc = p.x_calib if not bf16 else synth.bf16_bits_to_f32(p.x_calib)
        perm, tags, _ = ocal.calibrate_perm(ocal.channel_amax(xc), 10.0)
    _check_codes(p.x, tags, perm, bf16)


def test_quantize_perm_full_size_sampled():
    """LLaMA-3-70B down input (K = 28672) at M = 4096: the largest K the fused gather takes."""
    p = synth.make_unpermuted_problem(4096, 28672, 128, seed=9, m_calib=64)
    perm, tags, n = ocal.calibrate_perm(ocal.channel_amax(p.x_calib), 10.0)
    assert n == len(p.outlier_channels)
    rows = synth.sample_rows(4096, 16, p.x)
    _check_codes(p.x, tags, perm, False, rows=rows)


def test_identity_perm_equals_unpermuted_kernel():
    p = synth.make_problem(77, 4096, 128, frac=0.05, seed=4)
    x = torch.from_numpy(p.x).to(DEV)
    a0, s0 = cb.quantize_act(x, p.tags)
    a1, s1 = cb.quantize_act(x, p.tags, perm=torch.arange(4096, dtype=torch.int32, device=DEV))
    torch.cuda.synchronize()
    # codes and qsum bit-identical; corr is a binary32 sum in an implementation-defined order
    # (include/comet.h), so it is compared within the summation bound
    assert torch.equal(s0, s1)
    c0, _, q0, r0 = decode_act(a0.cpu().numpy(), s0.cpu().numpy(), 77, 4096, p.tags)
    c1, _, q1, r1 = decode_act(a1.cpu().numpy(), s1.cpu().numpy(), 77, 4096, p.tags)
    assert np.array_equal(c0, c1) and np.array_equal(q0, q1)
    assert np.allclose(r0, r1, rtol=32 * 2.0 ** -23, atol=0)


@pytest.mark.parametrize("M,K,bf16", [(1, 128, False), (100, 4096, False), (513, 8192, True), (3, 28672, False)])
def test_channel_amax_exact(M, K, bf16):
    p = synth.make_unpermuted_problem(M, K, 128, seed=K, bf16=bf16)
    a = cb.channel_amax(_dev16(p.x, bf16))
    torch.cuda.synchronize()
    xf = synth.bf16_bits_to_f32(p.x) if bf16 else p.x
    assert np.array_equal(a.cpu().numpy(), ocal.channel_amax(xf))


@pytest.mark.parametrize("N,K", [(128, 256), (384, 4096)])
def test_pack_weight_perm_layout(N, K):
    rng = np.random.default_rng(N * K)
    w = rng.integers(-8, 8, size=(N, K), dtype=np.int8)
    perm = rng.permutation(K).astype(np.int32)
    wp = cb.pack_weight(torch.from_numpy(w).to(DEV), perm=torch.from_numpy(perm).to(DEV))
    torch.cuda.synchronize()
    assert np.array_equal(unpack_weight(wp.cpu().numpy(), N, K), ocal.permute_channels(w, perm))


@pytest.mark.parametrize("M,K,N,orientation", [(16, 1024, 256, 1), (300, 2048, 512, 2), (4, 8192, 1024, 0)])
def test_calibrated_layer_end_to_end(M, K, N, orientation):
    """Calibrate on the GPU (channel_amax + calibrate_perm), permute-pack the weights, run the
    layer with the fused permutation; exact INT32 accumulators vs the oracle on x[:, perm] and
    w[:, perm]; FP32 output within tolerance; and within the quantiser's bound of X W^T."""
    p = synth.make_unpermuted_problem(M, K, N, seed=K + N)
    amax = cb.channel_amax(torch.from_numpy(p.x_calib).to(DEV))
    perm, tags, n = cb.calibrate_perm(amax)
    assert n == len(p.outlier_channels)
    perm_d = torch.from_numpy(perm).to(DEV)
    wp = cb.pack_weight(torch.from_numpy(p.w).to(DEV), perm=perm_d)
    sw = torch.from_numpy(p.s_w).to(DEV)
    plan = cb.Plan(M, N, K, tags, orientation=orientation)
    act, sc = cb.quantize_act(torch.from_numpy(p.x).to(DEV), tags, perm=perm_d)
    y, dacc = cb.w4ax_gemm(plan, act, sc, wp, sw, out_dtype=torch.float32, debug=True)
    torch.cuda.synchronize()
    xp, wpm = ocal.permute_channels(p.x, perm), ocal.permute_channels(p.w, perm)
    yref, acc, _, scales = oracle.w4ax(xp, tags, wpm, p.s_w)
    assert np.array_equal(dacc.cpu().numpy().astype(np.int64), acc.sum(0))
    got = y.cpu().numpy().astype(np.float64)
    assert np.allclose(got, yref, rtol=1e-3, atol=1e-2)
    wd = p.w.astype(np.float64) * p.s_w.astype(np.float64)[:, None]
    exact = p.x.astype(np.float64) @ wd.T
    half = np.repeat(scales.astype(np.float64), 128, axis=1) / 2 * (1 + 2.0 ** -20)
    bound = half @ np.abs(ocal.permute_channels(wd, perm)).T
    assert np.all(np.abs(got - exact) <= bound + 1e-2 * np.abs(exact) + 1e-2)
