"""GPU parity of comet_w4ax_linear: the decode layer with kernel 1 fused into the GEMM (two
warps per CTA quantise each pipeline stage's (token, K-block) pairs straight into the MMA
operand slot; P:L126 / P:L136-138 quantisation, P:L164-178 GEMM).

Exact inputs (synth.make_exact_problem: s_a = 2^e, s_w = 2^f, every partial sum exact in
binary32) make the FP32 output EQUAL the oracle at the BASELINE decode sizes (config 5, the
70B layers at M = 1, 4, 8, stream-K split tiles included) and on ragged small shapes; the
synthetic workload stays within the usual tolerance of the oracle and of the two-launch path
(comet_quantize_act + comet_w4ax_gemm)."""
import numpy as np
import pytest

import oracle
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

import paper_conf_asplos_liu0rxpwl0w25_b200 as cb   # noqa: E402
from test_gpu_parity import _close                   # noqa: E402

DEV = "cuda:0"


def _x_dev(x, bf16=False):
    if bf16:
        return torch.from_numpy(np.ascontiguousarray(x).view(np.int16)).to(DEV).view(torch.bfloat16)
    return torch.from_numpy(np.ascontiguousarray(x)).to(DEV)


@pytest.mark.parametrize("M,K,N,frac,split_mode,num_sms,bf16", [
    (1, 8192, 28672, 0.05, -1, 0, False),       # 70B gate/up, decode
    (4, 28672, 8192, 0.05, -1, 0, False),       # 70B down
    (8, 8192, 10240, 0.05, -1, 0, True),        # 70B qkv, BF16 input
    (8, 8192, 28672, 0.25, -1, 0, False),
    (3, 512, 384, 0.5, 1, 7, False),            # few K-blocks, ragged tokens, forced stream-K
    (5, 1152, 256, 1.0, 0, 0, False),           # all INT8 blocks, whole tiles
    (2, 2048, 640, 0.0, 1, 37, True),           # all INT4 blocks
])
@pytest.mark.parametrize("orientation", [1, 4])
def test_linear_exact(M, K, N, frac, split_mode, num_sms, bf16, orientation):
    """Both fused decode paths: the TMEM kernel's quantiser warps (orientation 1) and the
    warp-level kernel's fused staging (orientation 4)."""
    p = synth.make_exact_problem(M, K, N, frac=frac, seed=M * 7 + K, bf16=bf16,
                                 special_rows={0: "alternating"} if M > 1 else None)
    wp = cb.pack_weight(torch.from_numpy(p.w).to(DEV))
    sw = torch.from_numpy(p.s_w).to(DEV)
    plan = cb.Plan(M, N, K, p.tags, split_mode=split_mode, num_sms=num_sms, orientation=orientation)
    x = _x_dev(p.x, bf16)
    y32 = cb.w4ax_linear_fused(plan, x, wp, sw, out_dtype=torch.float32)
    y16 = cb.w4ax_linear_fused(plan, x, wp, sw, out_dtype=torch.float16)
    torch.cuda.synchronize()
    rows = np.arange(M, dtype=np.int64)
    yref, _, _, _ = oracle.w4ax_rows(p.x, p.tags, p.w, p.s_w, rows, bf16_bits=bf16)
    r32 = yref.astype(np.float32)
    assert np.array_equal(r32.astype(np.float64), yref), "oracle value not exact in binary32"
    g = y32.cpu().numpy()
    bad = g != r32
    assert not bad.any(), f"{bad.sum()} FP32 outputs differ; first {np.argwhere(bad)[0]}"
    assert np.array_equal(y16.cpu().numpy(), yref.astype(np.float16))


@pytest.mark.parametrize("M,K,N,frac", [(1, 8192, 2048, 0.05), (8, 4096, 1024, 0.25), (6, 2048, 512, 0.05)])
def test_linear_synthetic(M, K, N, frac):
    """The synthetic workload (N(0,1) with outlier channels): within tolerance of the oracle,
    and of the two-launch path."""
    p = synth.make_problem(M, K, N, frac=frac, seed=M + K)
    wp = cb.pack_weight(torch.from_numpy(p.w).to(DEV))
    sw = torch.from_numpy(p.s_w).to(DEV)
    plan = cb.Plan(M, N, K, p.tags)
    x = torch.from_numpy(p.x).to(DEV)
    y = cb.w4ax_linear_fused(plan, x, wp, sw, out_dtype=torch.float32)
    act, sc = cb.quantize_act(x, p.tags)
    y2 = cb.w4ax_gemm(plan, act, sc, wp, sw, out_dtype=torch.float32)
    torch.cuda.synchronize()
    yref, _, _, _ = oracle.w4ax(p.x, p.tags, p.w, p.s_w)
    _close(y, yref, torch.float32)
    a, b = y.cpu().numpy().astype(np.float64), y2.cpu().numpy().astype(np.float64)
    assert np.allclose(a, b, rtol=1e-5, atol=1e-5 * np.abs(b).max())


def test_linear_repeated_on_stream():
    """Back-to-back fused launches (programmatic dependents of each other) on one stream."""
    M, K, N = 4, 4096, 2048
    p = synth.make_exact_problem(M, K, N, frac=0.05, seed=5)
    wp = cb.pack_weight(torch.from_numpy(p.w).to(DEV))
    sw = torch.from_numpy(p.s_w).to(DEV)
    plan = cb.Plan(M, N, K, p.tags)
    x = _x_dev(p.x)
    y = torch.empty((M, N), dtype=torch.float32, device=DEV)
    for _ in range(50):
        cb.w4ax_linear_fused(plan, x, wp, sw, out=y)
    torch.cuda.synchronize()
    yref, _, _, _ = oracle.w4ax_rows(p.x, p.tags, p.w, p.s_w, np.arange(M))
    assert np.array_equal(y.cpu().numpy(), yref.astype(np.float32))


@pytest.mark.parametrize("M", [12, 32])
def test_linear_rejects_other_plans(M):
    """M > 8 (the fused path stages 8 input rows per K-block) and 32-token tiles are refused;
    cb.w4ax_linear then takes the two-launch path."""
    p = synth.make_problem(M, 1024, 256, frac=0.05, seed=1)
    wp = cb.pack_weight(torch.from_numpy(p.w).to(DEV))
    sw = torch.from_numpy(p.s_w).to(DEV)
    plan = cb.Plan(M, 256, 1024, p.tags)
    x = torch.from_numpy(p.x).to(DEV)
    with pytest.raises(cb.CometError) as e:
        cb.w4ax_linear_fused(plan, x, wp, sw)
    assert e.value.status == 2
    y = cb.w4ax_linear(plan, x, wp, sw, out_dtype=torch.float32)
    yref, _, _, _ = oracle.w4ax(p.x, p.tags, p.w, p.s_w)
    _close(y, yref, torch.float32)


@pytest.mark.parametrize("orientation", [1, 4])
@pytest.mark.parametrize("bf16", [False, True])
def test_linear_strided_input_exact(orientation, bf16):
    """x with a row stride ldx > K (a view into a wider activation buffer) on both fused paths,
    and the warp-level path's auto plan through cb.w4ax_linear (no kernel-1 launch)."""
    M, K, N = 5, 4096, 8192
    p = synth.make_exact_problem(M, K, N, frac=0.25, seed=41 + orientation, bf16=bf16,
                                 special_rows={1: "alternating"})
    wp = cb.pack_weight(torch.from_numpy(p.w).to(DEV))
    sw = torch.from_numpy(p.s_w).to(DEV)
    wide = torch.zeros((M, K + 384), dtype=torch.bfloat16 if bf16 else torch.float16, device=DEV)
    wide[:, 128:128 + K] = _x_dev(p.x, bf16)
    x = wide[:, 128:128 + K]                      # ldx = K + 384, 256-byte offset
    assert x.stride(0) == K + 384
    plan = cb.Plan(M, N, K, p.tags, orientation=orientation)
    y = cb.w4ax_linear_fused(plan, x, wp, sw, out_dtype=torch.float32)
    y2 = cb.w4ax_linear(plan, x, wp, sw, out_dtype=torch.float32)
    torch.cuda.synchronize()
    yref, _, _, _ = oracle.w4ax_rows(p.x, p.tags, p.w, p.s_w, np.arange(M), bf16_bits=bf16)
    r32 = yref.astype(np.float32)
    assert np.array_equal(y.cpu().numpy(), r32)
    assert np.array_equal(y2.cpu().numpy(), r32)
