"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle on the same seeded
inputs.  Codes, tags, scales, qsum, weight packing and the INT32 debug accumulators are
compared bit-exactly; the dequantised output within the north-star tolerance, tightened
(see _close; R10).  The production kernels' bit-exactness at full size is in
tests/test_gpu_exact.py."""
import numpy as np
import pytest

import oracle
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth
from _layout import decode_act, unpack_weight

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

import paper_conf_asplos_liu0rxpwl0w25_b200 as cb   # noqa: E402

DEV = "cuda:0"


def _x_dev(p: synth.Problem):
    if p.bf16:
        return torch.from_numpy(p.x.view(np.int16)).to(DEV).view(torch.bfloat16)
    return torch.from_numpy(p.x).to(DEV)


def _quant(p: synth.Problem):
    act, sc = cb.quantize_act(_x_dev(p), p.tags)
    torch.cuda.synchronize()
    return act, sc


def _check_quant(p, act, sc, rows=None):
    codes, scales, qsum, corr = decode_act(act.cpu().numpy(), sc.cpu().numpy(), p.M, p.K, p.tags)
    if rows is None:
        ref_codes, ref_scales = oracle.quantize(p.x, p.tags, bf16_bits=p.bf16)
        rows = np.arange(p.M)
    else:
        _, _, ref_codes, ref_scales = oracle.w4ax_rows(p.x, p.tags, np.zeros((128, p.K), np.int8),
                                                       np.ones(128, np.float32), rows, bf16_bits=p.bf16)
    assert np.array_equal(codes[rows], ref_codes), "codes differ"
    assert np.array_equal(scales[rows].view(np.uint32), ref_scales.view(np.uint32)), "scales differ"
    nb = p.K // 128
    ref_q = ref_codes.reshape(len(rows), nb, 128).astype(np.int64).sum(2)
    assert np.array_equal(qsum[:, rows].T.astype(np.int64), ref_q), "qsum differs"
    Mp = qsum.shape[1]
    assert np.all(qsum[:, p.M:] == 0) and np.all(sc.cpu().numpy().reshape(nb, Mp)[:, p.M:] == 0)
    # corr = 8 sum_{INT4 blocks} s q  (binary32 sum; compare with the exact value)
    terms = 8.0 * ref_scales.astype(np.float64) * ref_q * (p.tags == 0)[None, :]
    # binary32 summation: error bounded by ~nb ulps of the running magnitude
    bound = np.abs(terms).sum(1) * nb * 2.0 ** -23 + 1e-30
    assert np.all(np.abs(corr[rows] - terms.sum(1)) <= bound)
    return codes


# ------------------------------------------------------------------------------- kernel 1

@pytest.mark.parametrize("M,K,frac,bf16", [
    (16, 256, None, False),            # config 1
    (1, 4096, 0.05, False), (16, 4096, 0.05, False), (256, 11008, 0.05, False),   # config 2
    (33, 1024, 0.5, True), (1000, 512, 0.25, False), (7, 14336, 0.05, True),
    (1, 28672, 0.05, False), (32, 28672, 0.05, True), (3, 11008, 0.25, False),   # cluster-split rows
    # staged-ring kernel (M > 32): ragged groups (71 blocks: a 1-group last chunk of 7 blocks),
    # a sub-group row, more CTAs than a resident wave holds rows for
    (300, 9088, 0.25, True), (40, 640, 0.5, False), (777, 3200, 0.05, False), (4100, 1152, 0.05, True),
])
def test_quantize_parity(M, K, frac, bf16):
    if frac is None:
        p = synth.config1()
    else:
        p = synth.make_problem(M, K, 128, frac=frac, seed=M + K, bf16=bf16)
    act, sc = _quant(p)
    _check_quant(p, act, sc)


def test_quantize_edge_cases():
    # zero blocks, ties, bf16 binary32-subnormal block, all-INT8 and all-INT4
    x = np.zeros((3, 512), np.float16)
    x[1, :6] = [7.0, 2.5, 3.5, -2.5, -0.5, 1.5]
    x[2, 128:256] = -1.0
    x[2, 300] = 65504.0
    for tags in (np.array([0, 1, 0, 1], np.uint8), np.zeros(4, np.uint8), np.ones(4, np.uint8)):
        p = synth.Problem(x=x, tags=tags, w=np.zeros((128, 512), np.int8), s_w=np.ones(128, np.float32))
        act, sc = _quant(p)
        _check_quant(p, act, sc)
    # the same rows through the staged-ring kernel (M > 32), tiled to 67 rows
    xr = np.tile(x, (23, 1))[:67]
    for tags in (np.array([0, 1, 0, 1], np.uint8), np.ones(4, np.uint8)):
        p = synth.Problem(x=xr, tags=tags, w=np.zeros((128, 512), np.int8), s_w=np.ones(128, np.float32))
        act, sc = _quant(p)
        _check_quant(p, act, sc)
    xb = np.zeros((2, 128), np.uint16)
    xb[0, 0], xb[0, 1], xb[1, 5] = 0x0001, 0x8001, 0x3F80
    p = synth.Problem(x=xb, tags=np.array([0], np.uint8), w=np.zeros((128, 128), np.int8),
                      s_w=np.ones(128, np.float32), bf16=True)
    act, sc = _quant(p)
    _check_quant(p, act, sc)


def test_quantize_full_size_sampled():
    """LLaMA-3-8B down input at M=8192, K=14336 (config 3): sampled rows vs the oracle."""
    p = synth.make_problem(8192, 14336, 128, frac=0.05, seed=3)
    act, sc = _quant(p)
    rows = synth.sample_rows(p.M, 24, p.x)
    _check_quant(p, act, sc, rows=rows)


# ------------------------------------------------------------------------------- weight pack

@pytest.mark.parametrize("N,K", [(128, 128), (256, 4096), (1280, 8192)])
def test_pack_weight_layout(N, K):
    rng = np.random.default_rng(N + K)
    w = rng.integers(-8, 8, size=(N, K), dtype=np.int8)
    wp = cb.pack_weight(torch.from_numpy(w).to(DEV))
    torch.cuda.synchronize()
    assert np.array_equal(unpack_weight(wp.cpu().numpy(), N, K), w)


# ------------------------------------------------------------------------------- GEMM

def _run(p: synth.Problem, *, tile_n=0, split_mode=-1, out_dtype=torch.float32, debug=False,
         debug_blocks=False, num_sms=0, orientation=0):
    act, sc = _quant(p)
    wp = cb.pack_weight(torch.from_numpy(p.w).to(DEV))
    sw = torch.from_numpy(p.s_w).to(DEV)
    plan = cb.Plan(p.M, p.N, p.K, p.tags, tile_n=tile_n, split_mode=split_mode, num_sms=num_sms,
                   orientation=orientation)
    res = cb.w4ax_gemm(plan, act, sc, wp, sw, out_dtype=out_dtype, debug=debug, debug_blocks=debug_blocks)
    torch.cuda.synchronize()
    return res, plan


def _close(y, ref, dtype):
    """Dequantised output against the binary64 oracle (north star: rtol 1e-3; R10).
    FP32: |y - ref| <= 1e-3 |ref| + 1e-5 max|ref| (the GPU's binary32 summation of <= 224
    exact block terms errs by ~1e-6 of the terms; 1e-5 max|ref| still catches one dropped or
    mis-scaled block partial, ~1e-1).  FP16: within 1 FP16 ulp of ref (+ the same 1e-5 max|ref|
    binary32 slack).  BF16: within 1 BF16 ulp of the oracle rounded to BF16 (a true 1-ulp bound:
    the spacing of the binade of max(|r|, |y|))."""
    got = y.float().cpu().numpy().astype(np.float64)
    assert np.all(np.isfinite(got)), "non-finite outputs"
    slack = 1e-5 * float(np.abs(ref).max())
    if dtype == torch.bfloat16:
        r = torch.from_numpy(ref.astype(np.float32)).to(torch.bfloat16).double().numpy()
        mag = np.maximum(np.abs(r), np.abs(got))
        ulp = np.exp2(np.floor(np.log2(np.maximum(mag, 2.0 ** -126))) - 7)
        bad = np.abs(got - r) > ulp
        assert not bad.any(), f"{bad.sum()} bf16 outputs off by more than 1 ulp"
    elif dtype == torch.float16:
        mag = np.maximum(np.abs(ref), 2.0 ** -14)
        ulp = np.exp2(np.floor(np.log2(mag)) - 10)
        bad = np.abs(got - ref) > ulp + slack
        assert not bad.any(), f"{bad.sum()} fp16 outputs off by more than 1 ulp; max err {np.abs(got-ref).max()}"
    else:
        bad = np.abs(got - ref) > 1e-3 * np.abs(ref) + slack
        assert not bad.any(), f"{bad.sum()} outputs outside 1e-3 |ref| + 1e-5 max|ref|; max err {np.abs(got-ref).max()}"


@pytest.mark.parametrize("orientation", [1, 2])
def test_gemm_config1_bit_exact_blocks(orientation):
    p = synth.config1()
    (y, dacc, dblk), _ = _run(p, debug_blocks=True, orientation=orientation)
    yref, acc, _, _ = oracle.w4ax(p.x, p.tags, p.w, p.s_w)
    assert np.array_equal(dblk.cpu().numpy().astype(np.int64), acc), "per-block INT32 accumulators differ"
    assert np.array_equal(dacc.cpu().numpy().astype(np.int64), acc.sum(0))
    _close(y, yref, torch.float32)


@pytest.mark.parametrize("M,N,K,frac", [
    (1, 256, 512, 0.5), (17, 384, 1024, 0.25), (100, 512, 2048, 0.05), (300, 256, 768, 1.0),
    (64, 128, 256, 0.0),
])
@pytest.mark.parametrize("orientation", [1, 2])
def test_gemm_debug_accumulators_exact(M, N, K, frac, orientation):
    p = synth.make_problem(M, K, N, frac=frac, seed=M * 7 + K)
    (y, dacc), _ = _run(p, debug=True, orientation=orientation)
    yref, acc, _, _ = oracle.w4ax(p.x, p.tags, p.w, p.s_w)
    assert np.array_equal(dacc.cpu().numpy().astype(np.int64), acc.sum(0))
    _close(y, yref, torch.float32)


@pytest.mark.parametrize("orientation", [1, 2])
def test_gemm_all_int8_matches_torch_int_mm(orientation):
    """I1 on the GPU: all tags INT8 -> per-block accumulators equal cuBLASLt's INT8 GEMM."""
    p = synth.make_problem(64, 512, 256, frac=1.0, seed=5)
    (y, dacc, dblk), _ = _run(p, debug_blocks=True, orientation=orientation)
    codes, _ = oracle.quantize(p.x, p.tags)
    for b in range(4):
        a = torch.from_numpy(codes[:, b * 128:(b + 1) * 128].copy()).to(DEV)
        w = torch.from_numpy(p.w[:, b * 128:(b + 1) * 128].copy()).to(DEV)
        ref = torch._int_mm(a, w.t().contiguous())
        assert torch.equal(dblk[b], ref)


@pytest.mark.parametrize("tile_n", [16, 32, 64, 128])
@pytest.mark.parametrize("split_mode", [0, 1])
def test_gemm_tile_and_schedule_variants(tile_n, split_mode):
    p = synth.make_problem(230, 2048, 1024, frac=0.25, seed=tile_n)
    y, plan = _run(p, tile_n=tile_n, split_mode=split_mode, num_sms=37, orientation=1)
    yref, _, _, _ = oracle.w4ax(p.x, p.tags, p.w, p.s_w)
    _close(y, yref, torch.float32)


@pytest.mark.parametrize("M,N", [(230, 2048), (300, 1152), (129, 256), (1000, 384)])
@pytest.mark.parametrize("split_mode", [0, 1])
def test_gemm_normal_orientation_schedules(M, N, split_mode):
    """Tokens on the MMA M side (prefill kernel): ragged M, N % 256 == 128, stream-K."""
    p = synth.make_problem(M, 1024, N, frac=0.25, seed=M + N)
    y, plan = _run(p, split_mode=split_mode, num_sms=23, orientation=2)
    yref, _, _, _ = oracle.w4ax(p.x, p.tags, p.w, p.s_w)
    _close(y, yref, torch.float32)


@pytest.mark.parametrize("orientation", [1, 2])
@pytest.mark.parametrize("split_mode", [2, 3])
def test_gemm_unit_schedules(split_mode, orientation):
    p = synth.make_problem(96, 512, 1024, frac=0.25, seed=11)
    y, plan = _run(p, split_mode=split_mode, num_sms=13, orientation=orientation)
    assert plan.info()["n_split_tiles"] > 0
    yref, _, _, _ = oracle.w4ax(p.x, p.tags, p.w, p.s_w)
    _close(y, yref, torch.float32)


@pytest.mark.parametrize("orientation", [1, 2])
@pytest.mark.parametrize("dtype", [torch.float16, torch.bfloat16, torch.float32])
def test_gemm_output_dtypes(dtype, orientation):
    p = synth.make_problem(48, 1024, 512, frac=0.25, seed=21)
    y, _ = _run(p, out_dtype=dtype, orientation=orientation)
    yref, _, _, _ = oracle.w4ax(p.x, p.tags, p.w, p.s_w)
    _close(y, yref, dtype)


@pytest.mark.parametrize("frac", [0.0, 0.05, 0.25, 1.0])
def test_gemm_outlier_fraction_sweep(frac):
    """Config 3's sweep shape class at reduced M (full size is in test_gemm_full_size)."""
    p = synth.make_problem(200, 4096, 1024, frac=frac, seed=31)
    y, _ = _run(p)
    yref, _, _, _ = oracle.w4ax(p.x, p.tags, p.w, p.s_w)
    _close(y, yref, torch.float32)


@pytest.mark.parametrize("orientation", [1, 2])
def test_gemm_bf16_input(orientation):
    p = synth.make_problem(40, 1024, 384, frac=0.34, seed=41, bf16=True)
    (y, dacc), _ = _run(p, debug=True, orientation=orientation)
    yref, acc, _, _ = oracle.w4ax(p.x, p.tags, p.w, p.s_w, bf16_bits=True)
    assert np.array_equal(dacc.cpu().numpy().astype(np.int64), acc.sum(0))
    _close(y, yref, torch.float32)


FULL = [
    ("l2_7b_qkvo_m1", 1, 4096, 4096, 0.05),
    ("l2_7b_gateup_m16", 16, 4096, 11008, 0.05),
    ("l2_7b_down_m256", 256, 11008, 4096, 0.05),
    ("l2_7b_qkvo_m4096", 4096, 4096, 4096, 0.05),
    ("l3_8b_down_m8192", 8192, 14336, 4096, 0.05),
    ("l3_70b_gateup_m4096", 4096, 8192, 28672, 0.05),
    ("l3_70b_down_m4096", 4096, 28672, 8192, 0.05),
    ("l3_70b_qkv_m4096", 4096, 8192, 10240, 0.05),
    ("l3_70b_gateup_tp8_m32", 32, 8192, 3584, 0.05),
    ("l3_70b_down_tp8_m1", 1, 3584, 8192, 0.05),
    ("l3_70b_gateup_m1", 1, 8192, 28672, 0.05),      # config 5 (decode sweep of bench.py)
    ("l3_70b_down_m8", 8, 28672, 8192, 0.05),
    ("l3_70b_qkv_m32", 32, 8192, 10240, 0.05),
]


@pytest.mark.parametrize("name,M,K,N,frac", FULL, ids=[f[0] for f in FULL])
def test_gemm_full_size(name, M, K, N, frac):
    """BASELINE sizes, the bench's launch configuration (auto plan), the synthetic workload
    (N(0,1) activations with outlier channels), 64 sampled rows vs oracle (bit-exactness on
    these configurations is tests/test_gpu_exact.py)."""
    p = synth.make_problem(M, K, N, frac=frac, seed=sum(map(ord, name)))
    y, plan = _run(p, out_dtype=torch.float16)
    rows = synth.sample_rows(M, 64, p.x)
    yref, acc_sum, codes, scales = oracle.w4ax_rows(p.x, p.tags, p.w, p.s_w, rows)
    _close(y[torch.from_numpy(rows).to(DEV)], yref, torch.float16)


@pytest.mark.parametrize("M,K,N,mean", [(4096, 28672, 8192, 2.0), (16, 8192, 28672, -1.5), (300, 4096, 1024, 3.0)])
def test_gemm_nonzero_mean_activations(M, K, N, mean):
    """Activations with a non-zero mean: large code sums, so the offset-binary correction
    corr = 8 sum_b s_a qsum cancels a large part of the INT4 blocks' accumulators.
    FP32 output, tightened tolerance."""
    p = synth.make_problem(M, K, N, frac=0.05, seed=M + K)
    x = (p.x.astype(np.float32) + np.float32(mean)).astype(np.float16)
    p = synth.Problem(x=x, tags=p.tags, w=p.w, s_w=p.s_w)
    y, plan = _run(p, out_dtype=torch.float32)
    rows = synth.sample_rows(M, 64, p.x)
    yref, _, _, _ = oracle.w4ax_rows(p.x, p.tags, p.w, p.s_w, rows)
    _close(y[torch.from_numpy(rows).to(DEV)], yref, torch.float32)


# ------------------------------------------------------------------------------- host-buffer path

@pytest.mark.parametrize("M,blocking", [(300, True), (2500, True), (2500, False), (4096, False)])
def test_linear_host_pipeline(M, blocking):
    """comet_w4ax_linear_host(_async): pinned host x in, host y out.  M >= 2048 runs the
    1024-row chunk pipeline (three streams, sub-plans, ragged last chunk at 2500)."""
    K, N = 1024, 384
    p = synth.make_problem(M, K, N, frac=0.25, seed=M + 7)
    wp = cb.pack_weight(torch.from_numpy(p.w).to(DEV))
    sw = torch.from_numpy(p.s_w).to(DEV)
    plan = cb.Plan(M, N, K, p.tags)
    x_host = torch.from_numpy(p.x).pin_memory()
    y_host = torch.full((M, N), float("nan"), dtype=torch.float16).pin_memory()
    scratch = torch.empty(cb.linear_scratch_bytes(plan, cb.COMET_F16, cb.COMET_F16), dtype=torch.uint8, device=DEV)
    for _ in range(2):          # second call reuses the scratch (stream-K flags, epochs)
        y_host.fill_(float("nan"))
        cb.w4ax_linear_host(plan, x_host, wp, sw, y_host, scratch, blocking=blocking)
        if not blocking:
            cb.linear_host_wait(plan)
            torch.cuda.synchronize()
        yref, _, _, _ = oracle.w4ax(p.x, p.tags, p.w, p.s_w)
        _close(y_host, yref, torch.float16)


def test_gemm_single_cta_tiles_repeated():
    """Regression: the 192/160-wide single-CTA tiles (S = 3 pipeline slots) once alternated two
    widen groups and two MMA issuers over an odd slot count, so a role could pass a parity wait
    one phase early -- an intermittent launch failure (tools/stress_gemm.py).  Repeat them."""
    for it in range(12):
        for (M, N, sm, tw) in ((300, 1152, 1, 192), (230, 1280, 0, 160), (129, 384, 1, 192)):
            p = synth.make_problem(M, 1024, N, frac=0.25, seed=M + N)
            act, sc = _quant(p)
            wp = cb.pack_weight(torch.from_numpy(p.w).to(DEV))
            plan = cb.Plan(M, N, 1024, p.tags, split_mode=sm, num_sms=23, orientation=2, tile_w=tw)
            y = cb.w4ax_gemm(plan, act, sc, wp, torch.from_numpy(p.s_w).to(DEV), out_dtype=torch.float32)
            torch.cuda.synchronize()
            if it == 0:
                yref, _, _, _ = oracle.w4ax(p.x, p.tags, p.w, p.s_w)
                _close(y, yref, torch.float32)
