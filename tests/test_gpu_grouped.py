"""GPU parity of NEXT-3, group-wise weight scales s_w[b, n] (reading R18), through
comet_w4ax_gemm_grouped: exact INT32 accumulators against the oracle's int64 GEMM and the FP32
output within rtol 1e-3 / atol 1e-2 of oracle/grouped.py, over decode and forced-orientation-1
token counts, ragged tiles and stream-K splits; on the prefill pair kernel, bit-exact outputs
with exact inputs (power-of-two scales) up to the LLaMA-3-70B gate/up size."""
import numpy as np
import pytest

import oracle
from oracle import grouped
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

import paper_conf_asplos_liu0rxpwl0w25_b200 as cb   # noqa: E402

DEV = "cuda:0"


def _gs(N, K, seed):
    rng = np.random.default_rng(seed)
    return (rng.uniform(0.5, 1.5, size=(K // 128, N)) / (8.0 * np.sqrt(K))).astype(np.float32)


@pytest.mark.parametrize("M,N,K,frac,split_mode,num_sms", [
    (1, 256, 512, 0.5, -1, 0), (16, 384, 1024, 0.25, -1, 0), (7, 1024, 4096, 0.05, 1, 37),
    (100, 512, 2048, 0.25, 0, 0), (300, 256, 768, 1.0, -1, 0), (33, 128, 256, 0.0, 1, 5),
])
def test_grouped_gemm_parity(M, N, K, frac, split_mode, num_sms):
    p = synth.make_problem(M, K, N, frac=frac, seed=M + N + K)
    s_wg = _gs(N, K, M)
    act, sc = cb.quantize_act(torch.from_numpy(p.x).to(DEV), p.tags)
    wp = cb.pack_weight(torch.from_numpy(p.w).to(DEV))
    plan = cb.Plan(M, N, K, p.tags, orientation=1, split_mode=split_mode, num_sms=num_sms)
    swg = torch.from_numpy(s_wg).to(DEV)
    y = cb.w4ax_gemm_grouped(plan, act, sc, wp, swg, out_dtype=torch.float32)
    y2, dacc = cb.w4ax_gemm_grouped(plan, act, sc, wp, swg, out_dtype=torch.float32, debug=True)
    torch.cuda.synchronize()
    _, acc, codes, scales = oracle.w4ax(p.x, p.tags, p.w, p.s_w)
    ref = grouped.dequant_grouped(acc, scales, s_wg)
    assert np.array_equal(dacc.cpu().numpy().astype(np.int64), acc.sum(0))
    for got in (y, y2):
        g = got.cpu().numpy().astype(np.float64)
        bad = ~np.isclose(g, ref, rtol=1e-3, atol=1e-2)
        assert not bad.any(), f"{bad.sum()} outputs off; max err {np.abs(g - ref).max()}"


def test_grouped_full_size_decode_sampled():
    """LLaMA-3-70B gate/up at M = 4 (config 5 shape), FP16 output, sampled rows vs the oracle."""
    M, K, N = 4, 8192, 28672
    p = synth.make_problem(M, K, N, frac=0.05, seed=77)
    s_wg = _gs(N, K, 9)
    act, sc = cb.quantize_act(torch.from_numpy(p.x).to(DEV), p.tags)
    wp = cb.pack_weight(torch.from_numpy(p.w).to(DEV))
    plan = cb.Plan(M, N, K, p.tags, orientation=1)   # group-wise scales run on the TMEM decode kernel
    y = cb.w4ax_gemm_grouped(plan, act, sc, wp, torch.from_numpy(s_wg).to(DEV))
    torch.cuda.synchronize()
    cols = np.random.default_rng(1).choice(N, 512, replace=False)
    _, acc, codes, scales = oracle.w4ax(p.x, p.tags, p.w[cols], p.s_w[cols])
    ref = grouped.dequant_grouped(acc, scales, s_wg[:, cols])
    g = y.float().cpu().numpy()[:, cols].astype(np.float64)
    assert np.allclose(g, ref, rtol=1e-3, atol=1e-2)


def test_grouped_rejects_single_cta_prefill_orientation():
    p = synth.make_problem(200, 512, 256, frac=0.25, seed=3)
    act, sc = cb.quantize_act(torch.from_numpy(p.x).to(DEV), p.tags)
    wp = cb.pack_weight(torch.from_numpy(p.w).to(DEV))
    plan = cb.Plan(200, 256, 512, p.tags, orientation=2)
    with pytest.raises(cb.CometError) as e:
        cb.w4ax_gemm_grouped(plan, act, sc, wp, torch.from_numpy(_gs(256, 512, 1)).to(DEV))
    assert e.value.status == 2


# ----------------------------------------------------------------- the prefill pair kernel

def _pair_grouped(p, s_wg, split_mode=-1, out_dtype=torch.float32):
    act, sc = cb.quantize_act(torch.from_numpy(p.x).to(DEV), p.tags)
    wp = cb.pack_weight(torch.from_numpy(p.w).to(DEV))
    plan = cb.Plan(p.M, p.N, p.K, p.tags, orientation=3, split_mode=split_mode)
    y = cb.w4ax_gemm_grouped(plan, act, sc, wp, torch.from_numpy(s_wg).to(DEV), out_dtype=out_dtype)
    torch.cuda.synchronize()
    return y


def _ref_rows(p, s_wg, rows):
    codes, scales = oracle.quantize(p.x[rows], p.tags)
    acc = oracle.gemm_blocks(codes, p.w)
    return grouped.dequant_grouped(acc, scales, s_wg)


@pytest.mark.parametrize("M,N,K,frac,split_mode", [
    (300, 768, 1024, 0.25, -1), (1000, 1024, 2048, 0.05, 1), (512, 384, 768, 1.0, 0), (256, 256, 512, 0.0, 3),
])
def test_grouped_pair_kernel_parity(M, N, K, frac, split_mode):
    """NEXT-3 on the prefill pair kernel (grouped promotion, §7.3 / DESIGN §10): the synthetic
    workload within the FP32 tolerance of oracle/grouped.py."""
    p = synth.make_problem(M, K, N, frac=frac, seed=M + K)
    s_wg = _gs(N, K, M)
    y = _pair_grouped(p, s_wg, split_mode)
    rows = synth.sample_rows(M, 64, p.x)
    ref = _ref_rows(p, s_wg, rows)
    g = y[torch.from_numpy(rows).to(DEV)].cpu().numpy().astype(np.float64)
    bad = np.abs(g - ref) > 1e-3 * np.abs(ref) + 1e-5 * np.abs(ref).max()
    assert not bad.any(), f"{bad.sum()} outputs off; max err {np.abs(g - ref).max()}"


@pytest.mark.parametrize("M,K,N", [(4096, 8192, 28672), (1000, 4096, 2048)])
def test_grouped_pair_kernel_exact(M, K, N):
    """Exact inputs (synth.make_exact_problem) with power-of-two group scales s_w[b, n] = 2^g:
    y = sum_b 2^(e+g) acc_b is exact in binary32, so the pair kernel's grouped FP32 output must
    EQUAL the oracle (LLaMA-3-70B gate/up at M = 4096 included)."""
    p = synth.make_exact_problem(M, K, N, frac=0.05, seed=K + N)
    g = np.random.default_rng(M).integers(-9, -6, size=(K // 128, N))
    s_wg = np.exp2(g).astype(np.float32)
    y = _pair_grouped(p, s_wg)
    rows = np.unique(np.concatenate([np.arange(min(M, 256)), np.arange(M - 32, M)]))
    ref = _ref_rows(p, s_wg, rows)
    r32 = ref.astype(np.float32)
    assert np.array_equal(r32.astype(np.float64), ref), "reference not exact in binary32"
    got = y[torch.from_numpy(rows).to(DEV)].cpu().numpy()
    bad = got != r32
    assert not bad.any(), f"{bad.sum()} grouped outputs differ from the exact value"
