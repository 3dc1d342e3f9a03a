"""GPU parity of the PRODUCTION kernels, bit for bit, at the BASELINE.json sizes.

The debug-accumulator kernels (tests/test_gpu_parity.py) prove integer exactness of narrower
instantiations; this file proves it for the kernels bench.py times -- the cta_group::2 pair
kernel with whole-tile and stream-K plans, the single-CTA prefill kernel, the decode kernel
with its stream-K split -- with the default (auto) plans of configs 2-5 and config 3's
INT8-block-fraction sweep, through the C ABI.

Inputs come from synth.make_exact_problem: every (token, block) is q * 2^e with integer codes
q and one |q| = qmax, and s_w = 2^f, so s_a = 2^e exactly and every partial sum of the
dequantised output is exact in binary32 (P:L164-166 per-block INT accumulation, P:L206
dequantisation).  The FP32 output must then EQUAL the oracle's binary64 value (an integer
combination of powers of two) -- any wrong accumulator code unit, dropped or mis-scaled block
partial, or stream-K fix-up slip shows up as a mismatch.  The FP16 / BF16 outputs must equal
the oracle's value rounded once (RNE) to that type.  The oracle (oracle/) recomputes codes,
scales and accumulators from x on >= 256 sampled rows: one whole 256-token pair tile (every
32-row warp slice of both CTAs), the last 32 rows (ragged tail) and special rows (all-zero,
worst-case |sum q u| = 7 * 15 * 128 = 13,440 per INT4 block against an all-7 weight row,
alternating-sign cancellation)."""
import numpy as np
import pytest

import oracle
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

import paper_conf_asplos_liu0rxpwl0w25_b200 as cb   # noqa: E402
from test_gpu_parity import _check_quant, _quant    # noqa: E402

DEV = "cuda:0"


def _special(M):
    """Special rows: some at the start, some inside the checked pair tile, the last row."""
    t = _tile(M)
    rows = {0: "zero", 1: "all_pos", 2: "alternating", 3: "all_neg"}
    if M > 256:
        rows.update({256 * t + 37: "all_pos", 256 * t + 130: "alternating", 256 * t + 200: "zero",
                     256 * t + 255: "all_neg", M - 1: "all_pos"})
    return rows


def _tile(M):
    return (M // 256) // 2


def _rows(M, seed=0):
    """Rows compared: all rows for M <= 288; else one full 256-token tile, the last 32 rows,
    16 seeded others and the special rows."""
    if M <= 288:
        return np.arange(M, dtype=np.int64)
    t = _tile(M)
    rng = np.random.default_rng(seed)
    rows = set(range(256 * t, min(M, 256 * t + 256))) | set(range(M - 32, M)) | set(_special(M))
    rows |= set(int(r) for r in rng.integers(0, M, size=16))
    return np.array(sorted(rows), dtype=np.int64)


def _x_dev(p):
    if p.bf16:
        return torch.from_numpy(p.x.view(np.int16)).to(DEV).view(torch.bfloat16)
    return torch.from_numpy(p.x).to(DEV)


def run_exact(M, K, N, frac, seed, *, split_mode=-1, orientation=0, tile_w=0, tile_n=0, num_sms=0,
              out_dtypes=(torch.float32, torch.float16), bf16=False, n8=None):
    p = synth.make_exact_problem(M, K, N, frac=frac, seed=seed, bf16=bf16, n8=n8, special_rows=_special(M))
    act, sc = cb.quantize_act(_x_dev(p), p.tags)
    wp = cb.pack_weight(torch.from_numpy(p.w).to(DEV))
    sw = torch.from_numpy(p.s_w).to(DEV)
    plan = cb.Plan(M, N, K, p.tags, split_mode=split_mode, orientation=orientation, tile_w=tile_w,
                   tile_n=tile_n, num_sms=num_sms)
    rows = _rows(M, seed)
    rows_d = torch.from_numpy(rows).to(DEV)
    outs = {}
    for dt in out_dtypes:
        y = cb.w4ax_gemm(plan, act, sc, wp, sw, out_dtype=dt)
        outs[dt] = y[rows_d].cpu()
    torch.cuda.synchronize()
    yref, acc_sum, codes, scales = oracle.w4ax_rows(p.x, p.tags, p.w, p.s_w, rows, bf16_bits=bf16)
    # the generator's promise, checked through the oracle: codes are q, s_a = 2^e (0 for a zero row)
    assert np.array_equal(codes, p.q[rows])
    zero = ~np.any(p.q[rows].reshape(len(rows), -1, 128), axis=2)
    assert np.array_equal(scales, np.where(zero, 0.0, np.exp2(p.e[rows])).astype(np.float32))
    ref32 = yref.astype(np.float32)
    assert np.array_equal(ref32.astype(np.float64), yref), "oracle value not exact in binary32 (generator bound)"
    for dt, got in outs.items():
        if dt == torch.float32:
            g = got.numpy()
            bad = g != ref32
            assert not bad.any(), (f"{bad.sum()} FP32 outputs differ from the exact value; first at "
                                   f"{np.argwhere(bad)[0]}, got {g[bad][0]} want {ref32[bad][0]}")
        elif dt == torch.float16:
            g = got.numpy()
            r16 = yref.astype(np.float16)
            bad = g != r16
            assert not bad.any(), f"{bad.sum()} FP16 outputs differ from the RNE-rounded exact value"
        else:
            r = torch.from_numpy(ref32).to(torch.bfloat16)
            assert torch.equal(got, r), "BF16 outputs differ from the RNE-rounded exact value"
    return plan.info()


CFG2 = [(f"c2_l2_7b_{nm}_m{M}", M, K, N, 0.05)
        for nm, K, N in (("qkvo", 4096, 4096), ("gateup", 4096, 11008), ("down", 11008, 4096))
        for M in (1, 16, 256, 4096)]
CFG3 = [(f"c3_l3_8b_{nm}_m8192_f{int(f * 100)}", 8192, K, N, f)
        for nm, K, N in (("up", 4096, 14336), ("down", 14336, 4096)) for f in (0.0, 0.05, 0.25, 1.0)]
CFG4 = [("c4_l3_70b_gateup_m4096", 4096, 8192, 28672, 0.05), ("c4_l3_70b_down_m4096", 4096, 28672, 8192, 0.05),
        ("c4_l3_70b_qkv_m4096", 4096, 8192, 10240, 0.05)]
CFG5 = [(f"c5_l3_70b_{nm}_m{M}", M, K, N, 0.05)
        for nm, K, N in (("gateup", 8192, 28672), ("down", 28672, 8192), ("qkv", 8192, 10240))
        for M in (1, 4, 8, 32)]
ALL = CFG2 + CFG3 + CFG4 + CFG5


@pytest.mark.parametrize("name,M,K,N,frac", ALL, ids=[c[0] for c in ALL])
def test_production_exact_full_size(name, M, K, N, frac):
    info = run_exact(M, K, N, frac, seed=sum(map(ord, name)))
    # the launch configuration bench.py times: pair kernel for prefill, a decode kernel below 128
    # (the warp-level one for M <= 8 on layers of >= 32 MiB of packed weights)
    o4 = M <= 8 and (N * K // 2 >= (32 << 20) or (N * K // 2 >= (8 << 20) and N >= K))
    assert info["orientation"] == (3 if M >= 256 else (2 if M >= 128 else (4 if o4 else 1)))


O1_DECODE = [c for c in CFG5 if c[1] <= 8 and c[3] * c[2] // 2 >= (32 << 20)]


@pytest.mark.parametrize("name,M,K,N,frac", O1_DECODE, ids=[c[0] + "_o1" for c in O1_DECODE])
def test_tmem_decode_exact_where_auto_is_o4(name, M, K, N, frac):
    """The TMEM decode kernel (orientation 1) at the config-5 sizes whose auto plan is now
    orientation 4, so both decode kernels stay exact at every config-5 point."""
    info = run_exact(M, K, N, frac, seed=sum(map(ord, name)) + 1, orientation=1)
    assert info["orientation"] == 1


@pytest.mark.parametrize("split_mode", [0, 1, 2, 3])
def test_pair_kernel_schedules_exact(split_mode):
    """cta_group::2 pair kernel (256 x 256 tiles) under every scheduler mode, incl. forced
    stream-K with many split tiles (fix-up order) on a ragged M."""
    info = run_exact(1000, 4096, 4096, 0.25, seed=50 + split_mode, split_mode=split_mode, orientation=3)
    if split_mode in (1, 2, 3):
        assert info["n_split_tiles"] > 0


@pytest.mark.parametrize("split_mode", [0, 1, 2, 3])
def test_decode_kernel_schedules_exact(split_mode):
    info = run_exact(32, 8192, 10240, 0.05, seed=60 + split_mode, split_mode=split_mode, orientation=1)
    if split_mode == 1:
        assert info["n_split_tiles"] > 0


@pytest.mark.parametrize("M,tile_w", [(200, 192), (130, 160), (255, 128)])
def test_single_cta_prefill_exact(M, tile_w):
    run_exact(M, 4096, 2048, 0.25, seed=M, orientation=2, tile_w=tile_w)


@pytest.mark.parametrize("tile_w", [128, 160, 192])
def test_pair_tile_widths_exact(tile_w):
    run_exact(1000, 2048, 3840, 0.25, seed=tile_w, orientation=3, tile_w=tile_w)


@pytest.mark.parametrize("tile_n", [16, 32, 64, 128])
def test_decode_tile_widths_exact(tile_n):
    run_exact(100, 4096, 1024, 0.25, seed=tile_n, orientation=1, tile_n=tile_n)


GEMV = [(f"o4_l3_70b_{nm}_m{M}", M, K, N, 0.05)
        for nm, K, N in (("gateup", 8192, 28672), ("down", 28672, 8192), ("qkv", 8192, 10240))
        for M in (1, 4, 8)] + [(f"o4_l2_7b_{nm}_m1", 1, K, N, 0.05)
                               for nm, K, N in (("qkvo", 4096, 4096), ("gateup", 4096, 11008), ("down", 11008, 4096))]


@pytest.mark.parametrize("name,M,K,N,frac", GEMV, ids=[c[0] for c in GEMV])
def test_gemv_exact_full_size(name, M, K, N, frac):
    """Orientation 4 (gemm_v.cu: mma.sync u8 x s8, CTA-level stream-K + ordered reduction) at
    the decode sizes of configs 2 and 5."""
    info = run_exact(M, K, N, frac, seed=sum(map(ord, name)), orientation=4,
                     out_dtypes=(torch.float32, torch.float16, torch.bfloat16))
    assert info["orientation"] == 4


@pytest.mark.parametrize("M,K,N,frac,num_sms", [
    (3, 28672, 128, 0.25, 3),      # one row group over 6 CTAs: every CTA a segment of one group
    (5, 1024, 8192, 1.0, 2),       # all INT8 blocks; 4 CTAs: ranges of 16 groups (many segments)
    (8, 2048, 1024, 0.0, 148),     # more CTAs than units: empty ranges
    (2, 4096, 2048, 0.5, 7),       # ranges cutting groups at odd K-blocks
    (1, 128, 128, 0.0, 148),       # one unit: one CTA
    (7, 256, 128, 1.0, 148),       # one K-block, two groups, all INT8
])
def test_gemv_schedules_exact(M, K, N, frac, num_sms):
    info = run_exact(M, K, N, frac, seed=M * 7 + num_sms, orientation=4, num_sms=num_sms)
    assert info["orientation"] == 4


def test_bf16_inputs_and_outputs_exact():
    """Config 2's BF16 variant: bf16 activations in, bf16 / fp32 out."""
    run_exact(4096, 4096, 4096, 0.05, seed=77, bf16=True, out_dtypes=(torch.float32, torch.bfloat16))
    run_exact(16, 4096, 11008, 0.05, seed=78, bf16=True, out_dtypes=(torch.float32, torch.bfloat16))


def test_reduced_grid_exact():
    """A persistent grid smaller than the device (e.g. another kernel holds SMs)."""
    run_exact(2048, 4096, 4096, 0.05, seed=91, num_sms=30)
    run_exact(8, 8192, 8192, 0.05, seed=92, num_sms=17)


# ----------------------------------------------------------------------------- kernel 1, in full

def test_quantize_config3_full_oracle():
    """Kernel 1 on config 3's largest input (LLaMA-3-8B down, M = 8192, K = 14336): every code,
    scale, code sum and correction term against the oracle run IN FULL."""
    p = synth.make_problem(8192, 14336, 128, frac=0.05, seed=3)
    act, sc = _quant(p)
    _check_quant(p, act, sc)


@pytest.mark.parametrize("frac", [0.0, 0.25, 1.0])
def test_quantize_config3_sweep_full_oracle(frac):
    p = synth.make_problem(8192, 4096, 128, frac=frac, seed=4)
    act, sc = _quant(p)
    _check_quant(p, act, sc)


# ----------------------------------------------------------------------------- widening (I9)

@pytest.mark.parametrize("int8_block", [False, True])
def test_widen_exhaustive_all_words(int8_block):
    """Pin I9, exhaustive: the GEMM kernels' widening of every one of the 2^32
    packed words equals the layout definition of include/comet.h (byte i of the word holds
    channels i (low nibble) and i + 4 (high nibble), offset binary u = w + 8; INT4 block byte =
    u, INT8 block byte = 16 (u - 8)), written here in torch."""
    chunk = 1 << 28
    out = torch.empty((chunk, 2), dtype=torch.int32, device=DEV)
    sh = torch.arange(4, device=DEV, dtype=torch.int64) * 8
    for c in range((1 << 32) // chunk):
        first = c * chunk
        cb.debug_widen(first, chunk, int8_block, out=out)
        v = torch.arange(first, first + chunk, device=DEV, dtype=torch.int64)
        lo_u = (v[:, None] >> sh) & 0xF             # channels 0..3
        hi_u = (v[:, None] >> (sh + 4)) & 0xF       # channels 4..7
        if int8_block:
            lo_b, hi_b = (16 * (lo_u - 8)) & 0xFF, (16 * (hi_u - 8)) & 0xFF
        else:
            lo_b, hi_b = lo_u, hi_u
        lo_w = (lo_b << sh).sum(1)
        hi_w = (hi_b << sh).sum(1)
        got = out.to(torch.int64) & 0xFFFFFFFF
        assert torch.equal(got[:, 0], lo_w) and torch.equal(got[:, 1], hi_w), f"chunk {c}"


# ----------------------------------------------------------------------------- host-buffer path

def test_linear_host_async_small_m_wait():
    """comet_linear_host_wait must block until y_host is complete on the single-chunk path
    (M < 2048) too: no device synchronize here, only the wait."""
    M, K, N = 300, 4096, 4096
    p = synth.make_exact_problem(M, K, N, frac=0.05, seed=5)
    wp = cb.pack_weight(torch.from_numpy(p.w).to(DEV))
    sw = torch.from_numpy(p.s_w).to(DEV)
    plan = cb.Plan(M, N, K, p.tags)
    x_host = torch.from_numpy(p.x).pin_memory()
    y_host = torch.empty((M, N), dtype=torch.float16).pin_memory()
    scratch = torch.empty(cb.linear_scratch_bytes(plan, cb.COMET_F16, cb.COMET_F16), dtype=torch.uint8, device=DEV)
    yref, _, _, _ = oracle.w4ax(p.x, p.tags, p.w, p.s_w)
    r16 = yref.astype(np.float16)
    for it in range(3):
        y_host.fill_(float("nan"))
        torch.cuda._sleep(int(2e7))          # keep the stream busy so a non-blocking wait would be caught
        cb.w4ax_linear_host(plan, x_host, wp, sw, y_host, scratch, blocking=False)
        cb.linear_host_wait(plan)
        assert np.array_equal(y_host.numpy(), r16), f"iteration {it}: y_host incomplete after linear_host_wait"
