"""GPU tests of NEXT-2: the row-parallel layer's reduce-scatter fused into the
prefill GEMM epilogue (comet_w4ax_gemm_rs + comet_rs_reduce; "operator pipelining").

Tensor parallelism is simulated in one process on one GPU: `world` ranks each own a K shard of
the layer at 128-channel block boundaries (their own kernel 1 over their shard, their own plan)
and a receive buffer; every rank's GEMM writes its partial rows into the owners' buffers exactly
as it would into peer memory over NVLink (the pointers are plain device addresses either way),
then every owner reduces.  With exact inputs (synth.make_exact_problem) the per-shard partials
and their sum are exact in binary32, so the reassembled output must EQUAL the unsharded oracle;
on the synthetic workload it must match within the usual tolerance."""
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
from test_gpu_exact import _rows, _special           # noqa: E402

DEV = "cuda:0"


def _x_dev(x, bf16=False):
    if bf16:
        return torch.from_numpy(np.ascontiguousarray(x).view(np.int16)).to(DEV).view(torch.bfloat16)
    return torch.from_numpy(np.ascontiguousarray(x)).to(DEV)


def run_rs(p, world, out_dtype=torch.float32, split_mode=-1):
    M, K, N = p.M, p.K, p.N
    assert K % (128 * world) == 0
    kl = K // world
    recv = [torch.full((cb.rs_recv_bytes(M, N, world) // 4,), float("nan"), dtype=torch.float32, device=DEV)
            for _ in range(world)]
    ptrs = [t.data_ptr() for t in recv]
    plans = []
    for r in range(world):
        k0, k1 = r * kl, (r + 1) * kl
        tags = np.ascontiguousarray(p.tags[k0 // 128:k1 // 128])
        act, sc = cb.quantize_act(_x_dev(p.x[:, k0:k1], p.bf16), tags)
        wp = cb.pack_weight(torch.from_numpy(np.ascontiguousarray(p.w[:, k0:k1])).to(DEV))
        plan = cb.Plan(M, N, kl, tags, orientation=3, split_mode=split_mode)
        plans.append(plan)
        cb.w4ax_gemm_rs(plan, act, sc, wp, torch.from_numpy(p.s_w).to(DEV), ptrs, r)
    torch.cuda.synchronize()            # every rank's GEMM done before any owner reduces
    parts = [cb.rs_reduce(recv[r], world, r, M, N, out_dtype=out_dtype) for r in range(world)]
    torch.cuda.synchronize()
    return torch.cat(parts, dim=0)


@pytest.mark.parametrize("world", [1, 2, 4, 8])
def test_fused_rs_exact(world):
    """Row-parallel LLaMA-3-70B down shape class (K sharded), exact inputs: bit-exact FP32."""
    M, K, N = 1000, 8192, 2048
    p = synth.make_exact_problem(M, K, N, frac=0.05, seed=100 + world, special_rows=_special(M))
    y = run_rs(p, world)
    rows = _rows(M)
    yref, _, _, _ = oracle.w4ax_rows(p.x, p.tags, p.w, p.s_w, rows)
    got = y[torch.from_numpy(rows).to(DEV)].cpu().numpy()
    assert np.array_equal(got, yref.astype(np.float32)), "fused reduce-scatter output differs from the exact value"


def test_fused_rs_full_size_down_tp8():
    """LLaMA-3-70B down (28672 -> 8192) at M = 4096 over 8 simulated ranks (K shard 3584),
    exact inputs, stream-K plans: bit-exact FP32 and RNE-exact FP16 outputs."""
    M, K, N = 4096, 28672, 8192
    p = synth.make_exact_problem(M, K, N, frac=0.05, seed=7, special_rows=_special(M))
    rows = _rows(M)
    yref, _, _, _ = oracle.w4ax_rows(p.x, p.tags, p.w, p.s_w, rows)
    y32 = run_rs(p, 8)
    assert np.array_equal(y32[torch.from_numpy(rows).to(DEV)].cpu().numpy(), yref.astype(np.float32))
    y16 = run_rs(p, 8, out_dtype=torch.float16)
    assert np.array_equal(y16[torch.from_numpy(rows).to(DEV)].cpu().numpy(), yref.astype(np.float16))


@pytest.mark.parametrize("world,split_mode", [(2, 0), (4, 1)])
def test_fused_rs_synthetic_workload(world, split_mode):
    """The synthetic workload (N(0,1) activations with outlier channels): within tolerance of
    the unsharded oracle (the rank sum adds one more binary32 rounding per element)."""
    p = synth.make_problem(512, 4096, 1024, frac=0.05, seed=3)
    y = run_rs(p, world, split_mode=split_mode)
    yref, _, _, _ = oracle.w4ax(p.x, p.tags, p.w, p.s_w)
    _close(y, yref, torch.float32)


def test_fused_rs_rejects_non_pair_plan():
    p = synth.make_problem(64, 1024, 256, frac=0.05, seed=1)
    act, sc = cb.quantize_act(_x_dev(p.x), p.tags)
    wp = cb.pack_weight(torch.from_numpy(p.w).to(DEV))
    recv = torch.zeros(cb.rs_recv_bytes(64, 256, 1) // 4, device=DEV)
    plan = cb.Plan(64, 256, 1024, p.tags)          # decode orientation
    with pytest.raises(cb.CometError) as e:
        cb.w4ax_gemm_rs(plan, act, sc, wp, torch.from_numpy(p.s_w).to(DEV), [recv.data_ptr()], 0)
    assert e.value.status == 2
