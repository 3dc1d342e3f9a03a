"""GPU smoke of bench.py's N > 1 NEXT-2 comparison (bench.fused_rs_compare) in a one-rank NCCL
group: symmetric-memory receive buffer, fused GEMM + device barrier + owner reduction, and the
NCCL baselines all run and agree with each other on the reduced rows."""
import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

import bench                                          # noqa: E402
import paper_conf_asplos_liu0rxpwl0w25_b200 as cb     # noqa: E402
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth  # noqa: E402


def test_fused_rs_compare_one_rank():
    import torch.distributed as dist
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dev = torch.device("cuda", 0)
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=dev)
    try:
        M, K, N = bench.M_TOKENS, 1024, 1024
        p = synth.make_problem(M, K, N, frac=0.25, seed=4)
        act, sc = cb.quantize_act(torch.from_numpy(p.x).to(dev), p.tags)
        L = dict(name="down", K=K, N=N, kind="row", tags=p.tags, plan=cb.Plan(M, N, K, p.tags, orientation=3),
                 act=act, sc=sc, wp=cb.pack_weight(torch.from_numpy(p.w).to(dev)),
                 sw=torch.from_numpy(p.s_w).to(dev))
        out = bench.fused_rs_compare(cb, torch, dist, dev, [L], 0, 1, 3)
        assert "error" not in out, out
        for k in ("gemm_allreduce_ms", "gemm_nccl_reduce_scatter_ms", "fused_gemm_rs_ms"):
            assert out[k] > 0
    finally:
        dist.destroy_process_group()
