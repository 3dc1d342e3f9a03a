"""Multi-process (world size 2, gloo, CPU) tests of the tensor-parallel path bench.py runs at
N GPUs: the shard() split, local quantisation of a K shard, and
the collectives that reassemble the layer -- column-parallel layers need none (the N shards
are disjoint outputs), the row-parallel layer sums FP partials with all_reduce.  Each rank
computes its shard with the CPU oracle; the result must equal the unsharded oracle."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
from bench import shard
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth

WORLD = 2


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, port, kind, M, K, N, seed, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=WORLD)
    try:
        p = synth.make_problem(M, K, N, frac=0.25, seed=seed)
        k0, k1, n0, n1 = shard(K, N, kind, p.tags, rank, WORLD)
        x_l = np.ascontiguousarray(p.x[:, k0:k1])
        t_l = np.ascontiguousarray(p.tags[k0 // 128:k1 // 128])
        w_l = np.ascontiguousarray(p.w[n0:n1, k0:k1])
        y_l, acc_l, codes_l, scales_l = oracle.w4ax(x_l, t_l, w_l, p.s_w[n0:n1])
        y = torch.from_numpy(np.ascontiguousarray(y_l))
        if kind == "row":
            dist.all_reduce(y, op=dist.ReduceOp.SUM)          # the one collective of the path
            full = y
        else:
            parts = [torch.empty_like(y) for _ in range(WORLD)]
            dist.all_gather(parts, y)                         # test-side reassembly only
            full = torch.cat(parts, dim=1)
        codes_parts = [torch.empty_like(torch.from_numpy(codes_l)) for _ in range(WORLD)]
        dist.all_gather(codes_parts, torch.from_numpy(np.ascontiguousarray(codes_l)))
        if rank == 0:
            q.put((full.numpy(), [c.numpy() for c in codes_parts], (k0, k1, n0, n1)))
    finally:
        dist.destroy_process_group()


def _run(kind, M, K, N, seed):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, port, kind, M, K, N, seed, q)) for r in range(WORLD)]
    for p in procs:
        p.start()
    out = q.get(timeout=120)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    return out


def test_shard_bounds():
    # column: N split into equal multiples of 128; row: K split at 128-channel block boundaries
    for world in (2, 4, 8):
        for r in range(world):
            k0, k1, n0, n1 = shard(8192, 28672, "col", None, r, world)
            assert (k0, k1) == (0, 8192) and n1 - n0 == 28672 // world and n0 % 128 == 0
            k0, k1, n0, n1 = shard(28672, 8192, "row", None, r, world)
            assert (n0, n1) == (0, 8192) and k1 - k0 == 28672 // world and k0 % 128 == 0
    assert shard(256, 256, "row", None, 0, 1) == (0, 256, 0, 256)


@pytest.mark.parametrize("kind", ["col", "row"])
def test_tp2_matches_unsharded_oracle(kind):
    M, K, N, seed = 6, 512, 256, 11
    y_tp, codes_parts, _ = _run(kind, M, K, N, seed)
    p = synth.make_problem(M, K, N, frac=0.25, seed=seed)
    y, acc, codes, scales = oracle.w4ax(p.x, p.tags, p.w, p.s_w)
    if kind == "col":
        # disjoint output columns: bit-identical
        np.testing.assert_array_equal(y_tp, y)
        np.testing.assert_array_equal(codes_parts[0], codes)
    else:
        # local quantisation of each K shard is the full quantisation restricted to it
        # (scales are per (token, block), reading R1) ...
        np.testing.assert_array_equal(np.concatenate(codes_parts, axis=1), codes)
        # ... and the all-reduced partials equal the full sum up to binary64 summation order
        np.testing.assert_allclose(y_tp, y, rtol=1e-12, atol=1e-12)
