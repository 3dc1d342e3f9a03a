"""CPU (gloo, world size 2) tests of bench.py's multi-GPU harness: the
launcher bench.py uses for `--gpus N` without torchrun spawns N real rank processes with the
torchrun environment, a failing rank fails the launch, device timings are reduced with a MAX
over ranks, and the real rank entry point (bench.rank_main) runs the reference arm on rank 0
only while the other ranks exit 0."""
import json
import os

import pytest

import bench


def _gloo_worker(outdir):
    import torch
    import torch.distributed as dist
    rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
    assert os.environ["LOCAL_RANK"] == str(rank) and os.environ["MASTER_ADDR"] == "127.0.0.1"
    dist.init_process_group("gloo")
    try:
        assert dist.get_world_size() == world == 2
        got = bench.max_over_ranks([1.0 + rank, 10.0 - rank, 3.0], dist, torch, "cpu")
        shards = [bench.shard(28672, 8192, "row", None, rank, world), bench.shard(8192, 28672, "col", None, rank, world)]
        with open(os.path.join(outdir, f"rank{rank}.json"), "w") as f:
            json.dump({"max": got, "shards": shards}, f)
    finally:
        dist.destroy_process_group()
    return 0


def _failing_worker():
    if os.environ["RANK"] == "1":
        raise RuntimeError("rank 1 fails")
    return 0


def test_launch_ranks_gloo(tmp_path):
    bench.launch_ranks(2, _gloo_worker, (str(tmp_path),))
    r = [json.load(open(tmp_path / f"rank{i}.json")) for i in range(2)]
    assert r[0]["max"] == r[1]["max"] == [2.0, 10.0, 3.0]
    # row-parallel: disjoint K halves at block boundaries; column-parallel: disjoint N halves
    assert r[0]["shards"][0] == [0, 14336, 0, 8192] and r[1]["shards"][0] == [14336, 28672, 0, 8192]
    assert r[0]["shards"][1] == [0, 8192, 0, 14336] and r[1]["shards"][1] == [0, 8192, 14336, 28672]


def test_launch_ranks_failure_propagates():
    with pytest.raises(Exception):
        bench.launch_ranks(2, _failing_worker)


def test_world_size_mismatch_is_loud(monkeypatch):
    monkeypatch.setenv("WORLD_SIZE", "2")
    monkeypatch.setenv("RANK", "0")
    with pytest.raises(SystemExit):
        bench.rank_main(["--gpus", "1"])


def test_reference_arm_two_ranks(capfd):
    """The real rank logic through the launcher: rank 0 prints the reference line, rank 1 exits 0."""
    argv = ["--gpus", "2", "--impl", "reference", "--steps", "1", "--warmup", "0"]
    bench.launch_ranks(2, bench.rank_main, (argv,))
    lines = [l for l in capfd.readouterr().out.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["impl"] == "reference" and d["n_gpus"] == 2 and d["cpu_baseline"]["cores"] >= 1
