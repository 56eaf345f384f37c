"""World-size-2 gloo checks of bench.py's multi-GPU host logic (CPU only): replicas draw
distinct inputs, the job time is the max over ranks, and the whole-job throughput counts every
rank's bytes (independent replicas, no data-path collective)."""
import os
import socket

import pytest
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    import bench
    import synth
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    ms = [10.0, 25.0][rank]
    mx = bench._max_over_ranks(ms, dist)
    seed = bench.rank_seed(synth.seed_of(3, 0, 0, 1), rank)
    x = synth.relu_iid(4096, 0.5, seed=seed)
    gathered = [None] * world
    dist.all_gather_object(gathered, (seed, int(x[:64].sum())))
    q.put((rank, mx, gathered))
    dist.barrier()
    dist.destroy_process_group()


def test_gloo_two_ranks():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, mx, gathered in res:
        assert mx == 25.0  # slowest rank
        (s0, h0), (s1, h1) = gathered
        assert s0 != s1 and h0 != h1  # replicas swap different tensors


def test_job_throughput_counts_all_ranks():
    import bench
    raw = 2180.5 * 2**20
    one = bench.job_throughput(1, raw, 46.4)
    eight = bench.job_throughput(8, raw, 46.4)
    assert eight == pytest.approx(8 * one)
    assert one == pytest.approx(raw / 0.0464 / 1e9)
