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


def _run_bench(args, env_extra=None, timeout=240):
    import json
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = {k: v for k, v in os.environ.items() if k not in ("RANK", "LOCAL_RANK", "WORLD_SIZE", "MASTER_ADDR",
                                                            "MASTER_PORT", "LOCAL_WORLD_SIZE")}
    env.update(env_extra or {})
    p = subprocess.run([sys.executable, os.path.join(root, "bench.py"), *args], capture_output=True, text=True,
                       timeout=timeout, env=env, cwd=root)
    lines = [ln for ln in p.stdout.splitlines() if ln.startswith("{")]
    return p.returncode, [json.loads(ln) for ln in lines], p.stderr


def test_bench_gpus_n_spawns_n_replicas_stub():
    """`python bench.py --gpus 2` (no torchrun) starts two rank processes itself; they meet on a
    gloo barrier, rank 0 prints ONE line with n_gpus = 2, the job time is the slowest rank's and
    the throughput counts both ranks' bytes (stub workload: rank r takes 10 (r + 1) ms/step)."""
    rc, out, err = _run_bench(["--gpus", "2", "--stub", "--steps", "2", "--warmup", "3"])
    assert rc == 0, err
    assert len(out) == 1
    res = out[0]
    assert res["n_gpus"] == 2 and res["scaling"] == "weak"
    assert [p["rank"] for p in res["per_rank"]] == [0, 1]
    assert len({p["pid"] for p in res["per_rank"]}) == 2  # two processes
    assert res["ms_per_step"] == pytest.approx(20.0)
    assert res["value"] == pytest.approx(2 * (1 << 20) / 0.020 / 1e9, rel=1e-5)
    assert res["every_compressed_tensor_faster_all_ranks"] is True


def test_bench_rejects_gpu_count_mismatch():
    # under a launcher that started 2 ranks, --gpus 3 is an error (never a silent other N)
    rc, out, err = _run_bench(["--gpus", "3", "--stub"], {"WORLD_SIZE": "2", "RANK": "0", "LOCAL_RANK": "0"})
    assert rc == 2 and not out and "launcher started 2" in err
    # more GPUs than visible (none on this CPU box) is an error too
    rc, out, err = _run_bench(["--gpus", "4", "--no-extras"], timeout=120)
    assert rc == 2 and not out and "visible" in err
