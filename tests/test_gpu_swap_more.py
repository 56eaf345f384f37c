"""More swap-pipeline checks on the GPU: 16-bit swaps for every codec, the
forward-out / reverse-in schedule of bench.py with mixed codecs, streams, corrupted host
containers reported by cswap_handle_wait, the library error word, and selector behaviour on a
BERT-like fp16 set (BASELINE.json configs[3])."""
import ctypes

import numpy as np
import pytest

import synth
from oracle import oracle as O
from tests import gpu_util as G

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def C():
    c = G.lib()
    c.set_format(1 << 20, 1024, 65536)
    yield c
    c.set_format(1 << 22, 1024, 65536)


@pytest.mark.parametrize("dtype", [O.F16, O.BF16])
@pytest.mark.parametrize("codec", [O.NONE, O.ZVC, O.RLE, O.CSR, O.LZ4])
def test_swap_16bit_container_equals_oracle(C, dtype, codec):
    import torch
    n = (1 << 20) + 4097
    x = synth.relu_clustered(n, 0.6, 24, seed=codec * 7 + dtype, dtype=dtype)
    d = G.to_dev(x)
    h = C.swap_out(d, n, dtype, codec)
    h.wait()
    assert h.host_bytes() == O.compress(x, codec, dtype, F=1 << 20, param={3: 1024, 4: 65536}.get(codec, 0))
    out = G.poisoned_words(n, dtype)
    h.swap_in(out)
    h.wait()
    torch.cuda.synchronize()
    assert np.array_equal(G.from_dev(out)[:n], x)
    h.close()


def test_forward_out_reverse_in_schedule_mixed_codecs(C):
    """bench.py's step at small scale: swap out in forward order with different codecs (incl.
    AUTO), swap back in reverse order into fresh buffers; every container equals the oracle's
    and every tensor is restored bitwise."""
    import torch
    specs = [(300000, 0.5, O.ZVC), (70000, 0.9, O.CSR), (123457, 0.99, O.RLE), (200000, 0.3, O.LZ4),
             (50000, 0.0, O.NONE), (400000, 0.7, C.AUTO)]
    xs, hs = [], []
    for i, (n, s, codec) in enumerate(specs):
        x = synth.relu_iid(n, s, seed=100 + i)
        xs.append(x)
        hs.append(C.swap_out(G.to_dev(x), n, C.F32, codec))
    outs = []
    for x, h in reversed(list(zip(xs, hs))):
        o = G.poisoned_words(x.size, 0)
        h.swap_in(o)
        outs.append(o)
    outs.reverse()
    torch.cuda.synchronize()
    for x, h, o in zip(xs, hs, outs):
        h.wait()
        q = h.query()
        assert h.host_bytes() == O.compress(x, q["codec"], O.F32, F=1 << 20, param={3: 1024, 4: 65536}.get(q["codec"], 0))
        assert np.array_equal(G.from_dev(o)[:x.size], x)
        h.close()


def test_swap_on_side_stream_orders_after_pending_work(C):
    """swap_out is ordered after work already queued on the caller's stream."""
    import torch
    n = 1 << 20
    s = torch.cuda.Stream()
    x = synth.relu_iid(n, 0.5, seed=5)
    d = torch.zeros(n, dtype=torch.int32, device="cuda")
    src = G.to_dev(x)
    with torch.cuda.stream(s):
        torch.cuda._sleep(2_000_000)  # keep the stream busy, then fill d
        d.copy_(src)
        h = C.swap_out(d, n, C.F32, C.ZVC, stream=s)
        out = G.poison_like(d)
        h.swap_in(out, stream=s)
    s.synchronize()
    h.wait()
    assert h.host_bytes() == O.compress(x, O.ZVC, O.F32, F=1 << 20)
    assert np.array_equal(G.from_dev(out), x)
    h.close()


@pytest.mark.parametrize("codec", [O.ZVC, O.RLE, O.CSR, O.LZ4])
def test_corrupted_host_container_reported_by_wait(C, codec):
    import torch
    n = 1 << 18
    x = synth.relu_iid(n, 0.6, seed=9)
    h = C.swap_out(G.to_dev(x), n, C.F32, codec)
    h.wait()
    q = h.query()
    # flip the first frame-table entry (bytes 64..71): frame sizes no longer add up
    p = ctypes.cast(q["host"] + 64, ctypes.POINTER(ctypes.c_uint8))
    p[0] ^= 0x10
    out = G.poisoned_words(n, 0)
    h.swap_in(out)
    with pytest.raises(C.CswapError) as e:
        h.wait()
    assert e.value.status == 5  # CORRUPT
    torch.cuda.synchronize()
    h.close()


def test_library_error_word(C):
    import torch
    n = 5000
    x = synth.relu_iid(n, 0.5, seed=3)
    blob = bytearray(O.compress(x, O.ZVC, O.F32, F=1024))
    blob[0] ^= 1
    src = torch.from_numpy(np.frombuffer(bytes(blob), np.uint8).copy()).cuda()
    out = G.poisoned_words(n, 0)
    C.decompress(src, len(blob), out, n, C.F32, C.ZVC, fmt=(1024, 1024, 65536))  # err = NULL
    with pytest.raises(C.CswapError) as e:
        C.check_device_error()
    assert e.value.status == 5
    C.check_device_error()  # cleared


def test_bert_like_fp16_set_selection(C):
    """configs[3] (BERT-large fp16) at 1/32 scale: dense GELU outputs are never compressed;
    every decision equals the oracle selector's on the same probe counts; round trips exact."""
    import torch
    cal = C.get_calibration()
    oc = O.Calib()
    for f, _ in C.Calib._fields_:
        if f == "beta":
            for i in range(len(cal.beta)):
                oc.beta[i] = cal.beta[i]
        elif f != "reserved":
            setattr(oc, f, getattr(cal, f))
    for i, (name, shape, s) in enumerate(synth.bert_large_b8()[:8]):
        n = synth.numel(shape) // 32
        x = synth.relu_iid(n, s, seed=synth.seed_of(4, 1, 0, i), dtype=O.F16)
        h = C.swap_out(G.to_dev(x), n, C.F16, C.AUTO)
        h.wait()
        q = h.query()
        ref = O.select(n, O.F16, O.probe(x, O.F16), 0.0, 0.0, oc)
        assert q["codec"] == ref["codec"], name
        if s == 0.0:
            assert q["codec"] == O.NONE, name
        out = G.poisoned_words(n, O.F16)
        h.swap_in(out)
        h.wait()
        torch.cuda.synchronize()
        assert np.array_equal(G.from_dev(out)[:n], x)
        h.close()


def test_bench_two_ranks_on_one_gpu():
    """bench.py --gpus 2 end to end on the GPU box (both ranks share GPU 0 via BENCH_SHARE_GPU,
    so this checks the launcher / gloo barrier / max-over-ranks / gather path with the real swap
    workload, not scaling): one JSON line, n_gpus = 2, per-rank entries, value = 2 x raw / max."""
    import json
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = {k: v for k, v in os.environ.items() if k not in ("RANK", "LOCAL_RANK", "WORLD_SIZE", "MASTER_ADDR",
                                                            "MASTER_PORT")}
    env["BENCH_SHARE_GPU"] = "1"
    p = subprocess.run([sys.executable, os.path.join(root, "bench.py"), "--gpus", "2", "--steps", "2", "--warmup", "3",
                        "--no-extras", "--no-cpu"], capture_output=True, text=True, timeout=900, env=env, cwd=root)
    assert p.returncode == 0, p.stderr[-3000:]
    lines = [ln for ln in p.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1
    res = json.loads(lines[0])
    assert res["n_gpus"] == 2 and len(res["per_rank"]) == 2
    raw = res["config"]["raw_MiB_per_gpu"] * 2**20
    assert abs(res["value"] - 2 * raw / (res["ms_per_step"] * 1e-3) / 1e9) < 0.01 * res["value"]
