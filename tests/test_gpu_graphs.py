"""Launch groups replayed as CUDA graphs (api.cu run_group): the graph path is the
one that runs, a cached executable graph updated in place for a differently sized / shaped
call still produces the oracle's bytes, and the plain-launch path (CSWAP_GRAPHS=0, in a
subprocess) gives the same containers."""
import os
import subprocess
import sys

import numpy as np
import pytest

import synth
from oracle import oracle as O
from tests import gpu_util as G

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def C():
    return G.lib()


def test_swap_uses_graphs(C):
    import torch
    n = (1 << 21) + 77
    x = synth.relu_iid(n, 0.5, seed=3)
    d = G.to_dev(x)
    g0, _ = C.graph_stats()
    h = C.swap_out(d, n, C.F32, C.ZVC)
    out = G.poisoned_words(n, 0)
    h.swap_in(out)
    h.wait()
    torch.cuda.synchronize()
    g1, _ = C.graph_stats()
    assert g1 - g0 >= 2, "compress and decode groups should each be one graph launch"
    assert np.array_equal(G.from_dev(out)[:n], x)
    h.close()


@pytest.mark.parametrize("codec", [1, 2, 3, 4])
def test_graph_reuse_across_sizes(C, codec):
    """The same (stream, group) executable graph is updated with new pointers, sizes and grid
    shapes on every call: alternate sizes that change the frame count and the tail."""
    import torch
    C.set_format(1 << 20, 1024, 65536)
    try:
        for i, n in enumerate([5000, (1 << 20) * 3 + 17, 1 << 20, 33, (1 << 21) + 1024, 5000]):
            for dt in (0, 1):
                x = synth.relu_clustered(n, 0.6, 32, seed=100 + i, dtype=dt) if codec == 4 else \
                    synth.relu_iid(n, 0.6, seed=100 + i, dtype=dt)
                ref = O.compress(x, codec, dt, F=1 << 20, param={3: 1024, 4: 65536}.get(codec, 0))
                assert G.gpu_compress(C, x, codec, dt, fmt=(1 << 20, 1024, 65536)) == ref, (n, dt)
                y, err = G.gpu_decompress(C, ref, n, dt, codec, fmt=(1 << 20, 1024, 65536))
                assert err == 0 and np.array_equal(y, x), (n, dt)
                d = G.to_dev(x)
                h = C.swap_out(d, n, dt, codec)
                h.wait()
                assert h.host_bytes() == ref
                out = G.poisoned_words(n, dt)
                h.swap_in(out)
                h.wait()
                torch.cuda.synchronize()
                assert np.array_equal(G.from_dev(out)[:n], x)
                h.close()
    finally:
        C.set_format(1 << 22, 1024, 65536)


def test_plain_launch_path_matches():
    """CSWAP_GRAPHS=0: same containers through plainly launched kernels (fresh process)."""
    code = (
        "import numpy as np, torch, synth\n"
        "from oracle import oracle as O\n"
        "from tests import gpu_util as G\n"
        "C = G.lib()\n"
        "for codec in (1, 2, 3, 4):\n"
        "    n = (1 << 22) + 999\n"
        "    x = synth.relu_iid(n, 0.7, seed=codec)\n"
        "    d = G.to_dev(x)\n"
        "    h = C.swap_out(d, n, 0, codec); h.wait()\n"
        "    assert h.host_bytes() == O.compress(x, codec, 0), codec\n"
        "    out = G.poisoned_words(n, 0); h.swap_in(out); h.wait(); torch.cuda.synchronize()\n"
        "    assert np.array_equal(G.from_dev(out)[:n], x), codec\n"
        "    h.close()\n"
        "assert C.graph_stats()[0] == 0\n"
        "print('plain ok')\n")
    env = dict(os.environ, CSWAP_GRAPHS="0")
    r = subprocess.run([sys.executable, "-c", code], cwd=ROOT, env=env, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0 and "plain ok" in r.stdout, r.stderr[-3000:]


@pytest.mark.parametrize("grid,variant", [(1, 0), (7, 1), (148, 2), (296, 3), (0, 4), (5, 5),
                                           (148, 6), (0, 7), (300, 8), (0, 9), (3, 9), (0, -1)])
@pytest.mark.parametrize("dtype", [0, 1])
def test_zvc_launch_config_keeps_bytes(C, grid, variant, dtype):
    """cswap_set_zvc_launch changes only how the persistent compress runs, never its bytes (incl.
    variant 9's 24 KiB tiles: 683 tiles per 2^22-element frame, a short last tile per frame)."""
    n = (9 << 20) + 333 if dtype == 0 else (17 << 20) + 77  # 3 / 5 frames, ragged
    x = synth.relu_iid(n, 0.45, seed=11, dtype=dtype)
    ref = O.compress(x, O.ZVC, dtype)
    try:
        C.set_zvc_launch(grid, variant)
        assert G.gpu_compress(C, x, O.ZVC, dtype) == ref
    finally:
        C.set_zvc_launch(0, -1)


def test_zvc_launch_config_rejects_bad_variant(C):
    with pytest.raises(C.CswapError):
        C.set_zvc_launch(0, 10)


def test_timing_records_carry_device_clock(C):
    """Timed launch groups carry a device-clock duration (stamp kernels) next to the event time."""
    import torch
    n = 8 << 20
    x = synth.relu_iid(n, 0.5, seed=5)
    d = G.to_dev(x)
    out = G.poisoned_words(n, 0)
    C.collect_kernel_timing()
    C.set_kernel_timing(True)
    try:
        h = C.swap_out(d, n, C.F32, C.ZVC)
        h.swap_in(out)
        h.wait()
        torch.cuda.synchronize()
    finally:
        C.set_kernel_timing(False)
    recs = [r for r in C.collect_kernel_timing() if r["direction"] in (0, 1)]
    # the persistent ZVC compress clocks itself (no stamp kernels in its group); the decode
    # groups carry stamp kernels
    comp = [r for r in recs if r["direction"] == 0]
    dec = [r for r in recs if r["direction"] == 1]
    assert comp and all(0 < r["kernel_ms"] <= r["ms"] * 1.05 + 0.01 and r["device_ms"] == 0 for r in comp), comp
    assert dec and all(0 < r["device_ms"] <= r["ms"] * 1.05 + 0.01 and r["kernel_ms"] == 0 for r in dec), dec
    assert comp[0]["comp_bytes"] > 0, comp
    assert np.array_equal(G.from_dev(out)[:n], x)
    h.close()


def test_many_streams_evict_graph_cache(C):
    """More (stream, group) pairs than the executable-graph cache holds: evicted graphs must not
    disturb later launches."""
    import torch
    n = 100_000
    x = synth.relu_iid(n, 0.5, seed=9)
    ref = O.compress(x, O.ZVC, O.F32)
    d = G.to_dev(x)
    cap = C.max_compressed_size(n, C.F32, C.ZVC)
    size = torch.zeros(1, dtype=torch.int64, device="cuda")
    for i in range(80):
        s = torch.cuda.Stream()
        out = torch.zeros(cap, dtype=torch.uint8, device="cuda")
        s.wait_stream(torch.cuda.current_stream())
        C.compress(d, n, C.F32, C.ZVC, out, cap, size, stream=s)
        s.synchronize()
        assert out[: int(size.item())].cpu().numpy().tobytes() == ref, i
