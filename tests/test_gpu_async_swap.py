"""Swap-out is asynchronous and pipelined per frame (§8 row a11; "compression in
parallel before swapping", :228 async stream + cudaMemcpyAsync, Fig. 2 :64-72; R7):
a fixed-codec cswap_swap_out returns while the caller's stream is still busy, the container the
executor thread copies frame by frame equals the oracle's bytes, swap-in orders its H2D after the
D2H on the device, and a corrupted host container is reported, never read out of bounds."""
import time

import numpy as np
import pytest

import synth
from oracle import oracle as O
from tests import gpu_util as G

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def C():
    return G.lib()


@pytest.mark.parametrize("codec", [1, 2, 3, 4, 0])
def test_swap_out_returns_while_the_stream_is_busy(C, codec):
    import torch
    n = (3 << 22) + 777  # 4 frames, ragged
    x = synth.relu_iid(n, 0.6, seed=31 + codec)
    d = G.to_dev(x)
    h = C.swap_out(d, n, C.F32, codec)  # warm-up: graph instantiation, pools
    h.wait()
    h.close()
    torch.cuda.synchronize()
    torch.cuda._sleep(400_000_000)  # ~0.2 s of device time queued ahead of the swap-out
    t0 = time.perf_counter()
    h = C.swap_out(d, n, C.F32, codec)
    host_s = time.perf_counter() - t0
    still_busy = not torch.cuda.current_stream().query()
    assert still_busy and host_s < 0.02, host_s
    h.wait()
    assert h.host_bytes() == O.compress(x, codec, O.F32)
    out = G.poisoned_words(n, 0)
    h.swap_in(out)
    h.wait()
    assert np.array_equal(G.from_dev(out)[:n], x)
    h.close()


def test_swap_out_host_time_large_tensor(C):
    """VGG16 relu1_1 (784 MiB fp32, 49 frames): the call only enqueues (no device wait)."""
    import torch
    name, shape, s = synth.vgg16_b64()[0]
    n = synth.numel(shape)
    d = synth.relu_iid_torch(n, s, seed=synth.seed_of(3, 0, 0, 0), dtype=0, device="cuda")
    for _ in range(2):
        C.swap_out(d, n, C.F32, C.ZVC).close()
    torch.cuda.synchronize()
    torch.cuda._sleep(100_000_000)
    times = []
    hs = []
    for _ in range(3):
        t0 = time.perf_counter()
        hs.append(C.swap_out(d, n, C.F32, C.ZVC))
        times.append(time.perf_counter() - t0)
    assert min(times) < 2e-3, times  # includes the ctypes call from Python
    for h in hs:
        h.wait()
    out = G.poison_like(d)
    hs[-1].swap_in(out)
    hs[-1].wait()
    assert torch.equal(out, d)
    for h in hs:
        h.close()


@pytest.mark.parametrize("publish", ["auto", "1", "0"])
def test_many_outstanding_swaps_fifo(C, publish, monkeypatch):
    """20 swap-outs queued back to back (mixed codecs, f32/f16) complete in order and each
    container equals the oracle -- with per-frame publication from inside the ZVC kernel chosen
    by the runtime (link idle), forced on, or forced off (CSWAP_FRAME_PUBLISH)."""
    import torch
    if publish != "auto":
        monkeypatch.setenv("CSWAP_FRAME_PUBLISH", publish)
    items = []
    for i in range(20):
        dt = O.F32 if i % 3 else O.F16
        n = 100_000 + 37_123 * i
        x = synth.relu_clustered(n, 0.4 + 0.02 * i, 40, seed=100 + i, dtype=dt)
        items.append((x, dt, [1, 2, 3, 4, 0][i % 5]))
    ds = [G.to_dev(x) for x, _, _ in items]
    hs = [C.swap_out(d, x.size, dt, c) for d, (x, dt, c) in zip(ds, items)]
    for h, (x, dt, c) in zip(hs, items):
        h.wait()
        assert h.host_bytes() == O.compress(x, c, dt)
    for h, (x, dt, c) in zip(hs, items):
        out = G.poisoned_words(x.size, dt)
        h.swap_in(out)
        h.wait()
        assert np.array_equal(G.from_dev(out)[:x.size], x)
        h.close()
    torch.cuda.synchronize()


@pytest.mark.parametrize("codec", [1, 2, 3, 4])
def test_corrupted_multiframe_host_container_is_reported(C, codec):
    """a corrupted frame table in the host copy (K = 5 > 1 pipeline step) must be
    reported by cswap_handle_wait; the H2D ranges come from the kernel-published frame ends, so
    nothing is read or written out of bounds, and the next swap works."""
    import ctypes
    import torch
    C.set_format(1 << 20, 1024, 65536)
    try:
        n = (4 << 20) + 999
        x = synth.relu_iid(n, 0.5, seed=77)
        d = G.to_dev(x)
        for corrupt in ("swap", "huge"):
            h = C.swap_out(d, n, C.F32, codec)
            h.wait()
            q = h.query()
            fb = (ctypes.c_uint64 * 5).from_address(q["host"] + 64)
            if corrupt == "swap":  # same total, frames 1 and 2 exchanged sizes
                fb[1], fb[2] = fb[2], fb[1]
                if fb[1] == fb[2]:
                    fb[1] += 16
            else:
                fb[3] = 1 << 40
            out = G.poisoned_words(n, 0)
            h.swap_in(out)
            with pytest.raises(C.CswapError) as ei:
                h.wait()
            assert ei.value.status == 5
            h.close()
        h = C.swap_out(d, n, C.F32, codec)
        out = G.poisoned_words(n, 0)
        h.swap_in(out)
        h.wait()
        assert np.array_equal(G.from_dev(out)[:n], x)
        h.close()
        torch.cuda.synchronize()
    finally:
        C.set_format(1 << 22, 1024, 65536)


def test_release_cached_keeps_live_containers(C):
    """cswap_release_cached trims the staging pool and unpins empty host chunks; live containers
    stay intact and restorable."""
    n = 3 << 20
    x = synth.relu_iid(n, 0.5, seed=404)
    d = G.to_dev(x)
    live = C.swap_out(d, n, C.F32, C.ZVC)
    for _ in range(3):
        C.swap_out(d, n, C.F32, C.RLE).close()
    live.wait()
    C.release_cached(0)
    assert live.host_bytes() == O.compress(x, O.ZVC, O.F32)
    out = G.poisoned_words(n, 0)
    live.swap_in(out)
    live.wait()
    assert np.array_equal(G.from_dev(out)[:n], x)
    live.close()
    h = C.swap_out(d, n, C.F32, C.ZVC)  # pools grow again after the release
    h.wait()
    assert h.host_bytes() == O.compress(x, O.ZVC, O.F32)
    h.close()
