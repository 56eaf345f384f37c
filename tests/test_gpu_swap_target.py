"""NEXT-4b swap target (beyond the paper): containers stored in device memory
instead of pinned host memory -- a peer GPU over NVLink on a multi-GPU node, this GPU's own HBM
on the one-GPU box the tests run on (the same code path minus the NVLink hop).  The codec
kernels write the container straight into the target's pool and the decoders read it from
there; the container bytes equal the oracle's and the round trip is bitwise."""
import numpy as np
import pytest

import synth
from oracle import oracle as O
from tests import gpu_util as G

pytestmark = pytest.mark.gpu


@pytest.fixture()
def C():
    C = G.lib()
    C.set_swap_target(0)  # this device's HBM (the box has one GPU)
    yield C
    C.set_swap_target(-1)


@pytest.mark.parametrize("codec", [0, 1, 2, 3, 4])
@pytest.mark.parametrize("dtype", [O.F32, O.F16])
def test_device_target_container_equals_oracle_and_round_trips(C, codec, dtype):
    import torch
    assert C.get_swap_target() == 0
    n = (5 << 20) + 4321 if dtype == O.F32 else (9 << 20) + 77  # K = 2 / 3 frames, ragged
    x = synth.relu_clustered(n, 0.55, 30, seed=900 + codec, dtype=dtype)
    d = G.to_dev(x)
    h = C.swap_out(d, n, dtype, codec)
    q = h.query()
    assert q["host"] is None and q["codec"] == codec
    assert h.container_bytes() == O.compress(x, codec, dtype)
    for _ in range(2):  # swap-in may be repeated
        out = G.poisoned_words(n, dtype)
        h.swap_in(out)
        h.wait()
        assert np.array_equal(G.from_dev(out)[:n], x)
    h.close()
    torch.cuda.synchronize()


def test_device_target_auto_and_back_to_host(C):
    n = 1 << 22
    x = synth.relu_iid(n, 0.6, seed=5)
    d = G.to_dev(x)
    h = C.swap_out(d, n, O.F32, C.AUTO)
    out = G.poisoned_words(n, 0)
    h.swap_in(out)
    h.wait()
    assert np.array_equal(G.from_dev(out)[:n], x)
    assert h.container_bytes() == O.compress(x, h.query()["codec"], O.F32)
    h.close()
    C.set_swap_target(-1)
    h = C.swap_out(d, n, O.F32, C.ZVC)
    assert h.query()["host"] is not None
    h.wait()
    assert h.host_bytes() == h.container_bytes() == O.compress(x, O.ZVC, O.F32)
    h.close()


def test_unreachable_target_is_reported(C):
    with pytest.raises(C.CswapError) as e:
        C.set_swap_target(64)
    assert e.value.status == 1  # INVALID: no such device
    assert C.get_swap_target() == 0  # unchanged
