"""Swap-out / swap-in of the bench's mixed-structure set (iid, clustered, channel-dead, constant,
fp16 tensors of 32 MiB) with every codec, twice each and then AUTO, back to back -- the sequence
that bench.py's decision-accuracy pass runs -- with every host container checked against the
oracle and every restore against the input (poisoned outputs)."""
import numpy as np
import pytest

import synth
from oracle import oracle as O
from tests import gpu_util as G

pytestmark = pytest.mark.gpu


def mixed():
    n = 8 << 20
    out = []
    for i, (kind, s) in enumerate([("iid", 0.0), ("iid", 0.99), ("clustered", 0.5), ("clustered", 0.99),
                                   ("dead", 0.8), ("constant", 0.0), ("iid_f16", 0.7)]):
        seed = synth.seed_of(5, 0, 0, i)
        dt = O.F32
        if kind == "iid":
            x = synth.relu_iid(n, s, seed)
        elif kind == "clustered":
            x = synth.relu_clustered(n, s, 512, seed)
        elif kind == "dead":
            x = synth.channel_dead((64, 128, 32, 32), s, seed)
        elif kind == "constant":
            x = synth.constant(n, 0x3F800000)
        else:
            dt = O.F16
            x = synth.relu_iid(2 * n, s, seed, dtype=dt)
        out.append((f"{kind}_{s}", x, dt))
    return out


def test_mixed_set_all_codecs_back_to_back():
    import torch
    C = G.lib()
    for label, x, dt in mixed():
        d = G.to_dev(x)
        for codec in (0, 1, 2, 3, 4, 1, 2, 3, 4, C.AUTO):
            h = C.swap_out(d, x.size, dt, codec)
            out = G.poisoned_words(x.size, dt)
            h.swap_in(out)
            h.wait()
            used = h.query()["codec"]
            assert np.array_equal(G.from_dev(out)[:x.size], x), (label, codec)
            if codec in (1, 2, 3, 4) and x.size * (4 if dt == O.F32 else 2) <= (32 << 20):
                assert h.host_bytes() == O.compress(x, used, dt), (label, codec)
            h.close()
    torch.cuda.synchronize()
