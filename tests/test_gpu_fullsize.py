"""Full-size parity (BASELINE.json configs[1] top end: 1 GiB tensors; configs[3] f16) for every
codec, in the launch configuration bench.py uses (swap_out/swap_in, F = 2^22): the oracle checks
sampled frames one by one (frame 0, 1, the middle and the ragged last frame), the frame table
and the total are checked against the container geometry, and the round trip is checked in full."""
import struct

import numpy as np
import pytest

import synth
from oracle import oracle as O
from tests import gpu_util as G

pytestmark = pytest.mark.gpu

F = 1 << 22


@pytest.fixture(scope="module")
def C():
    c = G.lib()
    c.set_format(F, 1024, 65536)
    return c


def _a16(x):
    return (x + 15) // 16 * 16


@pytest.mark.parametrize("dtype,n", [(O.F32, (1 << 28) - 777), (O.F16, (1 << 29) - 4097)])
@pytest.mark.parametrize("codec", [O.ZVC, O.RLE, O.CSR, O.LZ4])
def test_full_size_sampled_frames(C, codec, dtype, n):
    import torch
    # 1 GiB, iid ReLU mask at s = 0.5 for the sparse codecs; RLE and LZ4 get the clustered
    # structure they are meant for (long zero runs) built on the device from a seeded mask
    d = synth.relu_iid_torch(n, 0.5, seed=synth.seed_of(2, 9, codec, dtype), dtype=dtype, device="cuda")
    if codec in (O.RLE, O.LZ4):
        g = torch.Generator(device="cuda")
        g.manual_seed(synth.seed_of(2, 9, codec, dtype) + 1)
        runs = torch.rand(-(-n // 512), generator=g, device="cuda") < 0.6  # 60 % of 512-blocks zeroed
        d.masked_fill_(runs.repeat_interleave(512)[:n], 0)
    h = C.swap_out(d, n, dtype, codec)
    h.wait()
    blob = h.host_bytes()
    K = -(-n // F)
    hdr = _a16(64 + 8 * K)
    magic, ver, cod, dt, n_h, F_h, K_h, param, total = struct.unpack_from("<4sHBBQQIIQ", blob, 0)
    assert (magic, ver, cod, dt, n_h, F_h, K_h, total) == (b"CSWP", 1, codec, dtype, n, F, K, len(blob))
    fb = np.array(struct.unpack_from(f"<{K}Q", blob, 64), dtype=np.int64)
    assert hdr + int(fb.sum()) == len(blob) and all(int(b) % 16 == 0 for b in fb)
    starts = hdr + np.concatenate([[0], np.cumsum(fb)[:-1]])
    x = G.from_dev(d)[:n]
    ds = _a16(64 + 8)
    prm = {O.CSR: 1024, O.LZ4: 65536}.get(codec, 0)
    for k in sorted({0, 1, K // 2, K - 1}):
        ref = O.compress(x[k * F:(k + 1) * F], codec, dtype, F=F, param=prm)
        assert blob[starts[k]:starts[k] + fb[k]] == ref[ds:], f"frame {k}"
    out = G.poison_like(d)
    h.swap_in(out)
    h.wait()
    assert torch.equal(out, d)
    h.close()
