"""GPU parity: the CUDA codecs (through the C ABI) against the CPU oracle, byte for byte,
on seeded synthetic inputs, plus round trips and corrupt-input handling."""
import numpy as np
import pytest

import synth
from oracle import oracle as O
from tests import gpu_util as G

pytestmark = pytest.mark.gpu

CODECS = [c for c in (O.NONE, O.ZVC, O.RLE, O.CSR, O.LZ4) if c in G.IMPLEMENTED]
PARAM = {O.CSR: 1024, O.LZ4: 65536}


@pytest.fixture(scope="module")
def C():
    return G.lib()


def fmt_of(F, codec, C_row=1024, B=65536):
    return (F, C_row, B)


def check_parity(C, x, codec, dtype, F=1 << 22, C_row=1024, B=65536):
    param = {O.CSR: C_row, O.LZ4: B}.get(codec, 0)
    ref = O.compress(x, codec, dtype, F=F, param=param)
    got = G.gpu_compress(C, x, codec, dtype, fmt=(F, C_row, B))
    assert len(got) == len(ref), f"size {len(got)} != oracle {len(ref)}"
    if got != ref:
        a, b = np.frombuffer(got, np.uint8), np.frombuffer(ref, np.uint8)
        bad = np.flatnonzero(a != b)
        raise AssertionError(f"{len(bad)} bytes differ, first at {bad[:8]} (of {len(ref)})")
    y, err = G.gpu_decompress(C, ref, x.size, dtype, codec, fmt=(F, C_row, B))
    assert err == 0
    assert np.array_equal(y, x)


@pytest.mark.parametrize("codec", CODECS)
def test_config1_parity(C, codec):
    """BASELINE.json configs[0]: 2^20 fp32 ReLU tensor, exactly 50 % zeros."""
    x = synth.relu_iid(1 << 20, 0.5, seed=synth.seed_of(1), exact=True)
    check_parity(C, x, codec, O.F32)


@pytest.mark.parametrize("codec", CODECS)
@pytest.mark.parametrize("dtype", [O.F32, O.F16, O.BF16])
@pytest.mark.parametrize("n,F", [(1, 1024), (31, 1024), (1000, 1024), (8192, 1024), (8193, 1 << 13),
                                 (100003, 1 << 14), (250000, 1 << 20), (3 * 16384 + 7, 16384)])
def test_ragged_sizes_and_frames(C, codec, dtype, n, F):
    x = synth.relu_iid(n, 0.55, seed=n ^ F ^ dtype, dtype=dtype)
    check_parity(C, x, codec, dtype, F=F)


@pytest.mark.parametrize("codec", CODECS)
@pytest.mark.parametrize("kind", ["zero", "dense", "const", "clustered", "special", "sparse99"])
def test_structures(C, codec, kind):
    n = 200000
    if kind == "zero":
        x = np.zeros(n, np.uint32)
    elif kind == "dense":
        x = synth.relu_iid(n, 0.0, seed=1)
    elif kind == "const":
        x = synth.constant(n, 0x3F800000)
    elif kind == "clustered":
        x = synth.relu_clustered(n, 0.8, 256, seed=2)
    elif kind == "sparse99":
        x = synth.relu_iid(n, 0.99, seed=3)
    else:
        rng = np.random.default_rng(4)
        x = rng.choice(np.array([0, 0x80000000, 0x7FC00001, 1, 0xFFFFFFFF], np.uint32), size=n)
    check_parity(C, x, codec, O.F32, F=1 << 16)


@pytest.mark.parametrize("codec", CODECS)
def test_empty(C, codec):
    check_parity(C, np.zeros(0, np.uint32), codec, O.F32)


@pytest.mark.parametrize("codec", [c for c in CODECS if c != O.NONE])
def test_corrupt_containers_flag_error_without_fault(C, codec):
    import torch
    x = synth.relu_iid(50000, 0.5, seed=9)
    ref = bytearray(O.compress(x, codec, O.F32, F=16384, param=PARAM.get(codec, 0)))
    fmt = (16384, 1024, 65536)
    bad = bytearray(ref)
    bad[0] ^= 0xFF  # magic
    _, err = G.gpu_decompress(C, bytes(bad), 50000, O.F32, codec, fmt=fmt)
    assert err != 0
    rng = np.random.default_rng(0)
    for _ in range(40):  # random flips in frame tables / payloads: error or a valid decode, never a fault
        b = bytearray(ref)
        i = int(rng.integers(64, len(b)))
        b[i] ^= int(rng.integers(1, 256))
        G.gpu_decompress(C, bytes(b), 50000, O.F32, codec, fmt=fmt)
    torch.cuda.synchronize()
    y, err = G.gpu_decompress(C, bytes(ref), 50000, O.F32, codec, fmt=fmt)  # still healthy
    assert err == 0 and np.array_equal(y, x)


def test_probe_matches_oracle(C):
    for n, s in [(1, 0.0), (1000, 0.5), (1 << 18, 0.3), ((1 << 18) + 1, 0.6), (1 << 22, 0.45)]:
        for dtype in (O.F32, O.F16):
            x = synth.relu_clustered(n, max(s, 0.05), 17, seed=n, dtype=dtype)
            d = G.to_dev(x)
            got = C.probe(d, n, dtype).tuple()
            assert got == O.probe(x, dtype)
