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
                                 (100003, 1 << 14), (250000, 1 << 20), (3 * 16384 + 7, 16384),
                                 # tiles per frame not a power of two (the compress kernel's divide path)
                                 (300001, 5 * 8192), (200000, 3 * 1024 * 7)])
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


def _lz4_offset_case(gap: int, repeat: bool) -> np.ndarray:
    """3 LZ4 blocks of incompressible words; in each, a periodic run of period `gap` (gap < 96),
    or a random 96-byte pattern, zeros, and the pattern again `gap` bytes after the first copy
    (positions inside the zero run's match are not inserted, so the first copy stays
    in the hash table).  repeat=False replaces the second copy by other random bytes (control)."""
    rng = np.random.default_rng(gap)
    x = rng.integers(1, 2**32, size=3 * 16384, dtype=np.uint64).astype(np.uint32)
    raw = x.view(np.uint8)
    pat, other = rng.integers(0, 256, size=(2, 96), dtype=np.uint8)
    for blk in range(3):
        p0 = blk * 65536 + 1000
        if gap < 96:
            raw[p0:p0 + 256] = np.resize(pat[:gap], 256) if repeat else np.resize(other, 256)
        else:
            raw[p0:p0 + 96] = pat
            raw[p0 + 96:p0 + gap] = 0
            raw[p0 + gap:p0 + gap + 96] = pat if repeat else other
    return x


@pytest.mark.parametrize("gap", [3, 31, 32, 33, 4000, 4064, 4065, 4070, 4090, 4095, 4096, 4097, 10000, 60000])
def test_lz4_match_offsets(C, gap):
    """Every match-offset class of the LZ4 decoder: overlapping short offsets (< 32 bytes,
    pattern replication), offsets served by the warp's 4 KiB recent-output ring, and offsets
    beyond it (read back from global memory).  The GPU must produce the oracle's bytes and
    decode them; the oracle's container is smaller than the control's, i.e. the repeats at
    distance `gap` were parsed as matches."""
    x = _lz4_offset_case(gap, True)
    ref = O.compress(x, O.LZ4, O.F32, F=1 << 22, param=65536)
    ctl = O.compress(_lz4_offset_case(gap, False), O.LZ4, O.F32, F=1 << 22, param=65536)
    assert len(ref) + 3 * 50 < len(ctl)
    check_parity(C, x, O.LZ4, O.F32)


@pytest.mark.parametrize("dtype", [O.F32, O.F16])
@pytest.mark.parametrize("F,C_row", [(3072, 1), (3072, 3), (3072, 48), (3072, 1536), (3072, 3072),
                                     (1 << 16, 32), (1 << 16, 64), (1 << 20, 16384), (1 << 20, 65536),
                                     (1 << 20, 1 << 20)])
def test_csr_row_widths(C, dtype, F, C_row):
    """CSR with every kind of row width the header allows (C divides F): rows shorter than a
    32-element warp row (C = 1, 3), non-power-of-two C (48, 1536, 3072: general emit path),
    power-of-two C >= 32 (the emit's fast path), and rows longer than a 32 KiB tile (16384 …
    F: a tile ends mid-row, the frame end closes the last row)."""
    n = 2 * F + F // 3 + 5
    x = synth.relu_iid(n, 0.6, seed=F ^ C_row ^ dtype, dtype=dtype)
    check_parity(C, x, O.CSR, dtype, F=F, C_row=C_row)


@pytest.mark.parametrize("B", [1024, 4096, 16384, 65536])
@pytest.mark.parametrize("kind", ["iid", "clustered"])
def test_lz4_block_sizes(C, B, kind):
    """LZ4 with every block size class the header allows (multiple of 1024, <= 65536)."""
    n = 3 * 16384 + 123
    x = synth.relu_iid(n, 0.5, seed=B) if kind == "iid" else synth.relu_clustered(n, 0.8, 64, seed=B)
    check_parity(C, x, O.LZ4, O.F32, F=1 << 16, B=B)
