"""Pins for the oracle codecs (CPU only).  Every check compares the oracle with something
other than itself: the paper's worked examples (tests/golden/), closed-form sizes,
numpy/scipy computations of the same sections, and decode round trips.
Citations: PAPER.md:220-224 (§IV-E)."""
import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

import synth
from oracle import oracle as O
from tests import container as CT
from tests.golden_io import read_pairs, words, ints

F1K = 1024


def f32(xs):
    return np.asarray(xs, dtype=np.uint32)


# ---------------------------------------------------------------- paper examples
def test_paper_zvc_example():
    g = read_pairs("paper_codec_examples.txt")
    x = words(g["zvc_A00B0C000.input"])
    c = O.compress(x, O.ZVC, O.F32, F=F1K)
    h = CT.header(c)
    assert (h["codec"], h["dtype"], h["n"], h["K"], h["version"]) == (O.ZVC, O.F32, 9, 1, 1)
    (_, Fk, p), = list(CT.frames(c))
    bm, vals = CT.zvc_sections(p, Fk, O.F32)
    assert list(bm) == ints(g["zvc_A00B0C000.bitmap"])
    assert np.array_equal(vals, words(g["zvc_A00B0C000.values"]))
    # container = 64 header + 8 frame table (-> 80) + 16 bitmap + 16 values
    assert len(c) == h["total"] == 80 + 16 + 16


def test_paper_rle_examples():
    g = read_pairs("paper_codec_examples.txt")
    for key in ("rle_A0000000", "rle_A00B0C000"):
        x = words(g[key + ".input"])
        c = O.compress(x, O.RLE, O.F32, F=F1K)
        (_, Fk, p), = list(CT.frames(c))
        r, lengths, vals, tail = CT.rle_sections(p, O.F32)
        assert list(lengths) == ints(g[key + ".lengths"])
        assert np.array_equal(vals, words(g[key + ".values"]))
        assert r == len(lengths)
        assert set(tail) <= {0}


def test_paper_csr_example():
    g = read_pairs("paper_codec_examples.txt")
    x = words(g["csr_A00B0C000.input"])
    c = O.compress(x, O.CSR, O.F32, F=F1K, param=1024)
    (_, Fk, p), = list(CT.frames(c))
    rp, col, vals = CT.csr_sections(p, Fk, 1024, O.F32)
    assert list(rp) == ints(g["csr_A00B0C000.row_ptr"])
    assert list(col) == ints(g["csr_A00B0C000.col_idx"])
    assert np.array_equal(vals, words(g["csr_A00B0C000.values"]))


# ---------------------------------------------------------------- closed forms
def test_config1_container_sizes():
    """Config 1 (BASELINE.json configs[0]): 2^20 fp32, exactly 524288 zeros.
    ZVC = n/8 + 4 nnz payload (BASELINE.json north_star; PAPER.md:222 bitmap = 1/32 of
    fp32 data, "memory overhead only 3%" PAPER.md:224); CSR = 4(R+1) + 8 nnz, i.e. ~50 %
    metadata at 50 % sparsity."""
    n = 1 << 20
    x = synth.relu_iid(n, 0.5, seed=1, exact=True)
    assert int((x == 0).sum()) == 524288
    z = O.compress(x, O.ZVC, O.F32)
    assert len(z) == 64 + 16 + 131072 + 2097152 == 2228304
    c = O.compress(x, O.CSR, O.F32)
    assert len(c) == 64 + 16 + 4112 + 2097152 + 2097152
    # metadata overhead relative to the raw tensor: ZVC 1/32 = 3.1 %, CSR index = 50 %
    assert 131072 / (4 * n) == pytest.approx(1 / 32)
    assert 2097152 / (4 * n) == pytest.approx(0.5)


@pytest.mark.parametrize("dtype", [O.F32, O.F16, O.BF16])
@pytest.mark.parametrize("n,F", [(1, 1024), (31, 1024), (1000, 1024), (4096, 1024), (5000, 2048), (70000, 1 << 14)])
def test_zvc_sections_match_numpy(n, F, dtype):
    x = synth.relu_iid(n, 0.6, seed=n + F + dtype, dtype=dtype)
    c = O.compress(x, O.ZVC, dtype, F=F)
    h = CT.header(c)
    assert h["K"] == -(-n // F)
    w = O.WIDTH[dtype]
    total = h["data_start"]
    for k, Fk, p in CT.frames(c):
        xf = x[k * F:k * F + Fk]
        bm, vals = CT.zvc_sections(p, Fk, dtype)
        bits = np.packbits(xf != 0, bitorder="little")
        bits = np.concatenate([bits, np.zeros((-len(bits)) % 4, np.uint8)]).view("<u4")
        assert np.array_equal(bm, bits)
        assert np.array_equal(vals, xf[np.flatnonzero(xf)])
        nnz = int(np.count_nonzero(xf))
        assert len(p) == CT.a16(4 * (-(-Fk // 32))) + CT.a16(w * nnz)
        total += len(p)
    assert total == len(c) == h["total"]


def test_zvc_closed_form_fp32():
    """Total ZVC payload for fp32 with 32 | n is n/8 + 4 nnz (before 16-byte padding)."""
    n = 32 * 777
    x = synth.relu_iid(n, 0.37, seed=5)
    c = O.compress(x, O.ZVC, O.F32, F=1 << 20)
    nnz = int(np.count_nonzero(x))
    assert len(c) == 64 + 16 + CT.a16(n // 8) + CT.a16(4 * nnz)


@pytest.mark.parametrize("dtype", [O.F32, O.F16])
def test_rle_runs_match_numpy(dtype):
    n, F = 9000, 2048
    x = synth.relu_clustered(n, 0.7, 12, seed=9, dtype=dtype)
    c = O.compress(x, O.RLE, dtype, F=F)
    for k, Fk, p in CT.frames(c):
        xf = x[k * F:k * F + Fk]
        starts = np.concatenate([[0], np.flatnonzero(np.diff(xf.astype(np.int64)) != 0) + 1])
        r, lengths, vals, _ = CT.rle_sections(p, dtype)
        assert r == 1 + np.count_nonzero(np.diff(xf.astype(np.int64)))
        assert np.array_equal(lengths, np.diff(np.concatenate([starts, [Fk]])))
        assert np.array_equal(vals, xf[starts])


def test_rle_all_zero_frame_is_one_run():
    x = np.zeros(3000, np.uint32)
    c = O.compress(x, O.RLE, O.F32, F=1024)
    for k, Fk, p in CT.frames(c):
        r, lengths, vals, _ = CT.rle_sections(p, O.F32)
        assert r == 1 and list(lengths) == [Fk] and list(vals) == [0]


def test_csr_matches_scipy():
    import scipy.sparse as sp
    C, F = 1024, 1 << 14
    n = 3 * F + 5 * C + 77  # ragged last frame and short last row
    x = synth.relu_iid(n, 0.8, seed=11)
    c = O.compress(x, O.CSR, O.F32, F=F, param=C)
    for k, Fk, p in CT.frames(c):
        xf = x[k * F:k * F + Fk]
        pad = np.zeros((-Fk) % C, np.uint32)
        m = sp.csr_matrix(np.concatenate([xf, pad]).view(np.float32).reshape(-1, C))
        rp, col, vals = CT.csr_sections(p, Fk, C, O.F32)
        assert np.array_equal(rp, m.indptr)
        assert np.array_equal(col, m.indices)
        assert np.array_equal(vals, m.data.view(np.uint32))


def test_none_is_raw():
    x = synth.relu_iid(5000, 0.5, seed=2)
    c = O.compress(x, O.NONE, O.F32, F=2048)
    got = b"".join(p[:Fk * 4] for _, Fk, p in CT.frames(c))
    assert got == x.tobytes()


def test_empty_tensor_is_header_only():
    for codec in range(5):
        c = O.compress(np.zeros(0, np.uint32), codec, O.F32)
        assert len(c) == 64
        h = CT.header(c)
        assert h["K"] == 0 and h["total"] == 64 and h["n"] == 0
        assert O.decompress(c, 0, O.F32).size == 0


# ---------------------------------------------------------------- round trips
SPECIAL_F32 = [0x80000000, 0x7FC00001, 0xFFFFFFFF, 0x00000001, 0x3F800000]  # -0.0, NaN payload, denormal


@st.composite
def tensors(draw):
    dtype = draw(st.sampled_from([O.F32, O.F16, O.BF16]))
    n = draw(st.integers(0, 5000))
    kind = draw(st.sampled_from(["iid", "clustered", "zero", "dense", "const", "special"]))
    seed = draw(st.integers(0, 2**31))
    s = draw(st.floats(0, 1))
    if kind == "iid":
        x = synth.relu_iid(n, s, seed, dtype)
    elif kind == "clustered":
        x = synth.relu_clustered(n, min(max(s, 0.05), 0.95), draw(st.integers(1, 64)), seed, dtype)
    elif kind == "zero":
        x = np.zeros(n, synth.WORD[dtype])
    elif kind == "dense":
        x = synth.relu_iid(n, 0.0, seed, dtype)
    elif kind == "const":
        x = synth.constant(n, 0x1234, dtype)
    else:
        rng = np.random.default_rng(seed)
        pool = SPECIAL_F32 + [0] if dtype == O.F32 else [0x8000, 0x7E01, 0xFFFF, 0x0001, 0]
        x = np.array(rng.choice(pool, size=n), dtype=synth.WORD[dtype])
    return dtype, x


@settings(max_examples=150, deadline=None)
@given(tensors(), st.sampled_from([O.NONE, O.ZVC, O.RLE, O.CSR, O.LZ4]), st.sampled_from([1024, 2048]))
def test_round_trip_property(t, codec, F):
    dtype, x = t
    param = {O.CSR: 256, O.LZ4: 1024}.get(codec, 0)
    c = O.compress(x, codec, dtype, F=F, param=param)
    assert len(c) % 16 == 0 and len(c) <= O.max_size(codec, dtype, len(x), F, param)
    y = O.decompress(c, len(x), dtype)
    assert np.array_equal(y, x)


def test_corrupt_inputs_are_rejected_not_crashing():
    x = synth.relu_iid(4096, 0.5, seed=3)
    rng = np.random.default_rng(0)
    for codec in (O.ZVC, O.RLE, O.CSR, O.LZ4):
        c = bytearray(O.compress(x, codec, O.F32, F=1024))
        assert O.decompress_rc(bytes(c[:-16]), 4096, O.F32) != 0  # truncated
        bad = bytearray(c)
        bad[0] ^= 1
        assert O.decompress_rc(bytes(bad), 4096, O.F32) != 0  # bad magic
        assert O.decompress_rc(bytes(c), 4095, O.F32) != 0  # n mismatch
        for _ in range(200):  # random byte flips: must return (ok or error), never fault
            b = bytearray(c)
            i = int(rng.integers(64, len(b)))
            b[i] ^= int(rng.integers(1, 256))
            O.decompress_rc(bytes(b), 4096, O.F32)
