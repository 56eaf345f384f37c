"""Pins for the oracle's LZ4 block encoder/decoder against liblz4 1.9.4 (an independent
implementation present on this box and the GPU box) and against the paper's worked
example, PAPER.md:220-222 (§IV-E): "(abcde_bcde) can be compressed as (abcde_(5,4))"."""
import ctypes
import ctypes.util
import struct

import numpy as np
import pytest

import synth
from oracle import oracle as O
from tests import container as CT
from tests.golden_io import lz4_cases


def _liblz4():
    try:
        L = ctypes.CDLL("liblz4.so.1")
    except OSError:
        pytest.skip("liblz4.so.1 not available")
    L.LZ4_compress_default.argtypes = [ctypes.c_char_p, ctypes.c_char_p, ctypes.c_int, ctypes.c_int]
    L.LZ4_decompress_safe.argtypes = [ctypes.c_char_p, ctypes.c_char_p, ctypes.c_int, ctypes.c_int]
    L.LZ4_compressBound.argtypes = [ctypes.c_int]
    return L


def lz4_ref_compress(data: bytes) -> bytes:
    L = _liblz4()
    cap = L.LZ4_compressBound(len(data))
    dst = ctypes.create_string_buffer(cap)
    n = L.LZ4_compress_default(data, dst, len(data), cap)
    return dst.raw[:n]


def lz4_ref_decompress(comp: bytes, L_out: int) -> bytes:
    L = _liblz4()
    dst = ctypes.create_string_buffer(max(L_out, 1))
    n = L.LZ4_decompress_safe(comp, dst, len(comp), L_out)
    assert n == L_out, f"liblz4 rejected the block (rc={n})"
    return dst.raw[:n]


@pytest.mark.parametrize("name", sorted(lz4_cases()))
def test_golden_examples_byte_equal_oracle_and_liblz4(name):
    src, expected = lz4_cases()[name]
    assert O.lz4_block(src) == expected
    assert lz4_ref_compress(src) == expected
    assert lz4_ref_decompress(expected, len(src)) == src


def test_paper_match_is_offset5_len4():
    """The (5,4) of PAPER.md:222 appears as the first sequence's offset and match length."""
    src, enc = lz4_cases()["paper_abcde_bcde_padded"]
    token = enc[0]
    nlit = token >> 4
    assert enc[1:1 + nlit] == b"abcde_"
    offset = struct.unpack_from("<H", enc, 1 + nlit)[0]
    assert (offset, (token & 15) + 4) == (5, 4)


def _blocks_under_test():
    rng = np.random.default_rng(7)
    out = []
    for s in (0.0, 0.2, 0.5, 0.8, 0.95, 1.0):
        out.append(synth.relu_iid(16384, s, seed=int(s * 100)).tobytes())
        out.append(synth.relu_clustered(16384, max(s, 0.05) if s < 1 else 0.99, 64, seed=3).tobytes())
        out.append(synth.relu_iid(32768, s, seed=5, dtype=synth.F16).tobytes())
    out.append(bytes(65536))                                # all zero: longest match lengths
    out.append(rng.integers(0, 256, 65536, dtype=np.uint8).tobytes())  # incompressible: long literals
    out.append(bytes(rng.integers(0, 4, 65536, dtype=np.uint8)))        # small alphabet
    for L in (0, 1, 12, 13, 14, 15, 16, 17, 30, 300, 4099):
        out.append(bytes(rng.integers(0, 3, L, dtype=np.uint8)))
    return out


def test_every_oracle_block_decodes_with_liblz4():
    L = _liblz4()
    for blk in _blocks_under_test():
        enc = O.lz4_block(blk)
        assert len(enc) <= L.LZ4_compressBound(len(blk))
        assert lz4_ref_decompress(enc, len(blk)) == blk
        assert O.lz4_block_decode(enc, len(blk)) == blk


def test_oracle_decoder_decodes_liblz4_output():
    """Pins the decoder independently of the oracle's encoder."""
    for blk in _blocks_under_test():
        enc = lz4_ref_compress(blk)
        assert O.lz4_block_decode(enc, len(blk)) == blk


def test_ratio_close_to_liblz4():
    """Canonical parse is a simplification of liblz4's (no ip-2 insert, no skip); its size
    stays within a few percent on ReLU-like data (R6)."""
    tot_o = tot_r = 0
    for s in (0.2, 0.5, 0.8):
        blk = synth.relu_iid(16384, s, seed=1).tobytes()
        tot_o += len(O.lz4_block(blk))
        tot_r += len(lz4_ref_compress(blk))
    assert 0.9 < tot_o / tot_r < 1.15


def test_container_blocks_decode_with_liblz4():
    x = synth.relu_clustered(70000, 0.8, 100, seed=8)
    F, B = 1 << 14, 4096
    c = O.compress(x, O.LZ4, O.F32, F=F, param=B)
    raw = x.tobytes()
    for k, Fk, p in CT.frames(c):
        blocks, tail = CT.lz4_blocks(p, Fk, B, O.F32)
        got = b"".join(lz4_ref_decompress(enc, L) for L, enc in blocks)
        assert got == raw[k * F * 4:(k * F + Fk) * 4]
        assert set(tail) <= {0} and len(tail) < 16
