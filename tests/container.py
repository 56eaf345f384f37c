"""Test-side parser of canonical container v1.  Independent of the oracle
and of the CUDA path: it is written from the format table and used to cut a container
into its sections so tests can compare each section with numpy/scipy/liblz4."""
import struct

import numpy as np

W = {0: 4, 1: 2, 2: 2}


def a16(x):
    return (x + 15) // 16 * 16


def header(buf: bytes) -> dict:
    assert buf[:4] == b"CSWP"
    version, codec, dtype = struct.unpack_from("<HBB", buf, 4)
    n, F, K, param, total = struct.unpack_from("<QQIIQ", buf, 8)
    fb = list(struct.unpack_from(f"<{K}Q", buf, 64)) if K else []
    return dict(version=version, codec=codec, dtype=dtype, n=n, F=F, K=K, param=param, total=total,
                frame_bytes=fb, data_start=a16(64 + 8 * K))


def frames(buf: bytes):
    """Yield (k, Fk, payload bytes) for each frame."""
    h = header(buf)
    pos = h["data_start"]
    for k in range(h["K"]):
        Fk = min(h["F"], h["n"] - k * h["F"])
        yield k, Fk, buf[pos:pos + h["frame_bytes"][k]]
        pos += h["frame_bytes"][k]


def word_dtype(dtype):
    return np.uint32 if W[dtype] == 4 else np.uint16


def zvc_sections(payload: bytes, Fk: int, dtype: int):
    nw = (Fk + 31) // 32
    bm = np.frombuffer(payload[:4 * nw], dtype="<u4")
    nnz = int(sum(bin(int(v)).count("1") for v in bm))
    v0 = a16(4 * nw)
    vals = np.frombuffer(payload[v0:v0 + W[dtype] * nnz], dtype=word_dtype(dtype))
    return bm, vals


def rle_sections(payload: bytes, dtype: int):
    r = struct.unpack_from("<I", payload, 0)[0]
    lengths = np.frombuffer(payload[16:16 + 4 * r], dtype="<u4")
    v0 = 16 + a16(4 * r)
    vals = np.frombuffer(payload[v0:v0 + W[dtype] * r], dtype=word_dtype(dtype))
    return r, lengths, vals, payload[v0 + W[dtype] * r:]


def csr_sections(payload: bytes, Fk: int, C: int, dtype: int):
    R = (Fk + C - 1) // C
    row_ptr = np.frombuffer(payload[:4 * (R + 1)], dtype="<u4")
    nnz = int(row_ptr[-1])
    c0 = a16(4 * (R + 1))
    col = np.frombuffer(payload[c0:c0 + 4 * nnz], dtype="<u4")
    v0 = c0 + a16(4 * nnz)
    vals = np.frombuffer(payload[v0:v0 + W[dtype] * nnz], dtype=word_dtype(dtype))
    return row_ptr, col, vals


def lz4_blocks(payload: bytes, Fk: int, B: int, dtype: int):
    nbytes = Fk * W[dtype]
    nblk = (nbytes + B - 1) // B
    cs = struct.unpack_from(f"<{nblk}I", payload, 0) if nblk else ()
    pos = a16(4 * nblk)
    out = []
    for b in range(nblk):
        L = min(B, nbytes - b * B)
        out.append((L, payload[pos:pos + cs[b]]))
        pos += cs[b]
    return out, payload[pos:]
