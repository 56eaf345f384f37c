"""Thin ctypes driver for the plain-C CPU oracle (oracle/cswap_oracle.c).

TEST INFRASTRUCTURE ONLY: only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / ``--impl reference`` legs may import this module.  The product package
never imports it.  This file only marshals arguments; every step of the arithmetic is
in cswap_oracle.c, which cites the PAPER.md passage it follows.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "cswap_oracle.c")
LIB = os.path.join(HERE, "liboracle.so")

NONE, ZVC, RLE, CSR, LZ4 = 0, 1, 2, 3, 4
F32, F16, BF16 = 0, 1, 2
WIDTH = {F32: 4, F16: 2, BF16: 2}
DEFAULT_F = 1 << 22
DEFAULT_C = 1024
DEFAULT_B = 65536


def build(force: bool = False) -> str:
    """Compile the oracle with plain gcc -O2 (scalar C, no SIMD intrinsics)."""
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(SRC):
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-Wall", "-Wextra", "-fPIC", "-shared",
                               "-o", LIB, SRC, "-lm"])
    return LIB


class Calib(ctypes.Structure):
    _fields_ = [
        ("alpha_d2h", ctypes.c_double), ("bw_d2h", ctypes.c_double),
        ("alpha_h2d", ctypes.c_double), ("bw_h2d", ctypes.c_double),
        ("beta", ctypes.c_double * (4 * 2 * 6 * 3)),
        ("lz4_gamma1", ctypes.c_double), ("lz4_gamma2", ctypes.c_double),
        ("margin", ctypes.c_double),
        ("mode", ctypes.c_int32), ("pad_", ctypes.c_int32),
        ("frame_elems", ctypes.c_uint64),
        ("csr_row", ctypes.c_uint32), ("lz4_block", ctypes.c_uint32),
        ("group_bytes", ctypes.c_double),
    ]


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(LIB)
        L.orc_compress.restype = ctypes.c_int64
        L.orc_compress.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_uint64,
                                   ctypes.c_uint64, ctypes.c_uint32, ctypes.c_void_p, ctypes.c_uint64]
        L.orc_decompress.restype = ctypes.c_int
        L.orc_decompress.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_void_p, ctypes.c_uint64,
                                     ctypes.c_int]
        L.orc_max_size.restype = ctypes.c_uint64
        L.orc_max_size.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_uint64, ctypes.c_uint64,
                                   ctypes.c_uint32]
        L.orc_lz4_block.restype = ctypes.c_int64
        L.orc_lz4_block.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_void_p]
        L.orc_lz4_block_decode.restype = ctypes.c_int64
        L.orc_lz4_block_decode.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_void_p,
                                           ctypes.c_uint64]
        L.orc_probe.restype = None
        L.orc_probe.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int,
                                ctypes.POINTER(ctypes.c_uint64)]
        L.orc_probe_estimates.restype = None
        L.orc_probe_estimates.argtypes = [ctypes.c_uint64, ctypes.POINTER(ctypes.c_uint64),
                                          ctypes.POINTER(ctypes.c_uint64)]
        L.orc_select.restype = ctypes.c_int
        L.orc_select.argtypes = [ctypes.c_uint64, ctypes.c_int, ctypes.POINTER(ctypes.c_uint64),
                                 ctypes.c_double, ctypes.c_double, ctypes.POINTER(Calib),
                                 ctypes.POINTER(ctypes.c_double)]
        L.orc_rae.restype = ctypes.c_double
        L.orc_rae.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64]
        _lib = L
    return _lib


def _buf(a: np.ndarray) -> ctypes.c_void_p:
    return ctypes.c_void_p(a.ctypes.data)


def default_param(codec: int) -> int:
    return DEFAULT_C if codec == CSR else DEFAULT_B if codec == LZ4 else 0


def max_size(codec: int, dtype: int, n: int, F: int = DEFAULT_F, param: int | None = None) -> int:
    p = default_param(codec) if param is None else param
    return int(lib().orc_max_size(codec, dtype, n, F, p))


def compress(x: np.ndarray, codec: int, dtype: int, F: int = DEFAULT_F, param: int | None = None) -> bytes:
    """x: contiguous array of raw words (uint32 for f32, uint16 for f16/bf16) or bytes view."""
    p = default_param(codec) if param is None else param
    x = np.ascontiguousarray(x)
    w = WIDTH[dtype]
    n = x.nbytes // w
    cap = max_size(codec, dtype, n, F, p)
    out = np.zeros(max(cap, 64), dtype=np.uint8)
    rc = lib().orc_compress(codec, dtype, _buf(x), n, F, p, _buf(out), out.nbytes)
    if rc < 0:
        raise ValueError(f"orc_compress failed rc={rc}")
    return out[:rc].tobytes()


def decompress(c: bytes, n: int, dtype: int) -> np.ndarray:
    """Returns raw words (uint32 for f32, uint16 otherwise).  Raises on corrupt input."""
    src = np.frombuffer(c, dtype=np.uint8).copy() if len(c) else np.zeros(1, np.uint8)
    out = np.zeros(n, dtype=np.uint32 if WIDTH[dtype] == 4 else np.uint16)
    rc = lib().orc_decompress(_buf(src), len(c), _buf(out) if n else None, n, dtype)
    if rc != 0:
        raise ValueError(f"orc_decompress failed rc={rc}")
    return out


def decompress_rc(c: bytes, n: int, dtype: int) -> int:
    src = np.frombuffer(c, dtype=np.uint8).copy() if len(c) else np.zeros(1, np.uint8)
    out = np.zeros(max(n, 1), dtype=np.uint32 if WIDTH[dtype] == 4 else np.uint16)
    return int(lib().orc_decompress(_buf(src), len(c), _buf(out), n, dtype))


def lz4_block(data: bytes) -> bytes:
    src = np.frombuffer(data, dtype=np.uint8).copy() if data else np.zeros(1, np.uint8)
    out = np.zeros(len(data) + len(data) // 255 + 16, dtype=np.uint8)
    rc = lib().orc_lz4_block(_buf(src), len(data), _buf(out))
    return out[:rc].tobytes()


def lz4_block_decode(data: bytes, out_cap: int) -> bytes:
    src = np.frombuffer(data, dtype=np.uint8).copy() if data else np.zeros(1, np.uint8)
    out = np.zeros(max(out_cap, 1), dtype=np.uint8)
    rc = lib().orc_lz4_block_decode(_buf(src), len(data), _buf(out), out_cap)
    if rc < 0:
        raise ValueError("corrupt lz4 block")
    return out[:rc].tobytes()


def probe(x: np.ndarray, dtype: int) -> tuple:
    x = np.ascontiguousarray(x)
    n = x.nbytes // WIDTH[dtype]
    c = (ctypes.c_uint64 * 5)()
    lib().orc_probe(_buf(x) if n else None, n, dtype, c)
    return tuple(int(v) for v in c)


def probe_estimates(n: int, counts) -> tuple:
    c = (ctypes.c_uint64 * 5)(*counts)
    e = (ctypes.c_uint64 * 4)()
    lib().orc_probe_estimates(n, c, e)
    return tuple(int(v) for v in e)


def make_calib(alpha_d2h=0.0, bw_d2h=50e9, alpha_h2d=0.0, bw_h2d=50e9, beta=None, lz4_gamma1=3.0,
               lz4_gamma2=1.0, margin=0.05, mode=0, frame_elems=DEFAULT_F, csr_row=DEFAULT_C,
               lz4_block=DEFAULT_B, group_bytes=float(32 << 20)) -> Calib:
    """beta: array-like [4 codecs][2 dirs][6 bands][3] (defaults to zeros)."""
    c = Calib()
    c.alpha_d2h, c.bw_d2h, c.alpha_h2d, c.bw_h2d = alpha_d2h, bw_d2h, alpha_h2d, bw_h2d
    b = np.zeros((4, 2, 6, 3)) if beta is None else np.asarray(beta, dtype=np.float64).reshape(4, 2, 6, 3)
    for i, v in enumerate(b.ravel()):
        c.beta[i] = float(v)
    c.lz4_gamma1, c.lz4_gamma2, c.margin, c.mode = lz4_gamma1, lz4_gamma2, margin, mode
    c.frame_elems, c.csr_row, c.lz4_block = frame_elems, csr_row, lz4_block
    c.group_bytes = group_bytes
    return c


def select(n: int, dtype: int, counts, hidden_f: float, hidden_b: float, calib: Calib) -> dict:
    c = (ctypes.c_uint64 * 5)(*counts)
    out = (ctypes.c_double * 19)()
    rc = lib().orc_select(n, dtype, c, hidden_f, hidden_b, ctypes.byref(calib), out)
    if rc != 0:
        raise ValueError("orc_select failed")
    o = list(out)
    return {"codec": int(o[0]), "t_pred": o[1], "t_prime": o[2], "t_codec": o[3:7],
            "size": o[7:11], "t_c": o[11:15], "t_dc": o[15:19]}


def rae(yhat, y) -> float:
    yh = np.ascontiguousarray(yhat, dtype=np.float64)
    yy = np.ascontiguousarray(y, dtype=np.float64)
    return float(lib().orc_rae(_buf(yh), _buf(yy), len(yy)))


def lstsq_fit(S, s, t) -> np.ndarray:
    """Time model of PAPER.md:164-168 (§IV-C): t = b0 + b1*S + b2*S*s fitted by ordinary
    least squares (numpy.linalg.lstsq is the library primitive for the fit step)."""
    S = np.asarray(S, dtype=np.float64)
    s = np.asarray(s, dtype=np.float64)
    X = np.stack([np.ones_like(S), S, S * s], axis=1)
    beta, *_ = np.linalg.lstsq(X, np.asarray(t, dtype=np.float64), rcond=None)
    return beta
