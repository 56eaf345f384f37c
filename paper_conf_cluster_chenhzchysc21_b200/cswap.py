"""ctypes binding of libcswap.so (include/cswap.h) — argument marshalling only.

Every function has the C name without the ``cswap_`` prefix; tensors may be passed as
``torch.Tensor`` (their ``data_ptr()`` is used) or as raw integer addresses, streams as
``torch.cuda.Stream`` or raw handles.  There is NO fallback: if the native library is missing
this module raises at import time.
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
# CSWAP_LIB_VARIANT=<tag> loads variants/libcswap_<tag>.so, an A/B build of the same sources with
# different compile-time switches (tools/build_variants.py); default: the in-tree libcswap.so
_VARIANT = os.environ.get("CSWAP_LIB_VARIANT") or None
LIB_PATH = (os.path.join(_HERE, "variants", f"libcswap_{_VARIANT}.so") if _VARIANT
            else os.path.join(_HERE, "libcswap.so"))
if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is missing: build it with `python -m paper_conf_cluster_chenhzchysc21_b200.build`"
                      " (there is no CPU fallback)")
_L = ctypes.CDLL(LIB_PATH)

NONE, ZVC, RLE, CSR, LZ4, AUTO = 0, 1, 2, 3, 4, 255
F32, F16, BF16 = 0, 1, 2
CODEC_NAMES = {NONE: "none", ZVC: "zvc", RLE: "rle", CSR: "csr", LZ4: "lz4"}
WIDTH = {F32: 4, F16: 2, BF16: 2}
STATUS = {0: "OK", 1: "INVALID", 2: "CUDA", 3: "NOMEM", 4: "CAPACITY", 5: "CORRUPT", 6: "UNSUPPORTED",
          7: "NOT_READY"}


class CswapError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        super().__init__(f"{where}: {STATUS.get(status, status)}: {_L.cswap_last_error().decode()}")


class Format(ctypes.Structure):
    _fields_ = [("frame_elems", ctypes.c_uint64), ("csr_row", ctypes.c_uint32), ("lz4_block", ctypes.c_uint32)]


class ProbeResult(ctypes.Structure):
    _fields_ = [(k, ctypes.c_uint64) for k in ("zeros", "zero_runs", "boundaries", "samples", "pairs")]

    def tuple(self):
        return (self.zeros, self.zero_runs, self.boundaries, self.samples, self.pairs)


class Calib(ctypes.Structure):
    _fields_ = [
        ("alpha_d2h", ctypes.c_double), ("bw_d2h", ctypes.c_double),
        ("alpha_h2d", ctypes.c_double), ("bw_h2d", ctypes.c_double),
        ("beta", ctypes.c_double * (4 * 2 * 6 * 3)),
        ("lz4_gamma1", ctypes.c_double), ("lz4_gamma2", ctypes.c_double),
        ("margin", ctypes.c_double),
        ("mode", ctypes.c_int32), ("reserved", ctypes.c_int32),
        ("frame_elems", ctypes.c_uint64),
        ("csr_row", ctypes.c_uint32), ("lz4_block", ctypes.c_uint32),
        ("group_bytes", ctypes.c_double),
    ]


class Decision(ctypes.Structure):
    _fields_ = [("codec", ctypes.c_int32), ("reserved", ctypes.c_int32),
                ("t_pred", ctypes.c_double), ("t_prime", ctypes.c_double),
                ("t_codec", ctypes.c_double * 4), ("size", ctypes.c_double * 4),
                ("t_c", ctypes.c_double * 4), ("t_dc", ctypes.c_double * 4)]

    def as_dict(self):
        return {"codec": self.codec, "t_pred": self.t_pred, "t_prime": self.t_prime,
                "t_codec": list(self.t_codec), "size": list(self.size), "t_c": list(self.t_c),
                "t_dc": list(self.t_dc)}


class KernelRecord(ctypes.Structure):
    _fields_ = [("codec", ctypes.c_int32), ("direction", ctypes.c_int32), ("raw_bytes", ctypes.c_uint64),
                ("comp_bytes", ctypes.c_uint64), ("ms", ctypes.c_double), ("device_ms", ctypes.c_double),
                ("kernel_ms", ctypes.c_double)]


_vp, _u64, _u32, _i, _d = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int, ctypes.c_double
_P = ctypes.POINTER
_SIGS = {
    "cswap_init": (_i, [_i]),
    "cswap_shutdown": (_i, []),
    "cswap_set_calibration": (_i, [_P(Calib)]),
    "cswap_get_calibration": (_i, [_P(Calib)]),
    "cswap_set_format": (_i, [_P(Format)]),
    "cswap_get_format": (_i, [_P(Format)]),
    "cswap_max_compressed_size": (_u64, [_u64, _i, _i, _P(Format)]),
    "cswap_compress": (_i, [_vp, _u64, _i, _i, _P(Format), _vp, _u64, _vp, _vp]),
    "cswap_decompress": (_i, [_vp, _u64, _vp, _u64, _i, _i, _P(Format), _vp, _vp]),
    "cswap_check_device_error": (_i, [_vp]),
    "cswap_probe": (_i, [_vp, _u64, _i, _P(ProbeResult), _vp]),
    "cswap_select_from_probe": (_i, [_u64, _i, _P(ProbeResult), _d, _d, _P(Calib), _P(Decision)]),
    "cswap_select": (_i, [_vp, _u64, _i, _d, _d, _vp, _P(Decision)]),
    "cswap_swap_out": (_i, [_vp, _u64, _i, _i, _d, _d, _vp, _P(_vp)]),
    "cswap_swap_in": (_i, [_vp, _vp, _vp]),
    "cswap_handle_wait": (_i, [_vp]),
    "cswap_handle_record_out": (_i, [_vp, _vp]),
    "cswap_handle_query": (_i, [_vp, _P(ctypes.c_int), _P(_u64), _P(_vp), _P(Decision)]),
    "cswap_handle_free": (None, [_vp]),
    "cswap_fit_time_model": (_i, [_P(_d), _P(_d), _P(_d), _u64, _P(_d)]),
    "cswap_fit_link": (_i, [_P(_d), _P(_d), _u64, _P(_d), _P(_d)]),
    "cswap_fit_linear": (_i, [_P(_d), _P(_d), _u64, _u32, _P(_d)]),
    "cswap_set_kernel_timing": (_i, [_i]),
    "cswap_collect_kernel_timing": (_u64, [_P(KernelRecord), _u64]),
    "cswap_status_string": (ctypes.c_char_p, [_i]),
    "cswap_last_error": (ctypes.c_char_p, []),
    "cswap_kernel_launches": (_u64, []),
    "cswap_graph_stats": (None, [_P(_u64), _P(_u64)]),
    "cswap_set_zvc_launch": (_i, [_u32, ctypes.c_int32]),
    "cswap_set_swap_target": (_i, [_i]),
    "cswap_get_swap_target": (_i, [_P(ctypes.c_int)]),
    "cswap_handle_copy_container": (_i, [_vp, _vp, _u64, _vp]),
    "cswap_release_cached": (_i, [_u64]),
}
for _name, (_res, _args) in _SIGS.items():
    _f = getattr(_L, _name)
    _f.restype = _res
    _f.argtypes = _args

EXPORTED = tuple(_SIGS)


def _ptr(x) -> int | None:
    if x is None:
        return None
    if isinstance(x, int):
        return x
    return x.data_ptr()


def _stream(s) -> int | None:
    if s is None:
        try:
            import torch
            if torch.cuda.is_available():
                return torch.cuda.current_stream().cuda_stream
        except Exception:  # pragma: no cover
            pass
        return None
    if isinstance(s, int):
        return s
    return s.cuda_stream


def _check(rc: int, where: str):
    if rc != 0:
        raise CswapError(rc, where)


def _fmt(fmt) -> ctypes.POINTER(Format) | None:
    if fmt is None:
        return None
    if isinstance(fmt, Format):
        return ctypes.pointer(fmt)
    f = Format(*fmt) if isinstance(fmt, (tuple, list)) else Format(**fmt)
    return ctypes.pointer(f)


# ---- lifecycle ------------------------------------------------------------------------------
def init(device: int = 0):
    _check(_L.cswap_init(device), "cswap_init")


def shutdown():
    _check(_L.cswap_shutdown(), "cswap_shutdown")


def set_calibration(c: Calib):
    _check(_L.cswap_set_calibration(ctypes.byref(c)), "cswap_set_calibration")


def get_calibration() -> Calib:
    c = Calib()
    _check(_L.cswap_get_calibration(ctypes.byref(c)), "cswap_get_calibration")
    return c


def set_format(frame_elems=1 << 22, csr_row=1024, lz4_block=65536):
    f = Format(frame_elems, csr_row, lz4_block)
    _check(_L.cswap_set_format(ctypes.byref(f)), "cswap_set_format")


def get_format() -> Format:
    f = Format()
    _check(_L.cswap_get_format(ctypes.byref(f)), "cswap_get_format")
    return f


# ---- codecs ---------------------------------------------------------------------------------
def max_compressed_size(n: int, dtype: int, codec: int, fmt=None) -> int:
    return int(_L.cswap_max_compressed_size(n, dtype, codec, _fmt(fmt)))


def compress(d_in, n: int, dtype: int, codec: int, out, out_cap: int, out_size, fmt=None, stream=None):
    _check(_L.cswap_compress(_ptr(d_in), n, dtype, codec, _fmt(fmt), _ptr(out), out_cap, _ptr(out_size),
                             _stream(stream)), "cswap_compress")


def decompress(src, in_size: int, d_out, n: int, dtype: int, codec: int, fmt=None, err=None, stream=None):
    _check(_L.cswap_decompress(_ptr(src), in_size, _ptr(d_out), n, dtype, codec, _fmt(fmt), _ptr(err),
                               _stream(stream)), "cswap_decompress")


def check_device_error(stream=None):
    _check(_L.cswap_check_device_error(_stream(stream)), "cswap_check_device_error")


def probe(d_in, n: int, dtype: int, stream=None) -> ProbeResult:
    r = ProbeResult()
    _check(_L.cswap_probe(_ptr(d_in), n, dtype, ctypes.byref(r), _stream(stream)), "cswap_probe")
    return r


def select_from_probe(n: int, dtype: int, probe_counts, hidden_f=0.0, hidden_b=0.0, calib: Calib | None = None
                      ) -> Decision:
    p = probe_counts if isinstance(probe_counts, ProbeResult) else ProbeResult(*probe_counts)
    d = Decision()
    _check(_L.cswap_select_from_probe(n, dtype, ctypes.byref(p), hidden_f, hidden_b,
                                      ctypes.byref(calib) if calib is not None else None, ctypes.byref(d)),
           "cswap_select_from_probe")
    return d


def select(d_in, n: int, dtype: int, hidden_f=0.0, hidden_b=0.0, stream=None) -> Decision:
    d = Decision()
    _check(_L.cswap_select(_ptr(d_in), n, dtype, hidden_f, hidden_b, _stream(stream), ctypes.byref(d)),
           "cswap_select")
    return d


# ---- swaps ----------------------------------------------------------------------------------
class Handle:
    """Owns a cswap_handle*; freed on close()/__del__."""

    def __init__(self, raw: int):
        self.raw = raw

    def swap_in(self, d_out, stream=None):
        _check(_L.cswap_swap_in(self.raw, _ptr(d_out), _stream(stream)), "cswap_swap_in")

    def wait(self):
        _check(_L.cswap_handle_wait(self.raw), "cswap_handle_wait")

    def record_out(self, stream=None):
        _check(_L.cswap_handle_record_out(self.raw, _stream(stream)), "cswap_handle_record_out")

    def codec(self) -> int:
        """The codec the swap-out used (known when cswap_swap_out returns; does not wait)."""
        c = ctypes.c_int()
        _check(_L.cswap_handle_query(self.raw, ctypes.byref(c), None, None, None), "cswap_handle_query")
        return c.value

    def query(self):
        """Codec, container bytes, host pointer and decision; waits until the swap-out's copies
        are issued (not for the device)."""
        codec = ctypes.c_int()
        nbytes = ctypes.c_uint64()
        host = ctypes.c_void_p()
        dec = Decision()
        _check(_L.cswap_handle_query(self.raw, ctypes.byref(codec), ctypes.byref(nbytes), ctypes.byref(host),
                                     ctypes.byref(dec)), "cswap_handle_query")
        return {"codec": codec.value, "bytes": nbytes.value, "host": host.value, "decision": dec}

    def copy_container(self, dst, cap: int, stream=None):
        """Copy the container (any swap target) into dst (host or device, >= cap bytes)."""
        _check(_L.cswap_handle_copy_container(self.raw, _ptr(dst), cap, _stream(stream)),
               "cswap_handle_copy_container")

    def container_bytes(self) -> bytes:
        """The container's bytes, read through cswap_handle_copy_container (any target)."""
        n = self.query()["bytes"]
        buf = ctypes.create_string_buffer(max(n, 1))
        if n:
            self.copy_container(ctypes.addressof(buf), n)
        return buf.raw[:n]

    def host_bytes(self) -> bytes:
        q = self.query()
        return ctypes.string_at(q["host"], q["bytes"]) if q["bytes"] else b""

    def close(self):
        if self.raw:
            _L.cswap_handle_free(self.raw)
            self.raw = 0

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def set_swap_target(device: int = -1):
    """-1 = pinned host memory (default); else a device (this one or a peer over NVLink)."""
    _check(_L.cswap_set_swap_target(device), "cswap_set_swap_target")


def release_cached(keep_bytes: int = 0):
    """Trim the staging pool to keep_bytes and unpin empty host chunks (like torch.cuda.empty_cache)."""
    _check(_L.cswap_release_cached(keep_bytes), "cswap_release_cached")


def get_swap_target() -> int:
    d = ctypes.c_int()
    _check(_L.cswap_get_swap_target(ctypes.byref(d)), "cswap_get_swap_target")
    return d.value


def swap_out(d_in, n: int, dtype: int, codec: int = AUTO, hidden_f=0.0, hidden_b=0.0, stream=None) -> Handle:
    h = ctypes.c_void_p()
    _check(_L.cswap_swap_out(_ptr(d_in), n, dtype, codec, hidden_f, hidden_b, _stream(stream), ctypes.byref(h)),
           "cswap_swap_out")
    return Handle(h.value)


# ---- calibration ----------------------------------------------------------------------------
def fit_time_model(S, s, t):
    m = len(t)
    A = (ctypes.c_double * m)
    beta = (ctypes.c_double * 3)()
    _check(_L.cswap_fit_time_model(A(*S), A(*s), A(*t), m, beta), "cswap_fit_time_model")
    return list(beta)


def fit_link(nbytes, t):
    m = len(t)
    A = (ctypes.c_double * m)
    a, bw = ctypes.c_double(), ctypes.c_double()
    _check(_L.cswap_fit_link(A(*nbytes), A(*t), m, ctypes.byref(a), ctypes.byref(bw)), "cswap_fit_link")
    return a.value, bw.value


def fit_linear(X, y):
    """OLS y = X beta; X is a list of rows (p <= 8 columns)."""
    m, p = len(X), len(X[0])
    flat = (ctypes.c_double * (m * p))(*[v for row in X for v in row])
    beta = (ctypes.c_double * p)()
    _check(_L.cswap_fit_linear(flat, (ctypes.c_double * m)(*y), m, p, beta), "cswap_fit_linear")
    return list(beta)


def set_kernel_timing(enable: bool):
    _check(_L.cswap_set_kernel_timing(1 if enable else 0), "cswap_set_kernel_timing")


def collect_kernel_timing(cap: int = 1 << 16):
    buf = (KernelRecord * cap)()
    k = int(_L.cswap_collect_kernel_timing(buf, cap))
    return [{"codec": r.codec, "direction": r.direction, "raw_bytes": r.raw_bytes, "comp_bytes": r.comp_bytes,
             "ms": r.ms, "device_ms": r.device_ms, "kernel_ms": r.kernel_ms} for r in buf[:k]]


def kernel_launches() -> int:
    return int(_L.cswap_kernel_launches())


def set_zvc_launch(grid: int = 0, variant: int = -1):
    """Persistent ZVC compress launch: grid CTAs (0 = auto) and stage/tile variant (-1 = default)."""
    _check(_L.cswap_set_zvc_launch(grid, variant), "cswap_set_zvc_launch")


def graph_stats() -> tuple[int, int]:
    """(graph launches, graph instantiations) since init."""
    a, b = _u64(0), _u64(0)
    _L.cswap_graph_stats(ctypes.byref(a), ctypes.byref(b))
    return int(a.value), int(b.value)


def status_string(s: int) -> str:
    return _L.cswap_status_string(s).decode()
