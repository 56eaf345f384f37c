"""Helpers for the -m gpu tests: move raw-word numpy arrays to the device and call the
product C ABI.  No method arithmetic here."""
import numpy as np

IMPLEMENTED = (0, 1, 2, 3, 4)  # codecs with CUDA kernels in this build (all)


def lib():
    import torch
    from paper_conf_cluster_chenhzchysc21_b200 import cswap
    cswap.init(0)
    torch.cuda.init()
    return cswap


def to_dev(x: np.ndarray):
    import torch
    if x.dtype == np.uint32:
        t = torch.from_numpy(x.view(np.int32).copy())
    else:
        t = torch.from_numpy(x.view(np.int16).copy())
    return t.cuda()


def from_dev(t) -> np.ndarray:
    a = t.cpu().numpy()
    return a.view(np.uint32) if a.dtype == np.int32 else a.view(np.uint16)


def empty_like_words(n, dtype):
    import torch
    return torch.empty(max(n, 1), dtype=torch.int32 if dtype == 0 else torch.int16, device="cuda")


def poisoned_words(n, dtype):
    """Output buffer filled with 0xA5 bytes: a decoder that skips writing any element (zeros
    included) leaves the poison there, whatever the allocator happened to return."""
    t = empty_like_words(n, dtype)
    t.fill_(-0x5A5A5A5B if dtype == 0 else -0x5A5B)  # 0xA5A5A5A5 / 0xA5A5
    return t


def poison_like(t):
    """0xA5-filled tensor with t's shape / dtype / device."""
    import torch
    out = torch.empty_like(t)
    out.view(torch.uint8).fill_(0xA5)
    return out


def gpu_compress(C, x: np.ndarray, codec: int, dtype: int, fmt=None, stream=None) -> bytes:
    import torch
    n = x.size
    d_in = to_dev(x) if n else empty_like_words(0, dtype)
    cap = C.max_compressed_size(n, dtype, codec, fmt)
    out = torch.full((cap,), 0xA5, dtype=torch.uint8, device="cuda")  # poison: padding must be written
    size = torch.zeros(1, dtype=torch.int64, device="cuda")
    C.compress(d_in, n, dtype, codec, out, cap, size, fmt=fmt, stream=stream)
    torch.cuda.synchronize()
    return out[: int(size.item())].cpu().numpy().tobytes()


def gpu_decompress(C, blob: bytes, n: int, dtype: int, codec: int, fmt=None):
    """Returns (words, err)."""
    import torch
    src = torch.from_numpy(np.frombuffer(blob, dtype=np.uint8).copy()).cuda()
    out = poisoned_words(n, dtype)
    err = torch.zeros(1, dtype=torch.int32, device="cuda")
    C.decompress(src, len(blob), out, n, dtype, codec, fmt=fmt, err=err)
    torch.cuda.synchronize()
    return from_dev(out)[:n], int(err.item())
