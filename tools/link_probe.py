"""Host-link throughput by host allocation kind (cudaHostAlloc vs THP + cudaHostRegister),
buffer instance and copy size — explains the per-copy spread seen in tools/timeline_probe.py."""
import ctypes

import torch

cudart = torch.cuda.cudart()
NB = 512 << 20
dev = torch.empty(NB, dtype=torch.uint8, device='cuda')


def bw(host, nbytes, d2h=True, reps=5):
    out = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        if d2h:
            host[:nbytes].copy_(dev[:nbytes], non_blocking=True)
        else:
            dev[:nbytes].copy_(host[:nbytes], non_blocking=True)
        b.record()
        b.synchronize()
        out.append(a.elapsed_time(b))
    out.sort()
    return round(nbytes / out[len(out) // 2] / 1e6, 2)


libc = ctypes.CDLL('libc.so.6')
libc.madvise.argtypes = [ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int]
libc.posix_memalign.argtypes = [ctypes.POINTER(ctypes.c_void_p), ctypes.c_size_t, ctypes.c_size_t]


def thp_buffer(nb, advise=True):
    p = ctypes.c_void_p()
    libc.posix_memalign(ctypes.byref(p), 2 << 20, nb)
    if advise:
        libc.madvise(p, nb, 14)
    ctypes.memset(p, 0, nb)
    cudart.cudaHostRegister(p.value, nb, 0)
    return torch.frombuffer((ctypes.c_uint8 * nb).from_address(p.value), dtype=torch.uint8)


bufs = {f'hostalloc{i}': torch.empty(NB, dtype=torch.uint8).pin_memory() for i in range(3)}
bufs['thp0'] = thp_buffer(NB)
bufs['thp1'] = thp_buffer(NB)
bufs['reg4k'] = thp_buffer(NB, advise=False)
for name, h in bufs.items():
    row = []
    for mb in (6, 32, 128, 512):
        row.append((mb, bw(h, mb << 20, True), bw(h, mb << 20, False)))
    print(name, 'MiB: (d2h, h2d) GB/s', row)
# offsets inside one buffer: 16 MiB copies at different offsets
h = bufs['hostalloc0']
print('hostalloc0 16MiB d2h by offset', [bw(h[o << 20:], 16 << 20) for o in range(0, 496, 48)])
h = bufs['thp0']
print('thp0 16MiB d2h by offset', [bw(h[o << 20:], 16 << 20) for o in range(0, 496, 48)])
