"""Does a concurrent PCIe copy slow the ZVC kernels?  Times compress / decompress of one tensor
alone, with a D2H / H2D copy running on a side stream from (a) cudaHostAlloc'd memory and
(b) 2 MiB-aligned THP memory registered with cudaHostRegister."""
import ctypes
import mmap
import sys

import torch

sys.path.insert(0, '.')
import synth  # noqa: E402
from paper_conf_cluster_chenhzchysc21_b200 import cswap as C  # noqa: E402

C.init(0)
side = torch.cuda.Stream()


def ev_time(fn, reps=7):
    out = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        b.synchronize()
        out.append(a.elapsed_time(b) * 1e3)
    out.sort()
    return round(out[len(out) // 2], 1)


NB = 1 << 30
host_pin = torch.empty(NB, dtype=torch.uint8).pin_memory()
dev_big = torch.empty(NB, dtype=torch.uint8, device='cuda')

# THP host buffer registered with the driver
libc = ctypes.CDLL('libc.so.6')
libc.madvise.argtypes = [ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int]
libc.posix_memalign.argtypes = [ctypes.POINTER(ctypes.c_void_p), ctypes.c_size_t, ctypes.c_size_t]
p = ctypes.c_void_p()
libc.posix_memalign(ctypes.byref(p), 2 << 20, NB)
print('madvise', libc.madvise(p, NB, 14))  # MADV_HUGEPAGE
ctypes.memset(p, 1, NB)
thp = torch.frombuffer((ctypes.c_uint8 * NB).from_address(p.value), dtype=torch.uint8)
r = torch.cuda.cudart().cudaHostRegister(p.value, NB, 0)
print('register', r)
try:
    print(open('/sys/kernel/mm/transparent_hugepage/enabled').read().strip())
    print([l for l in open('/proc/meminfo') if 'AnonHuge' in l or 'HugePages_T' in l])
except OSError:
    pass

for mib in (24.5, 98, 392):
    n = int(mib * (1 << 18))
    x = synth.relu_iid_torch(n, 0.5, seed=1, dtype=0, device='cuda')
    y = torch.empty_like(x)
    cap = C.max_compressed_size(n, 0, C.ZVC)
    buf = torch.empty(cap, dtype=torch.uint8, device='cuda')
    sz = torch.zeros(1, dtype=torch.int64, device='cuda')
    err = torch.zeros(1, dtype=torch.int32, device='cuda')
    comp = lambda: C.compress(x, n, 0, C.ZVC, buf, cap, sz)  # noqa: E731
    comp()
    torch.cuda.synchronize()
    nb = int(sz.item())
    dec = lambda: C.decompress(buf, nb, y, n, 0, C.ZVC, err=err)  # noqa: E731
    def slept(fn):
        def g():
            torch.cuda._sleep(20000)
            fn()
        return g
    res = {'alone': (ev_time(slept(comp)), ev_time(slept(dec)))}
    for name, src in (('pinned', host_pin), ('thp', thp)):
        for dirn in ('d2h', 'h2d'):
            def with_copy(fn):
                def g():
                    with torch.cuda.stream(side):
                        if dirn == 'd2h':
                            src.copy_(dev_big, non_blocking=True)
                        else:
                            dev_big.copy_(src, non_blocking=True)
                    torch.cuda._sleep(20000)
                    fn()
                return g
            res[f'{name}_{dirn}'] = (ev_time(with_copy(comp)) , ev_time(with_copy(dec)))
            torch.cuda.synchronize()
    # device-to-device copy engine traffic for comparison
    d2 = torch.empty(NB, dtype=torch.uint8, device='cuda')
    def with_d2d(fn):
        def g():
            with torch.cuda.stream(side):
                d2.copy_(dev_big, non_blocking=True)
            torch.cuda._sleep(20000)
            fn()
        return g
    res['d2d'] = (ev_time(with_d2d(comp)), ev_time(with_d2d(dec)))
    torch.cuda.synchronize()
    print(mib, 'MiB  (compress us, decompress us, sleep ~10us incl. when copying):', res)
    del d2
