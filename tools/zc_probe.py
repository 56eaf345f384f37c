"""SM-driven (zero-copy) vs copy-engine transfers: throughput by CTA count, and the slowdown
each inflicts on a concurrent ZVC compress (see tools/zc_probe.cu)."""
import ctypes
import os
import sys

import torch

sys.path.insert(0, '.')
import synth  # noqa: E402
from paper_conf_cluster_chenhzchysc21_b200 import cswap as C  # noqa: E402

so = os.path.join(os.path.dirname(os.path.abspath(__file__)), 'zc_probe.so')
L = ctypes.CDLL(so)
L.zc_d2h.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int, ctypes.c_void_p]
L.zc_h2d.argtypes = L.zc_d2h.argtypes
C.init(0)
NB = 512 << 20
cudart = torch.cuda.cudart()
# mapped pinned host memory (cudaHostAllocMapped = 2 | portable 1)
hp = ctypes.c_void_p()
lib = ctypes.CDLL('libcudart.so.12') if os.path.exists('/usr/local/cuda/lib64/libcudart.so.12') else None
host_t = torch.empty(NB, dtype=torch.uint8).pin_memory()  # torch pins with cudaHostAlloc (mapped on UVA)
dev = torch.empty(NB, dtype=torch.uint8, device='cuda')
side = torch.cuda.Stream()


def ev(fn, reps=5, stream=None):
    st = stream or torch.cuda.current_stream()
    out = []
    for _ in range(reps):
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(st)
        fn()
        b.record(st)
        b.synchronize()
        out.append(a.elapsed_time(b))
    out.sort()
    return out[len(out) // 2]


cs = torch.cuda.current_stream().cuda_stream
print('CE d2h GB/s', round(NB / ev(lambda: host_t.copy_(dev, non_blocking=True)) / 1e6, 2),
      'CE h2d GB/s', round(NB / ev(lambda: dev.copy_(host_t, non_blocking=True)) / 1e6, 2))
for ctas in (4, 8, 16, 32, 64, 148, 296):
    d = ev(lambda: L.zc_d2h(dev.data_ptr(), host_t.data_ptr(), NB, ctas, cs))
    h = ev(lambda: L.zc_h2d(host_t.data_ptr(), dev.data_ptr(), NB, ctas, cs))
    print(f'SM copy ctas={ctas}: d2h {NB / d / 1e6:.2f} GB/s  h2d {NB / h / 1e6:.2f} GB/s')

# interference on compress of a 24.5 MiB and a 98 MiB tensor
for mib in (24.5, 98):
    n = int(mib * (1 << 18))
    x = synth.relu_iid_torch(n, 0.5, seed=1, dtype=0, device='cuda')
    cap = C.max_compressed_size(n, 0, C.ZVC)
    buf = torch.empty(cap, dtype=torch.uint8, device='cuda')
    sz = torch.zeros(1, dtype=torch.int64, device='cuda')
    comp = lambda: C.compress(x, n, 0, C.ZVC, buf, cap, sz)  # noqa: E731
    comp()

    def run(bg):
        def f():
            if bg:
                with torch.cuda.stream(side):
                    bg()
            torch.cuda._sleep(20000)
            comp()
        return f
    res = {'alone': ev(run(None)), 'ce_d2h': ev(run(lambda: host_t.copy_(dev, non_blocking=True))),
           'ce_h2d': ev(run(lambda: dev.copy_(host_t, non_blocking=True)))}
    for ctas in (8, 16, 32):
        res[f'sm_d2h_{ctas}'] = ev(run(lambda: L.zc_d2h(dev.data_ptr(), host_t.data_ptr(), NB, ctas, side.cuda_stream)))
        res[f'sm_h2d_{ctas}'] = ev(run(lambda: L.zc_h2d(host_t.data_ptr(), dev.data_ptr(), NB, ctas, side.cuda_stream)))
    print(mib, 'MiB compress us (incl ~10us sleep):', {k: round(v * 1e3, 1) for k, v in res.items()})
