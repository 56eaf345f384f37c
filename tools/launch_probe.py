"""Per-boundary cost of a kernel chain (device %globaltimer stamps) alone, during a D2H copy and
during an H2D copy, launched plainly vs from an uploaded CUDA graph (tools/launch_probe.cu)."""
import ctypes
import os
import statistics

import torch

L = ctypes.CDLL(os.path.join(os.path.dirname(os.path.abspath(__file__)), 'launch_probe.so'))
for f in (L.chain_plain, L.chain_graph_build):
    f.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_int, ctypes.c_void_p]
L.chain_graph_launch.argtypes = [ctypes.c_void_p]
L.chain_graph2_build.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_int, ctypes.c_void_p]
L.chain_graph2_launch.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_void_p]
import time

NB = 1 << 30
host = torch.empty(NB, dtype=torch.uint8).pin_memory()
dev = torch.empty(NB, dtype=torch.uint8, device='cuda')
side = torch.cuda.Stream()
st = torch.cuda.Stream()
N = 40
t = torch.zeros(N, dtype=torch.int64, device='cuda')


def spacing():
    v = t.cpu().tolist()
    d = [(v[i + 1] - v[i]) / 1e3 for i in range(N - 1)]
    return round(statistics.median(d), 2), round(max(d), 1)


def run(mode, copy, blocks):
    res = []
    for _ in range(5):
        torch.cuda.synchronize()
        if copy == 'd2h':
            with torch.cuda.stream(side):
                host.copy_(dev, non_blocking=True)
        elif copy == 'h2d':
            with torch.cuda.stream(side):
                dev.copy_(host, non_blocking=True)
        with torch.cuda.stream(st):
            torch.cuda._sleep(100000)  # let the copy reach steady state
            if mode == 'plain':
                L.chain_plain(t.data_ptr(), N, blocks, st.cuda_stream)
            elif mode == 'graph':
                L.chain_graph_launch(st.cuda_stream)
            else:
                h0 = time.perf_counter()
                r = L.chain_graph2_launch(t.data_ptr(), {'setp': 0, 'inst+up': 1, 'inst': 2}[mode], st.cuda_stream)
                host_us.append((time.perf_counter() - h0) * 1e6)
                assert r == 0, r
        torch.cuda.synchronize()
        res.append(spacing())
    res.sort()
    return res[len(res) // 2]


host_us = []
for blocks in (1, 296):
    L.chain_graph_build(t.data_ptr(), N, blocks, st.cuda_stream)
    L.chain_graph2_build(t.data_ptr(), N, blocks, st.cuda_stream)
    torch.cuda.synchronize()
    for copy in ('none', 'd2h', 'h2d'):
        row = {m: run(m, copy, blocks) for m in ('plain', 'graph', 'setp', 'inst+up', 'inst')}
        print(f'blocks={blocks:4d} copy={copy:4s} us/boundary (median, max): {row}', flush=True)
print('host us per graph2 launch call (40 nodes) median', sorted(host_us)[len(host_us) // 2])
