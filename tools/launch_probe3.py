"""Elapsed time of CUDA events around a plain 4-kernel chain vs the same chain as a graph,
alone and during a D2H copy (tools/launch_probe.cu)."""
import ctypes
import os
import statistics

import torch

L = ctypes.CDLL(os.path.join(os.path.dirname(os.path.abspath(__file__)), 'launch_probe.so'))
L.chain_plain.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_int, ctypes.c_void_p]
L.chain_graph_build.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_int, ctypes.c_void_p]
L.chain_graph_launch.argtypes = [ctypes.c_void_p]
L.chain_graph3_build.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p,
                                 ctypes.c_void_p]
L.chain_graph3_launch.argtypes = [ctypes.c_void_p]
host = torch.empty(1 << 30, dtype=torch.uint8).pin_memory()
dev = torch.empty(1 << 30, dtype=torch.uint8, device='cuda')
side, st = torch.cuda.Stream(), torch.cuda.Stream()
N = 4
t = torch.zeros(N, dtype=torch.int64, device='cuda')
ea, eb = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
# (timing events cannot be recorded inside a capture: cudaEventRecordWithFlags(External) on a
# timing event fails with cudaErrorStreamCaptureUnsupported, so the events stay outside)
print('build plain-graph', L.chain_graph_build(t.data_ptr(), N, 296, st.cuda_stream))
torch.cuda.synchronize()


def run(mode, copy):
    res = []
    for _ in range(7):
        torch.cuda.synchronize()
        if copy:
            with torch.cuda.stream(side):
                host.copy_(dev, non_blocking=True)
        with torch.cuda.stream(st):
            torch.cuda._sleep(100000)
            if mode == 'plain':
                ea.record(st); L.chain_plain(t.data_ptr(), N, 296, st.cuda_stream); eb.record(st)
            elif mode == 'graph_ev_outside':
                ea.record(st); L.chain_graph_launch(st.cuda_stream); eb.record(st)
            else:
                L.chain_graph3_launch(st.cuda_stream)
        torch.cuda.synchronize()
        v = t.cpu().tolist()
        res.append((ea.elapsed_time(eb) * 1e3, (v[-1] - v[0]) / 1e3))
    return round(statistics.median(r[0] for r in res), 2), round(statistics.median(r[1] for r in res), 2)


for copy in (False, True):
    for mode in ('plain', 'graph_ev_outside'):
        print(f'copy={"d2h" if copy else "none"} {mode:18s} (event us, first->last stamp us) {run(mode, copy)}', flush=True)
