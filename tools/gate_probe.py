"""Event time of a tiny kernel and of a ZVC compress while a D2H copy runs, with and without a
host gate that holds the stream until the launch group is fully enqueued (tools/gate_probe.cu)."""
import ctypes
import os
import sys

import torch

sys.path.insert(0, '.')
import synth  # noqa: E402
from paper_conf_cluster_chenhzchysc21_b200 import cswap as C  # noqa: E402

L = ctypes.CDLL(os.path.join(os.path.dirname(os.path.abspath(__file__)), 'gate_probe.so'))
L.gate_close.argtypes = [ctypes.c_void_p, ctypes.c_uint32]
L.gate_open.argtypes = [ctypes.c_uint32]
L.tiny.argtypes = [ctypes.c_void_p, ctypes.c_void_p]
print('gate_init', L.gate_init())
C.init(0)
NB = 1 << 30
host = torch.empty(NB, dtype=torch.uint8).pin_memory()
dev = torch.empty(NB, dtype=torch.uint8, device='cuda')
side = torch.cuda.Stream()
st = torch.cuda.current_stream()
cnt = torch.zeros(1, dtype=torch.int32, device='cuda')
seq = [0]
n = int(24.5 * (1 << 18))
x = synth.relu_iid_torch(n, 0.5, seed=1, dtype=0, device='cuda')
cap = C.max_compressed_size(n, 0, C.ZVC)
buf = torch.empty(cap, dtype=torch.uint8, device='cuda')
sz = torch.zeros(1, dtype=torch.int64, device='cuda')


def run(fn, copy, gate, reps=9):
    out = []
    for _ in range(reps):
        torch.cuda.synchronize()
        if copy:
            with torch.cuda.stream(side):
                host.copy_(dev, non_blocking=True)
            torch.cuda._sleep(200000)
            torch.cuda.synchronize() if False else None
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        if gate:
            seq[0] += 1
            L.gate_close(st.cuda_stream, seq[0])
        a.record(st)
        fn()
        b.record(st)
        if gate:
            L.gate_open(seq[0])
        b.synchronize()
        out.append(a.elapsed_time(b) * 1e3)
    torch.cuda.synchronize()
    out.sort()
    return round(out[len(out) // 2], 1)


tiny = lambda: L.tiny(cnt.data_ptr(), st.cuda_stream)  # noqa: E731
comp = lambda: C.compress(x, n, 0, C.ZVC, buf, cap, sz)  # noqa: E731
for name, fn in (('tiny', tiny), ('zvc_compress_24MiB', comp)):
    print(name, 'us: alone', run(fn, False, False), 'alone+gate', run(fn, False, True),
          '| with D2H', run(fn, True, False), 'with D2H+gate', run(fn, True, True))
