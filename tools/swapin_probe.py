"""Diagnose swap-in decompress group time: back-to-back vs idle gaps vs concurrent H2D."""
import sys
import torch
sys.path.insert(0, '.')
import synth
from paper_conf_cluster_chenhzchysc21_b200 import cswap as C

C.init(0)
n = 16 << 20  # one 64 MiB group (4 frames of 2^22)
x = synth.relu_iid_torch(n, 0.45, seed=1, dtype=0, device='cuda')
y = torch.empty_like(x)
cap = C.max_compressed_size(n, C.F32, C.ZVC)
buf = torch.empty(cap, dtype=torch.uint8, device='cuda')
sz = torch.zeros(1, dtype=torch.int64, device='cuda')
err = torch.zeros(1, dtype=torch.int32, device='cuda')
C.compress(x, n, C.F32, C.ZVC, buf, cap, sz)
torch.cuda.synchronize()
nb = int(sz.item())
host = torch.empty(256 << 20, dtype=torch.uint8).pin_memory()
dev2 = torch.empty(256 << 20, dtype=torch.uint8, device='cuda')
side = torch.cuda.Stream()


def t(fn, reps=10):
    fn(); torch.cuda.synchronize()
    out = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); fn(); b.record(); b.synchronize()
        out.append(a.elapsed_time(b))
    out.sort()
    return round(out[len(out) // 2] * 1000, 1)


dec = lambda: C.decompress(buf, nb, y, n, C.F32, C.ZVC, err=err)  # noqa: E731
print('back-to-back us', t(dec))
def gap():
    torch.cuda._sleep(1_000_000)  # ~0.5 ms of idle-ish spinning on the stream
    torch.cuda.synchronize()
print('after host sync gap us', t(lambda: (gap(), dec())))
import time
def idle():
    torch.cuda.synchronize(); time.sleep(0.001)
res = []
for _ in range(10):
    idle()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(); dec(); b.record(); b.synchronize(); res.append(a.elapsed_time(b))
res.sort(); print('after 1 ms idle us', round(res[5] * 1000, 1))
# concurrent H2D on a side stream
res = []
for _ in range(10):
    torch.cuda.synchronize()
    with torch.cuda.stream(side):
        dev2.copy_(host, non_blocking=True)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(); dec(); b.record(); b.synchronize(); res.append(a.elapsed_time(b))
    torch.cuda.synchronize()
res.sort(); print('with concurrent H2D us', round(res[5] * 1000, 1))
