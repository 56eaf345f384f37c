"""Why do the bench step's D2H copies run at ~52 GB/s when a lone copy runs at 57?
Times one 784 MiB D2H (a) torch tensor -> torch pinned tensor, (b) through cswap_swap_out(NONE)
(copy engine on the library's stream into its pinned pool), (c) torch tensor -> the library's
pinned container memory with torch's copy (same destination pages as (b))."""
import ctypes
import json
import os
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_cluster_chenhzchysc21_b200 import cswap as C  # noqa: E402

C.init(0)
n = 196 << 20  # 784 MiB of f32
d = torch.randn(n, device="cuda").relu_().view(torch.int32)
hp = torch.empty(n, dtype=torch.int32).pin_memory()
st = torch.cuda.current_stream()


def ev(fn, reps=3):
    best = 1e9
    for _ in range(reps):
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(st)
        fn()
        b.record(st)
        b.synchronize()
        best = min(best, a.elapsed_time(b))
    return round(n * 4 / (best * 1e-3) / 1e9, 2)


res = {"torch_to_torch_pinned": ev(lambda: hp.copy_(d, non_blocking=True))}
walls = []
for _ in range(3):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    h = C.swap_out(d, n, C.F32, C.NONE)
    h.wait()
    walls.append(time.perf_counter() - t0)
    q = h.query()
    host_ptr = q["host"]
    keep = h
res["cswap_none_wall"] = round(n * 4 / min(walls) / 1e9, 2)
# the library's container memory as a torch tensor (same pages as (b)), data after the 80 B header
buf = (ctypes.c_int32 * n).from_address(host_ptr + 80)
ht = torch.frombuffer(buf, dtype=torch.int32)
res["torch_to_cswap_pinned"] = ev(lambda: ht.copy_(d, non_blocking=True))
keep.close()
print(json.dumps(res))
