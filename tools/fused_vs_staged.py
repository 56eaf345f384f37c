"""Swap-out design choice (SURVEY R7 options): FUSED — the ZVC compress kernel
stores the container straight into mapped pinned host memory (SM stores over PCIe, no staging, no
copy engine) — vs STAGED — compress into device memory, then copy-engine D2H (what cswap_swap_out
does, per frame).  Per tensor of the VGG16 b64 set (sizes 24.5-784 MiB): device time of each, and
for FUSED also with the grid capped at 16 CTAs (8 SMs), since a fused kernel runs at link speed.

    python tools/fused_vs_staged.py > fused_vs_staged.jsonl
"""
import json
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth  # noqa: E402
from paper_conf_cluster_chenhzchysc21_b200 import cswap as C  # noqa: E402

C.init(0)
st = torch.cuda.current_stream()


def ev_ms(fn, reps=5):
    out = []
    for _ in range(reps + 1):
        torch.cuda.synchronize()
        torch.cuda._sleep(50_000)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(st)
        fn()
        b.record(st)
        b.synchronize()
        out.append(a.elapsed_time(b))
    return round(statistics.median(out[1:]), 4)


spec = synth.vgg16_b64()
cap_max = max(C.max_compressed_size(synth.numel(s), 0, C.ZVC) for _, s, _ in spec)
host = torch.empty(cap_max, dtype=torch.uint8).pin_memory()  # cudaHostAlloc: mapped under UVA
dev = torch.empty(cap_max, dtype=torch.uint8, device="cuda")
size = torch.zeros(1, dtype=torch.int64, device="cuda")
for i in (0, 2, 4, 9):
    name, shape, s = spec[i]
    n = synth.numel(shape)
    x = synth.relu_iid_torch(n, s, seed=synth.seed_of(3, 0, 0, i), dtype=0, device="cuda")
    cap = C.max_compressed_size(n, 0, C.ZVC)
    C.compress(x, n, 0, C.ZVC, dev, cap, size)
    torch.cuda.synchronize()
    nb = int(size.item())
    row = {"tensor": name, "MiB": n * 4 / 2**20, "container_MB": nb / 1e6}
    row["compress_device_ms"] = ev_ms(lambda: C.compress(x, n, 0, C.ZVC, dev, cap, size))
    row["d2h_copy_ms"] = ev_ms(lambda: host[:nb].copy_(dev[:nb], non_blocking=True))
    row["staged_ms"] = ev_ms(lambda: (C.compress(x, n, 0, C.ZVC, dev, cap, size),
                                      host[:nb].copy_(dev[:nb], non_blocking=True)))
    for grid in (0, 16):
        C.set_zvc_launch(grid, -1)
        row[f"fused_ms_grid{grid or 'all'}"] = ev_ms(lambda: C.compress(x, n, 0, C.ZVC, host.data_ptr(), cap, size))
    C.set_zvc_launch(0, -1)
    torch.cuda.synchronize()
    row["fused_bytes_equal"] = bool(torch.equal(host[:nb].cuda(), dev[:nb]))
    row["fused_GBps"] = round(nb / (row["fused_ms_gridall"] * 1e-3) / 1e9, 2)
    print(json.dumps(row), flush=True)
