"""Kernel-level timeline (CUPTI) of ZVC compress / decompress on small tensors, back to back."""
import json
import sys

import torch
from torch.profiler import ProfilerActivity, profile

sys.path.insert(0, '.')
import synth  # noqa: E402
from paper_conf_cluster_chenhzchysc21_b200 import cswap as C  # noqa: E402

C.init(0)
for mib in [float(a) for a in sys.argv[1:]] or [24.5]:
    n = int(mib * (1 << 18))
    x = synth.relu_iid_torch(n, 0.5, seed=1, dtype=0, device='cuda')
    y = torch.empty_like(x)
    cap = C.max_compressed_size(n, 0, C.ZVC)
    buf = torch.empty(cap, dtype=torch.uint8, device='cuda')
    sz = torch.zeros(1, dtype=torch.int64, device='cuda')
    err = torch.zeros(1, dtype=torch.int32, device='cuda')
    C.compress(x, n, 0, C.ZVC, buf, cap, sz)
    torch.cuda.synchronize()
    nb = int(sz.item())
    for _ in range(3):
        C.compress(x, n, 0, C.ZVC, buf, cap, sz)
        C.decompress(buf, nb, y, n, 0, C.ZVC, err=err)
    torch.cuda.synchronize()
    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        for _ in range(3):
            C.compress(x, n, 0, C.ZVC, buf, cap, sz)
            C.decompress(buf, nb, y, n, 0, C.ZVC, err=err)
        torch.cuda.synchronize()
    prof.export_chrome_trace('/tmp/t.json')
    ev = [e for e in json.load(open('/tmp/t.json'))['traceEvents'] if e.get('ph') == 'X' and e.get('cat') in ('kernel', 'gpu_memset', 'gpu_memcpy')]
    ev.sort(key=lambda e: e['ts'])
    t0 = ev[0]['ts']
    print(f'--- {mib} MiB  (algorithmic c {n*4*(1+0.5+1/32)/1e6:.1f} MB)')
    prev = None
    for e in ev[-12:]:
        gap = e['ts'] - prev if prev else 0
        print(f"  t={e['ts']-t0:8.1f} gap={gap:6.1f} dur={e['dur']:7.1f}  {e['name'][:50]}")
        prev = e['ts'] + e['dur']
