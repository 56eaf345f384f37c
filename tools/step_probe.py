"""Diagnose whole-step swap latency: per-step ms for NONE / ZVC / AUTO over several steps,
and the same with a host sync between swap-out and swap-in (no D2H/H2D overlap)."""
import sys
import time

import torch

sys.path.insert(0, '.')
import synth  # noqa: E402
from paper_conf_cluster_chenhzchysc21_b200 import calibrate, cswap as C  # noqa: E402

C.init(0)
calibrate.load('calib/b200.json')
spec = synth.vggs = synth.vgg16_b64()
ts, outs, ns = [], [], []
for i, (name, shape, s) in enumerate(spec):
    n = synth.numel(shape)
    ts.append(synth.relu_iid_torch(n, s, seed=synth.seed_of(3, 0, 0, i), dtype=0, device='cuda'))
    outs.append(torch.empty_like(ts[-1]))
    ns.append(n)
st = torch.cuda.current_stream()


def step(codec, sync_mid=False):
    a, m, b = (torch.cuda.Event(enable_timing=True) for _ in range(3))
    a.record(st)
    hs = [C.swap_out(t, n, 0, codec) for t, n in zip(ts, ns)]
    if sync_mid:
        for h in hs:
            h.wait()
    m.record(st)
    for o, h in zip(reversed(outs), reversed(hs)):
        h.swap_in(o)
    b.record(st)
    t0 = time.perf_counter()
    b.synchronize()
    for h in hs:
        h.close()
    return round(a.elapsed_time(b), 2), round(time.perf_counter() - t0, 4)


for codec in (C.NONE, C.ZVC, C.AUTO, C.NONE):
    print(C.CODEC_NAMES.get(codec, codec), [step(codec) for _ in range(6)])
    print('  sync-mid', [step(codec, True) for _ in range(3)])

# ---- per-tensor kernel times: inside the step vs standalone back-to-back ----------------
C.collect_kernel_timing()
C.set_kernel_timing(True)
for _ in range(3):
    step(C.ZVC)
C.set_kernel_timing(False)
recs = C.collect_kernel_timing()
comp = [r for r in recs if r['direction'] == 0][-len(ts):]
dec = [r for r in recs if r['direction'] == 1][-len(ts):]
print('in-step compress  us', [round(r['ms'] * 1e3, 1) for r in comp])
print('in-step decomp us', [round(r['ms'] * 1e3, 1) for r in dec])
bufs = []
for t, n in zip(ts, ns):
    cap = C.max_compressed_size(n, 0, C.ZVC)
    bufs.append((torch.empty(cap, dtype=torch.uint8, device='cuda'), cap, torch.zeros(1, dtype=torch.int64, device='cuda')))
err = torch.zeros(1, dtype=torch.int32, device='cuda')
for mode in ('b2b', 'sync'):
    C.set_kernel_timing(True)
    for _ in range(3):
        for (b, cap, sz), t, n in zip(bufs, ts, ns):
            C.compress(t, n, 0, C.ZVC, b, cap, sz)
            if mode == 'sync':
                torch.cuda.synchronize()
    for (b, cap, sz), o, n in zip(bufs, outs, ns):
        C.decompress(b, int(sz.item()), o, n, 0, C.ZVC, err=err)
        if mode == 'sync':
            torch.cuda.synchronize()
    C.set_kernel_timing(False)
    recs = C.collect_kernel_timing()
    c = [r for r in recs if r['direction'] == 0][-len(ts):]
    d = [r for r in recs if r['direction'] == 1][-len(ts):]
    print(mode, 'compress us', [round(r['ms'] * 1e3, 1) for r in c])
    print(mode, 'decomp us', [round(r['ms'] * 1e3, 1) for r in d])
