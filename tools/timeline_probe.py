"""Timeline of one bench step (CUPTI via torch.profiler): per-direction link busy time, the
gaps between copies, and kernel intervals, to see where the step exceeds the transfer bound."""
import json
import sys

import torch
from torch.profiler import ProfilerActivity, profile

sys.path.insert(0, '.')
import synth  # noqa: E402
from paper_conf_cluster_chenhzchysc21_b200 import calibrate, cswap as C  # noqa: E402

C.init(0)
calibrate.load('calib/b200.json')
ts, outs, ns = [], [], []
for i, (name, shape, s) in enumerate(synth.vgg16_b64()):
    n = synth.numel(shape)
    ts.append(synth.relu_iid_torch(n, s, seed=synth.seed_of(3, 0, 0, i), dtype=0, device='cuda'))
    outs.append(torch.empty_like(ts[-1]))
    ns.append(n)
codec = int(sys.argv[1]) if len(sys.argv) > 1 else C.AUTO


def step():
    hs = [C.swap_out(t, n, 0, codec) for t, n in zip(ts, ns)]
    for o, h in zip(reversed(outs), reversed(hs)):
        h.swap_in(o)
    return hs


for _ in range(3):
    for h in step():
        h.close()
torch.cuda.synchronize()
with profile(activities=[ProfilerActivity.CUDA]) as prof:
    hs = step()
    torch.cuda.synchronize()
for h in hs:
    h.close()
prof.export_chrome_trace('/tmp/trace.json')
ev = json.load(open('/tmp/trace.json'))['traceEvents']
gpu = [e for e in ev if e.get('ph') == 'X' and e.get('cat') in ('kernel', 'gpu_memcpy', 'gpu_memset')]
t0 = min(e['ts'] for e in gpu)
end = max(e['ts'] + e['dur'] for e in gpu)
print(f'step span {(end - t0) / 1e3:.3f} ms, events {len(gpu)}')
for kind in ('DtoH', 'HtoD'):
    cp = sorted([e for e in gpu if e['cat'] == 'gpu_memcpy' and kind in e['name']], key=lambda e: e['ts'])
    busy = sum(e['dur'] for e in cp)
    nbytes = sum(e.get('args', {}).get('bytes', 0) for e in cp)
    gaps = [(b['ts'] - (a['ts'] + a['dur'])) for a, b in zip(cp, cp[1:])]
    big = sorted(gaps, reverse=True)[:8]
    print(f'{kind}: copies {len(cp)} busy {busy / 1e3:.3f} ms bytes {nbytes / 1e6:.1f} MB -> {nbytes / busy / 1e3:.2f} GB/s;'
          f' first at {(cp[0]["ts"] - t0) / 1e3:.3f} ms, last end {(cp[-1]["ts"] + cp[-1]["dur"] - t0) / 1e3:.3f} ms;'
          f' gaps total {sum(gaps) / 1e3:.3f} ms, largest us {[round(g, 1) for g in big]}')
ks = sorted([e for e in gpu if e['cat'] == 'kernel'], key=lambda e: e['ts'])
print('kernels', len(ks), 'busy ms', round(sum(e['dur'] for e in ks) / 1e3, 3))
for e in ks[:6] + ks[-6:]:
    print(f"  {(e['ts'] - t0) / 1e3:8.3f} ms  {e['dur']:8.1f} us  {e['name'][:60]}")
print('per-kernel (swap-out phase):')
for e in ks:
    if 'compress' in e['name'] or 'probe' in e['name']:
        print(f"  {(e['ts'] - t0) / 1e3:8.3f} ms  {e['dur']:8.1f} us  {e['name'][:45]}")
for kind in ('DtoH', 'HtoD'):
    cp = sorted([e for e in gpu if e['cat'] == 'gpu_memcpy' and kind in e['name']], key=lambda e: e['ts'])
    print(kind, 'per copy: start_ms MB GB/s')
    print('  ', [(round((e['ts'] - t0) / 1e3, 2), round(e['args'].get('bytes', 0) / 1e6, 1),
                 round(e['args'].get('bytes', 0) / e['dur'] / 1e3, 1)) for e in cp])
