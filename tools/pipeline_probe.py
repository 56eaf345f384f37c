"""Swap pipeline diagnostics on the VGG16 b64 set (bench workload): ms per step for several
swap-in pipeline granularities (CSWAP_SWAPIN_FRAMES) with kernel timing off / on, and a CUPTI
timeline (torch.profiler) of one step: per-direction link busy time, gaps between copies, first
copy start, kernel busy time.  Usage: python tools/pipeline_probe.py [codec] > out.jsonl"""
import json
import os
import statistics
import sys

import torch
from torch.profiler import ProfilerActivity, profile

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth  # noqa: E402
from paper_conf_cluster_chenhzchysc21_b200 import calibrate, cswap as C  # noqa: E402

C.init(0)
calibrate.load(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), 'calib', 'b200.json'))
ts, outs, ns = [], [], []
# PROBE_WORKLOAD = vgg16 (default) | resnet50 | bert: bench.py's sets and dtypes
WL = os.environ.get('PROBE_WORKLOAD', 'vgg16')
SPEC, DT = {'vgg16': (synth.vgg16_b64, 0), 'resnet50': (synth.resnet50_b64, 0), 'resnet50_f16': (synth.resnet50_b64, 1),
            'bert': (synth.bert_large_b8, 1)}[WL]
for i, (name, shape, s) in enumerate(SPEC()):
    n = synth.numel(shape)
    ts.append(synth.relu_iid_torch(n, s, seed=synth.seed_of(3, 0, 0, i), dtype=DT, device='cuda'))
    outs.append(torch.empty_like(ts[-1]))
    ns.append(n)
codec = int(sys.argv[1]) if len(sys.argv) > 1 else C.AUTO
st = torch.cuda.current_stream()


E2E = bool(os.environ.get('PROBE_E2E'))
if E2E:  # bench.py's e2e step: inputs copied H2D from pinned host memory inside the step
    hosts = [t.cpu().pin_memory() for t in ts]
    cs = torch.cuda.Stream()
    landed = [torch.cuda.Event() for _ in ts]


def step():
    if E2E:
        cs.wait_stream(st)
        with torch.cuda.stream(cs):
            for hst, t, e in zip(hosts, ts, landed):
                t.copy_(hst, non_blocking=True)
                e.record(cs)
        hs = []
        for t, n, e in zip(ts, ns, landed):
            st.wait_event(e)
            hs.append(C.swap_out(t, n, DT, codec))
    else:
        hs = [C.swap_out(t, n, DT, codec) for t, n in zip(ts, ns)]
    for o, h in zip(reversed(outs), reversed(hs)):
        h.swap_in(o)
    return hs


def ms_per_step(reps=5):
    for _ in range(2):
        for h in step():
            h.close()
    torch.cuda.synchronize()
    out = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(st)
        hs = step()
        b.record(st)
        b.synchronize()
        out.append(a.elapsed_time(b))
        for h in hs:
            h.close()
    return round(statistics.median(out), 3), [round(v, 2) for v in out]


def timeline():
    for h in step():
        h.close()
    torch.cuda.synchronize()
    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        hs = step()
        torch.cuda.synchronize()
    for h in hs:
        h.close()
    path = '/tmp/pipeline_trace.json'
    prof.export_chrome_trace(path)
    ev = json.load(open(path))['traceEvents']
    gpu = [e for e in ev if e.get('ph') == 'X' and e.get('cat') in ('kernel', 'gpu_memcpy', 'gpu_memset')]
    t0 = min(e['ts'] for e in gpu)
    end = max(e['ts'] + e['dur'] for e in gpu)
    res = {'span_ms': round((end - t0) / 1e3, 3)}
    for kind in ('DtoH', 'HtoD'):
        cp = sorted([e for e in gpu if e['cat'] == 'gpu_memcpy' and kind in e['name']], key=lambda e: e['ts'])
        busy = sum(e['dur'] for e in cp)
        nbytes = sum(e.get('args', {}).get('bytes', 0) for e in cp)
        # union of copy intervals (two H2D streams may overlap)
        union, cur_s, cur_e = 0.0, None, None
        for e in cp:
            s, f = e['ts'], e['ts'] + e['dur']
            if cur_e is None or s > cur_e:
                if cur_e is not None:
                    union += cur_e - cur_s
                cur_s, cur_e = s, f
            else:
                cur_e = max(cur_e, f)
        if cur_e is not None:
            union += cur_e - cur_s
        first, last = cp[0]['ts'] - t0, cp[-1]['ts'] + cp[-1]['dur'] - t0
        if os.environ.get('PROBE_PER_COPY'):
            res[kind + '_per_copy'] = [(round((e['ts'] - t0) / 1e3, 3), round(e['args'].get('bytes', 0) / 2**20, 2),
                                        round(e['args'].get('bytes', 0) / e['dur'] / 1e3, 2)) for e in cp]
        res[kind] = {'copies': len(cp), 'MB': round(nbytes / 1e6, 1), 'busy_union_ms': round(union / 1e3, 3),
                     'first_ms': round(first / 1e3, 3), 'last_end_ms': round(last / 1e3, 3),
                     'idle_inside_ms': round((last - first - union) / 1e3, 3),
                     'GBps_while_busy': round(nbytes / union / 1e3, 2)}
    ks = [e for e in gpu if e['cat'] == 'kernel']
    res['kernels'] = len(ks)
    res['kernel_busy_ms'] = round(sum(e['dur'] for e in ks) / 1e3, 3)
    comp = sorted([e for e in ks if 'compress' in e['name']], key=lambda e: e['ts'])
    if comp:
        res['first_compress'] = {'start_ms': round((comp[0]['ts'] - t0) / 1e3, 3), 'us': round(comp[0]['dur'], 1)}
        d2h = sorted([e for e in gpu if e['cat'] == 'gpu_memcpy' and 'DtoH' in e['name']], key=lambda e: e['ts'])
        c0_end = comp[0]['ts'] + comp[0]['dur']
        res['first_tensor_d2h_copies_started_before_its_compress_ended'] = sum(1 for e in d2h if e['ts'] < c0_end)
    return res


if os.environ.get('PROBE_TIMELINE_ONLY'):
    print(json.dumps({'codec': codec, 'timeline': timeline()}))
    sys.exit(0)
for copy_mb, group_mb in (('32', '32'), ('8', '8'), ('100000', '32'), ('32', '64'), ('32', '100000')):
    os.environ['CSWAP_COPY_MB'] = copy_mb
    os.environ['CSWAP_SWAPIN_GROUP_MB'] = group_mb
    for timing in ((False, True) if copy_mb == group_mb == '32' else (False,)):
        C.set_kernel_timing(timing)
        ms, allv = ms_per_step()
        C.set_kernel_timing(False)
        C.collect_kernel_timing()
        print(json.dumps({'copy_mb': float(copy_mb), 'swapin_group_mb': float(group_mb), 'timing': timing,
                          'ms_per_step': ms, 'all': allv}), flush=True)
    if copy_mb in ('32', '8') and group_mb == copy_mb:
        print(json.dumps({'copy_mb': float(copy_mb), 'swapin_group_mb': float(group_mb), 'timeline': timeline()}),
              flush=True)
