"""bench.py — CSWAP hot path on B200: compressed swap-out + swap-in of the VGG16 batch-64
activation set (BASELINE.json configs[2]) with cost-model codec selection.

One step = the whole hot path over one batch: for each of the 12 conv-input ReLU/MAX tensors
in forward order, probe + select + compress + D2H to pinned host (swap-out); then for each in
reverse order, H2D + decompress (swap-in) (Fig. 2, :64-:72; vDNN policy :251).
value = raw tensor bytes swapped out and back in per second, summed over ranks (GB/s).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                    [--workload vgg16|resnet50|resnet50_f16|bert] [--calibrate] [--no-extras]
Multi-GPU ("replicas only"): one process per GPU, each swapping its own replica
of the set (no collective on the data path, "scaling": "weak"); time = the slowest rank's device
time.  Under torchrun the ranks come from the environment; `python bench.py --gpus N` without
torchrun starts the N rank processes itself (RANK / LOCAL_RANK / WORLD_SIZE set per child).  The
ranks meet only on a CPU (gloo) barrier and one MAX / gather of per-rank numbers.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "compressed swap-out+in latency & codec GB/s vs HBM roofline, 1/2/4/8 B200"
CALIB_PATH = os.path.join(ROOT, "calib", "b200.json")
NCU_SUMMARY = os.path.join(ROOT, "profiles", "ncu_r02.json")


def log(*a):
    if int(os.environ.get("RANK", "0")) == 0:
        print(*a, file=sys.stderr, flush=True)


def workload(name: str):
    import synth
    if name == "vgg16":
        return "vgg16_b64_swapset", synth.vgg16_b64(), synth.F32
    if name == "resnet50":
        return "resnet50_b64_swapset", synth.resnet50_b64(), synth.F32
    if name == "resnet50_f16":  # BASELINE configs[3]: the same set in fp16 (1197.4 MiB)
        return "resnet50_b64_f16_swapset", synth.resnet50_b64(), synth.F16
    if name == "bert":
        return "bert_large_b8_swapset", synth.bert_large_b8(), synth.F16
    raise SystemExit(f"unknown workload {name}")


# ------------------------------------------------------------------------------------ clocks
class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled every 200 ms during the timed region."""
    FIELDS = ["clocks.sm", "clocks.max.sm", "clocks_event_reasons.hw_slowdown",
              "clocks_event_reasons.hw_thermal_slowdown", "clocks_event_reasons.sw_thermal_slowdown",
              "clocks_event_reasons.sw_power_cap"]

    def __init__(self, device: int):
        self.device = device
        self.proc = None

    def __enter__(self):
        self.first = ""
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.device), "--query-gpu=" + ",".join(self.FIELDS),
                 "--format=csv,noheader,nounits", "-lms", "200"], stdout=subprocess.PIPE,
                stderr=subprocess.DEVNULL, text=True)
            # wait for the first sample: nvidia-smi's start-up (NVML init, first query) then falls
            # before the caller's warm-up and timed steps, not inside them
            import select
            if select.select([self.proc.stdout], [], [], 10.0)[0]:
                self.first = self.proc.stdout.readline()
        except OSError:
            self.proc = None
        return self

    def __exit__(self, *exc):
        self.out = ""
        if self.proc:
            self.proc.terminate()
            try:
                self.out, _ = self.proc.communicate(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()
        self.out = getattr(self, "first", "") + (self.out or "")

    def summary(self) -> dict:
        sms, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in (getattr(self, "out", "") or "").splitlines():
            parts = [p.strip() for p in line.split(",")]
            if len(parts) != len(self.FIELDS):
                continue
            try:
                sms.append(float(parts[0]))
                mx = float(parts[1])
            except ValueError:
                continue
            for nm, v in zip(names, parts[2:]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sms) if sms else None, "sm_max_mhz": mx, "samples": len(sms),
                "reasons": sorted(reasons)}


# ------------------------------------------------------------------------------------ ours
def _bind_local_cpus(device: int) -> str:
    """Pin this process to the CPUs NVML reports as closest to `device` before any pinned host
    memory is allocated (each GPU's pinned pool NUMA-local; with 8 replicas the
    host links and DRAM are the shared resources)."""
    try:
        import pynvml
        pynvml.nvmlInit()
        h = pynvml.nvmlDeviceGetHandleByIndex(device)
        pynvml.nvmlDeviceSetCpuAffinity(h)
        return f"nvml cpu affinity: {len(os.sched_getaffinity(0))} cpus"
    except Exception as e:  # no NVML / not permitted: leave the affinity alone
        return f"unchanged ({type(e).__name__})"


def run_ours(args, rank: int, world: int, local_rank: int, dist) -> dict | None:
    import torch

    import synth
    from paper_conf_cluster_chenhzchysc21_b200 import calibrate, cswap as C

    torch.cuda.set_device(local_rank)
    numa = _bind_local_cpus(local_rank)
    C.init(local_rank)  # the pinned pools are first-touched by this (now GPU-local) thread
    if args.swap_target != "host":
        if args.swap_target == "peer" and world < 2:
            raise SystemExit("bench.py: --swap-target peer needs --gpus >= 2")
        C.set_swap_target(local_rank if args.swap_target == "self" else (local_rank + 1) % world)
    codecs_built = [c for c in (C.ZVC, C.RLE, C.CSR, C.LZ4) if _codec_built(C, c)]
    if args.calibrate or not calibrate.load(CALIB_PATH):
        log(f"calibrating on the box (codecs {codecs_built}) ...")
        calibrate.run(codecs_built, quick=not args.calibrate, path=CALIB_PATH if args.calibrate else None, log=log)
    cal = C.get_calibration()

    wname, tensors_spec, dtype = workload(args.workload)
    w = C.WIDTH[dtype]
    dev = torch.device("cuda", local_rank)
    tensors, outs, sizes = [], [], []
    for i, (name, shape, s) in enumerate(tensors_spec):
        n = synth.numel(shape)
        tensors.append(synth.relu_iid_torch(n, s, seed=rank_seed(synth.seed_of(3, 0, 0, i), rank), dtype=dtype,
                                            device=dev))
        outs.append(torch.empty_like(tensors[-1]))
        sizes.append(n)
    raw_bytes = sum(sizes) * w
    torch.cuda.synchronize()
    stream = torch.cuda.current_stream()

    def step(codec):
        hs = [C.swap_out(t, n, dtype, codec) for t, n in zip(tensors, sizes)]
        for o, h in zip(reversed(outs), reversed(hs)):
            h.swap_in(o)
        return hs

    def barrier():
        torch.cuda.synchronize()
        if dist is not None:
            dist.barrier()
        torch.cuda.synchronize()

    def timed(codec, steps, warmup, record=False, clocks=False):
        # the clock sampler starts before the warm-up so that nvidia-smi is already sampling
        # (every 200 ms) when the short timed region begins; it stops right after it
        sampler = ClockSampler(local_rank) if clocks and not os.environ.get("BENCH_NO_CLOCKS") else None
        if sampler:
            sampler.__enter__()
        for _ in range(warmup):
            for h in step(codec):
                h.close()
        barrier()
        launches0 = C.kernel_launches()
        if record:
            C.collect_kernel_timing()
            C.set_kernel_timing(True)
        t0 = time.perf_counter()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        hs_last = None
        marks = []  # an event at every step boundary: per-step times (steady state vs first steps)
        for i in range(steps):
            hs = step(codec)
            if i + 1 < steps:
                marks.append(torch.cuda.Event(enable_timing=True))
                marks[-1].record(stream)
                for h in hs:
                    h.close()
            else:
                hs_last = hs
        b.record(stream)
        b.synchronize()
        bounds = [a] + marks + [b]
        step_ms = [round(x.elapsed_time(y), 3) for x, y in zip(bounds, bounds[1:])]
        wall = time.perf_counter() - t0
        if sampler:
            sampler.__exit__(None, None, None)
        if record:
            C.set_kernel_timing(False)
        launches = C.kernel_launches() - launches0
        ms = a.elapsed_time(b)
        recs = C.collect_kernel_timing() if record else []
        barrier()
        info = [h.query() for h in hs_last]
        for h in hs_last:
            h.close()
        return {"ms": ms, "wall_s": wall, "launches": launches, "records": recs, "handles": info,
                "clocks": sampler.summary() if sampler else None, "step_ms": step_ms}

    # ---- headline: AUTO selection ---------------------------------------------------------
    main = timed(C.AUTO, args.steps, args.warmup, record=True, clocks=True)
    ms_max = _max_over_ranks(main["ms"], dist)
    ms_per_step = ms_max / args.steps
    value = job_throughput(world, raw_bytes, ms_per_step)
    for o, t in zip(outs, tensors):  # the last step restored every tensor bitwise
        assert torch.equal(o, t), "swap round trip mismatch"

    roof = _roofline(main["records"], args.steps)
    roof["isolated"] = _isolated(C, torch, tensors, sizes, dtype, w, [q["codec"] for q in main["handles"]], stream,
                                 roof.get("peak"))
    result = {
        "metric": METRIC, "value": round(value, 3), "unit": "GB/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": round(ms_per_step, 4), "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "u32" if w == 4 else "u16", "data": "synthetic",
        "config": {"workload": wname, "tensors": len(sizes), "raw_MiB_per_gpu": raw_bytes / 2**20,
                   "elem": synth.NAMES[dtype], "selector": "pipelined" if cal.mode == 0 else "paper",
                   "frame_elems": int(C.get_format().frame_elems),
                   "l2": "working set 2.2 GB >> 126 MB L2: every step streams from HBM (no flush needed)",
                   "parallelism": f"replicas x{world}", "host_binding": numa, "swap_target": args.swap_target},
        "gpu_launches": main["launches"],
        "step_ms": main["step_ms"],
        "clocks": main["clocks"],
        "roofline": roof,
    }
    decisions = [q["codec"] for q in main["handles"]]
    comp_bytes = [q["bytes"] for q in main["handles"]]
    result["config"]["codecs_chosen"] = [C.CODEC_NAMES[c] for c in decisions]
    result["config"]["compressed_MiB"] = sum(comp_bytes) / 2**20

    if not args.no_extras:
        result["extras"] = _extras(args, C, torch, tensors, outs, sizes, dtype, w, timed, main, dist, raw_bytes,
                                   world)
        result["e2e"] = _e2e(args, C, torch, tensors, outs, sizes, dtype, w, dist, world, stream)
    # per-rank numbers, measured with every rank running at once (replicas share the host links)
    rank_info = {"rank": rank, "ms_per_step": round(main["ms"] / args.steps, 4), "host_binding": numa}
    if "extras" in result:
        ex = result["extras"]
        rank_info.update(link=ex["link"], every_compressed_tensor_faster=ex["every_compressed_tensor_faster"],
                         swap_latency_reduction_vs_vdnn=round(ex["swap_latency_reduction_vs_vdnn"], 4))
    per_rank = _gather(dist, rank_info)
    result["per_rank"] = per_rank
    if "extras" in result:
        result["every_compressed_tensor_faster_all_ranks"] = all(p["every_compressed_tensor_faster"] for p in per_rank)
    if rank == 0 and world == 1 and not args.no_cpu:
        result["cpu_baseline"] = _cpu_baseline(tensors, sizes, decisions, dtype)
    return result


def _codec_built(C, codec) -> bool:
    import torch
    x = torch.zeros(1024, dtype=torch.int32, device="cuda")
    cap = C.max_compressed_size(1024, C.F32, codec)
    buf = torch.empty(cap, dtype=torch.uint8, device="cuda")
    sz = torch.zeros(1, dtype=torch.int64, device="cuda")
    try:
        C.compress(x, 1024, C.F32, codec, buf, cap, sz)
        torch.cuda.synchronize()
        return True
    except C.CswapError as e:
        if e.status == 6:
            return False
        raise


def _max_over_ranks(v: float, dist) -> float:
    """Device time of the slowest rank (the job's time)."""
    if dist is None or not dist.is_initialized():
        return v
    import torch
    t = torch.tensor([v], dtype=torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def rank_seed(base: int, rank: int) -> int:
    """Each replica swaps its own tensors: distinct seeds per rank, same recipe."""
    return base + 7919 * rank


def job_throughput(world: int, raw_bytes_per_rank: int, ms_max: float) -> float:
    """Whole-job GB/s: bytes swapped out and back in by all ranks / the slowest rank's time."""
    return world * raw_bytes_per_rank / (ms_max * 1e-3) / 1e9


def _peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return d.get("hbm_gbs", 6650.0), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md)"


def _roofline(records, steps: int = 1) -> dict:
    """Dominant kernel = the codec launch group with the largest total device time in the timed
    region; algorithmic bytes = raw bytes + container bytes per launch."""
    peak, src = _peaks()
    groups = {}
    for r in records:
        if r["direction"] == 2:
            continue
        key = (r["codec"], r["direction"])
        g = groups.setdefault(key, {"ms": 0.0, "bytes": 0, "launches": 0, "dev_ms": 0.0, "dev_n": 0, "k_ms": 0.0,
                                    "k_n": 0})
        g["ms"] += r["ms"]
        if r.get("device_ms", 0.0) > 0:
            g["dev_ms"] += r["device_ms"]
            g["dev_n"] += 1
        if r.get("kernel_ms", 0.0) > 0:
            g["k_ms"] += r["kernel_ms"]
            g["k_n"] += 1
        g["bytes"] += r["raw_bytes"] + r["comp_bytes"]
        g["launches"] += 1
    if not groups:
        return {"bound": "hbm", "achieved": None, "peak": peak, "unit": "GB/s", "frac": None, "traffic": None}
    # the dominant single kernel: compress (one launch per tensor).  A decompress group is
    # count + scan + expand (+ prep); its largest kernel (expand) has a smaller share of the
    # step than compress in the committed launch list (profiles/launches_r01.txt).
    single = {kk: v for kk, v in groups.items() if kk[1] == 0} or groups
    (codec, d), g = max(single.items(), key=lambda kv: kv[1]["ms"])
    achieved = g["bytes"] / (g["ms"] * 1e-3) / 1e9
    names = {0: "none", 1: "zvc", 2: "rle", 3: "csr", 4: "lz4"}
    # traffic: DRAM read+write bytes per launch group of the same kernels in one step of this
    # bench, from the committed `ncu --set full` capture (profiles/ncu_r01.json, "bench_step")
    traffic = None
    if os.path.exists(NCU_SUMMARY):
        with open(NCU_SUMMARY) as f:
            prof = json.load(f).get("bench_step", {})
        stem = {0: "none", 1: "zvc", 2: "rle", 3: "csr", 4: "lz4"}[codec]
        parts = ["compress"] if d == 0 else ["count", "scan", "expand", "dscan", "decode", "prep"]
        tot = sum(v["dram_bytes_per_launch"] * v["launches"] for kname, v in prof.items()
                  if (kname.startswith(stem) or (d == 1 and kname.startswith("prep")))
                  and any(p in kname for p in parts))
        if tot:
            traffic = round(tot / (g["launches"] / steps))  # per launch group, like `achieved`
    out = {"bound": "hbm", "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
           "frac": round(achieved / peak, 4), "traffic": traffic,
           "kernel": f"{names[codec]}_{'compress' if d == 0 else 'decompress'}", "launches": g["launches"],
           "algorithmic_bytes_per_launch": g["bytes"] / g["launches"], "avg_launch_ms": g["ms"] / g["launches"],
           "peak_source": src}
    out["note"] = ("in-step CUDA events around each launch group include a timing event's own cost while the "
                   "concurrent D2H streams over PCIe (~32 us of stream time per record, tools/event_gap_probe.cu, "
                   "DESIGN.md §7.3); kernel_clock times the same compress launches by the kernel's own %globaltimer "
                   "span, isolated the same tensors without a copy running")
    if g["dev_n"] == g["launches"] and g["dev_ms"] > 0:
        dev = g["bytes"] / (g["dev_ms"] * 1e-3) / 1e9
        out["device_clock"] = {
            "achieved": round(dev, 1), "frac": round(dev / peak, 4), "avg_launch_ms": round(g["dev_ms"] / g["launches"], 4),
            "how": "same launches, same bytes; duration = %globaltimer between 1-thread stamp kernels placed first and "
                   "last in each launch group's graph (no event record waiting behind the concurrent D2H's PCIe writes)"}
    if g["k_n"] == g["launches"] and g["k_ms"] > 0:
        kc = g["bytes"] / (g["k_ms"] * 1e-3) / 1e9
        out["kernel_clock"] = {
            "achieved": round(kc, 1), "frac": round(kc / peak, 4), "avg_launch_ms": round(g["k_ms"] / g["launches"], 4),
            "how": "same launches, same bytes; duration = the persistent compress kernel's own %globaltimer span "
                   "(CTA 0's start to the last CTA's finish, before its host-memory stores; the grid is co-resident), "
                   "written to device memory; the timed compress groups carry no stamp kernels"}
    out["all_kernels"] = {f"{names[c]}_{'c' if dd == 0 else 'dc'}": {
        "GBps": round(v["bytes"] / (v["ms"] * 1e-3) / 1e9, 1), "frac": round(v["bytes"] / (v["ms"] * 1e-3) / 1e9 / peak, 4),
        "ms_total": round(v["ms"], 3), "launches": v["launches"]} for (c, dd), v in groups.items()}
    return out


def _isolated(C, torch, tensors, sizes, dtype, w, codecs, stream, peak, reps=3) -> dict:
    """The same codec launches with no copy engine running: each tensor of the set compressed
    (device -> device) and decompressed with its chosen codec, CUDA events around every call.
    In the timed step every launch group shares the GPU with a D2H / H2D copy, and then each
    event record and kernel boundary waits ~10-20 us behind the copy's queued PCIe writes
    (tools/launch_probe*.py); this shows what the kernels reach without that."""
    out = {}
    work = [(t, n, c) for t, n, c in zip(tensors, sizes, codecs) if c != C.NONE]
    if not work:
        return out
    cap = max(C.max_compressed_size(n, dtype, c) for _, n, c in work)
    buf = torch.empty(cap, dtype=torch.uint8, device="cuda")
    size = torch.zeros(1, dtype=torch.int64, device="cuda")
    dst = torch.empty(max(n for _, n, _ in work) * w, dtype=torch.uint8, device="cuda")
    err = torch.zeros(1, dtype=torch.int32, device="cuda")
    tc = td = 0.0
    nbytes = 0
    for t, n, c in work:
        for r in range(reps + 1):
            a, b, d = (torch.cuda.Event(enable_timing=True) for _ in range(3))
            # keep the stream busy while the host enqueues, so that the events time the device
            # work and not the host-side capture of the launch group
            torch.cuda._sleep(100000)
            a.record(stream)
            C.compress(t, n, dtype, c, buf, cap, size, stream=stream)
            b.record(stream)
            C.decompress(buf, cap, dst, n, dtype, c, err=err, stream=stream)
            d.record(stream)
            d.synchronize()
            if r:  # the first round is a warm-up
                tc += a.elapsed_time(b)
                td += b.elapsed_time(d)
                nbytes += n * w + int(size.item())
    assert int(err.item()) == 0
    for name, ms in (("compress", tc), ("decompress", td)):
        gbs = nbytes / (ms * 1e-3) / 1e9
        out[name] = {"achieved": round(gbs, 1), "frac": round(gbs / peak, 4) if peak else None,
                     "avg_launch_ms": round(ms / (reps * len(work)), 4)}
    out["how"] = (f"every tensor of the set with its chosen codec, device->device, no copy running, "
                  f"{reps} reps after a warm-up, CUDA events per call on the launching stream")
    return out


def _link(torch, nbytes=256 << 20, reps=5) -> dict:
    host = torch.empty(nbytes, dtype=torch.uint8).pin_memory()
    dev = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    res = {}
    for name, fn in (("d2h", lambda: host.copy_(dev, non_blocking=True)),
                     ("h2d", lambda: dev.copy_(host, non_blocking=True))):
        fn()
        torch.cuda.synchronize()
        best = 1e9
        for _ in range(reps):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            fn()
            b.record()
            b.synchronize()
            best = min(best, a.elapsed_time(b))
        res[name + "_GBps"] = round(nbytes / (best * 1e-3) / 1e9, 2)
    return res


def _extras(args, C, torch, tensors, outs, sizes, dtype, w, timed, main, dist, raw_bytes, world) -> dict:
    """Baselines in the same run: vDNN (NONE), SC (always ZVC), the Orac bound; link GB/s;
    per-tensor latency check (compressed < uncompressed for every tensor the selector compressed)."""
    ex = {}
    if dist is not None:  # all ranks measure the link at the same time (shared PCIe / host DRAM)
        torch.cuda.synchronize()
        dist.barrier()
    link = _link(torch)
    ex["link"] = link
    steps_b = max(2, min(args.steps, 3))
    none = timed(C.NONE, steps_b, 3)
    sc = timed(C.ZVC, steps_b, 3)
    ex["latency_ms"] = {"auto": main["ms"] / args.steps, "vdnn_none": none["ms"] / steps_b,
                        "sc_always_zvc": sc["ms"] / steps_b}
    comp = sum(q["bytes"] for q in main["handles"])
    orac = comp / (link["d2h_GBps"] * 1e9) + comp / (link["h2d_GBps"] * 1e9)
    ex["latency_ms"]["orac_bound"] = orac * 1e3
    ex["latency_ms"]["raw_link_bound"] = (raw_bytes / (link["d2h_GBps"] * 1e9) + raw_bytes / (link["h2d_GBps"] * 1e9)) * 1e3
    ex["swap_latency_reduction_vs_vdnn"] = 1 - ex["latency_ms"]["auto"] / ex["latency_ms"]["vdnn_none"]
    # per-tensor: the selector's choice vs NONE, measured one tensor at a time (on every rank at
    # once: SURVEY §8(d) asks for compressed < uncompressed with all GPUs swapping concurrently)
    if dist is not None:
        torch.cuda.synchronize()
        dist.barrier()
    per = []
    stream = torch.cuda.current_stream()
    for i, (t, o, n) in enumerate(zip(tensors, outs, sizes)):
        q = main["handles"][i]
        row = {"i": i, "MiB": n * w / 2**20, "codec": C.CODEC_NAMES[q["codec"]], "ratio": q["bytes"] / (n * w)}
        for label, codec in (("none_ms", C.NONE), ("chosen_ms", q["codec"])):
            best = 1e9
            for _ in range(3):
                torch.cuda.synchronize()
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(stream)
                h = C.swap_out(t, n, dtype, codec)
                h.swap_in(o)
                b.record(stream)
                b.synchronize()
                h.close()
                best = min(best, a.elapsed_time(b))
            row[label] = round(best, 4)
        per.append(row)
    ex["per_tensor"] = per
    ex["every_compressed_tensor_faster"] = all(r["chosen_ms"] < r["none_ms"] for r in per if r["codec"] != "none")
    # decision accuracy (PAPER.md:305 analogue): the selector's codec vs the measured-fastest of
    # the five choices, per tensor, on the workload set and on a mixed set whose sparsity
    # structure makes every codec the right answer somewhere
    ex["decision_accuracy"] = {
        "workload": _decision_accuracy(C, torch, list(zip(tensors, outs, sizes)), dtype,
                                       [r["codec"] for r in per]),
        "mixed_set": _decision_accuracy(C, torch, _mixed_set(torch), None, None),
    }
    # overheads: probe kernel + readback, host selector
    tp = []
    for t, n in zip(tensors, sizes):
        t0 = time.perf_counter()
        pr = C.probe(t, n, dtype)
        t1 = time.perf_counter()
        C.select_from_probe(n, dtype, pr)
        t2 = time.perf_counter()
        tp.append((t1 - t0, t2 - t1))
    ex["overheads_us"] = {"probe_incl_readback": round(1e6 * sum(a for a, _ in tp) / len(tp), 2),
                          "select_host": round(1e6 * sum(b for _, b in tp) / len(tp), 2)}
    # host time of a fixed-codec swap-out call while the stream is busy (it only enqueues: no
    # device wait), for the largest tensor of the set; a no-op call through the same binding
    # gives the Python / ctypes share
    big = max(range(len(tensors)), key=lambda i: sizes[i])
    for rep in range(2):  # the first pass grows the staging / pinned pools to 10 outstanding swaps
        torch.cuda.synchronize()
        torch.cuda._sleep(200_000_000)
        hs, th = [], []
        for _ in range(10):
            t0 = time.perf_counter()
            hs.append(C.swap_out(tensors[big], sizes[big], dtype, C.ZVC))
            th.append(time.perf_counter() - t0)
        if rep == 0:
            for h in hs:
                h.close()
    t_noop = []
    for _ in range(10):
        t0 = time.perf_counter()
        C.kernel_launches()
        t_noop.append(time.perf_counter() - t0)
    for h in hs:
        h.close()
    ex["overheads_us"]["swap_out_call_busy_stream"] = {
        "tensor_MiB": sizes[big] * w / 2**20, "median_us": round(1e6 * statistics.median(th), 1),
        "min_us": round(1e6 * min(th), 1), "noop_binding_call_us": round(1e6 * statistics.median(t_noop), 1)}
    return ex


def _swap_ms(C, torch, t, o, n, dtype, codec, reps=2):
    """Best-of-reps device time of one swap out + swap in of a single tensor; returns
    (ms, codec actually used)."""
    stream = torch.cuda.current_stream()
    best, used = 1e9, codec
    for _ in range(reps):
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        h = C.swap_out(t, n, dtype, codec)
        h.swap_in(o)
        b.record(stream)
        b.synchronize()
        used = h.query()["codec"]
        h.close()
        best = min(best, a.elapsed_time(b))
    return best, used


def _mixed_set(torch):
    """32 MiB tensors (f32 unless noted) spanning the sparsity structures of DESIGN.md §5:
    iid ReLU masks, clustered zero runs, dead channels, a constant non-zero tensor, f16."""
    import numpy as np

    import synth
    n = 8 << 20
    specs = [("iid", s) for s in (0.0, 0.3, 0.6, 0.9, 0.99)] + \
            [("clustered", s) for s in (0.5, 0.9, 0.99)] + [("dead", s) for s in (0.3, 0.8)] + \
            [("constant", 0.0), ("iid_f16", 0.7)]
    out = []
    for i, (kind, s) in enumerate(specs):
        seed = synth.seed_of(5, 0, 0, i)
        dt = synth.F32
        if kind == "iid":
            x = synth.relu_iid(n, s, seed)
        elif kind == "clustered":
            x = synth.relu_clustered(n, s, 512, seed)
        elif kind == "dead":
            x = synth.channel_dead((64, 128, 32, 32), s, seed)
        elif kind == "constant":
            x = synth.constant(n, 0x3F800000)
        else:
            dt = synth.F16
            x = synth.relu_iid(2 * n, s, seed, dtype=dt)
        t = torch.from_numpy(x.view(np.int32 if dt == synth.F32 else np.int16)).cuda()
        out.append((t, torch.empty_like(t), x.size, dt, f"{kind}_{s}"))
    return out


def _decision_accuracy(C, torch, items, dtype, chosen) -> dict:
    """Selector's codec (AUTO) vs the measured-fastest codec per tensor. A choice within 2 % of
    the fastest also counts as correct (`within_2pct`): the cost model cannot separate those."""
    rows, exact, near = [], 0, 0
    for i, it in enumerate(items):
        if dtype is None:
            t, o, n, dt, label = it
        else:
            (t, o, n), dt, label = it, dtype, str(i)
        times = {C.CODEC_NAMES[c]: round(_swap_ms(C, torch, t, o, n, dt, c)[0], 4)
                 for c in (C.NONE, C.ZVC, C.RLE, C.CSR, C.LZ4)}
        if chosen is None:
            ms_auto, used = _swap_ms(C, torch, t, o, n, dt, C.AUTO, reps=1)
            pick = C.CODEC_NAMES[used]
        else:
            pick = chosen[i]
        fastest = min(times, key=times.get)
        exact += pick == fastest
        near += times[pick] <= 1.02 * times[fastest]
        rows.append({"tensor": label, "chosen": pick, "fastest": fastest, "ms": times})
    k = len(rows)
    return {"exact": exact, "within_2pct": near, "total": k, "frac": round(exact / k, 4),
            "frac_within_2pct": round(near / k, 4), "per_tensor": rows}


def _e2e(args, C, torch, tensors, outs, sizes, dtype, w, dist, world, stream) -> dict:
    """Same metric through the public API with HOST inputs: per step the 12 inputs are copied
    H2D from pinned host memory (input i+1's copy overlapping tensor i's swap-out), swapped out
    and back in, and 16 bytes of every restored tensor are read back D2H."""
    hosts = [t.cpu().pin_memory() for t in tensors]
    probe_back = torch.empty(len(tensors), 4, dtype=torch.int32).pin_memory()
    steps = max(2, min(args.steps, 5))
    # the input copies run on their own stream, one event per tensor, so the H2D of input i+1
    # overlaps the swap-out (compress + D2H) of tensor i: PCIe is full duplex
    cs = torch.cuda.Stream()
    landed = [torch.cuda.Event() for _ in tensors]

    def one():
        cs.wait_stream(stream)
        with torch.cuda.stream(cs):
            for hst, t, e in zip(hosts, tensors, landed):
                t.copy_(hst, non_blocking=True)
                e.record(cs)
        hs = []
        for t, n, e in zip(tensors, sizes, landed):
            stream.wait_event(e)
            hs.append(C.swap_out(t, n, dtype, C.AUTO))
        for o, h in zip(reversed(outs), reversed(hs)):
            h.swap_in(o)
        for i, o in enumerate(outs):
            probe_back[i].copy_(o[:4 * 4 // w].view(torch.int32)[:4], non_blocking=True)
        return hs

    for h in one():
        h.close()
    torch.cuda.synchronize()
    if dist is not None:
        dist.barrier()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(stream)
    marks = []
    for i in range(steps):
        for h in one():
            h.close()
        if i + 1 < steps:
            marks.append(torch.cuda.Event(enable_timing=True))
            marks[-1].record(stream)
    b.record(stream)
    b.synchronize()
    bounds = [a] + marks + [b]
    step_ms = [round(x.elapsed_time(y), 3) for x, y in zip(bounds, bounds[1:])]
    ms = _max_over_ranks(a.elapsed_time(b), dist) / steps
    raw = sum(sizes) * w
    return {"value": round(world * raw / (ms * 1e-3) / 1e9, 3), "unit": "GB/s", "ms_per_step": round(ms, 3),
            "h2d_bytes_per_step": raw, "d2h_bytes_per_step": 16 * len(tensors), "steps": steps, "step_ms": step_ms}


def _cpu_model() -> str:
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except OSError:
        pass
    import platform
    return platform.processor() or "unknown"


def _oracle_seconds(xs, codec: int, dtype: int, threads: int) -> float:
    """Seconds for the plain-C oracle, as it stands, to compress and then decompress every
    array of `xs` with `codec`, frame by frame (F = 2^22 elements, the container default).
    With threads > 1 the frames of all arrays are spread over a pool of host threads (the
    ctypes call releases the GIL, so each thread runs the scalar C code on its own frames: the
    "OpenMP over frames, timing only" of SURVEY §8(d)); the oracle itself is unchanged."""
    import concurrent.futures as cf

    from oracle import oracle as O
    F = O.DEFAULT_F
    frames = [x[k:k + F] for x in xs for k in range(0, x.size, F)]

    def one(fr):
        blob = O.compress(fr, codec, dtype)
        O.decompress(blob, fr.size, dtype)

    t0 = time.perf_counter()
    if threads <= 1:
        for fr in frames:
            one(fr)
    else:
        with cf.ThreadPoolExecutor(max_workers=threads) as ex:
            list(ex.map(one, frames))
    return time.perf_counter() - t0


def _cpu_baseline(tensors, sizes, decisions, dtype) -> dict:
    """The plain-C oracle on the host cores (SURVEY §8(d) "oracle timing"; PAPER.md:251 compares
    with vDNN++'s 64 CPU threads): compress + decompress with the codec the selector chose for
    each tensor (NONE = raw copy), on a bounded sample of every tensor of the set.  `value` = all
    host cores (frames spread over threads), `single_thread` on a smaller sample."""
    import numpy as np
    w = 4 if dtype == 0 else 2
    cores = len(os.sched_getaffinity(0)) if hasattr(os, "sched_getaffinity") else (os.cpu_count() or 1)

    def sample(mib):
        xs, tot = [], 0
        for t, n in zip(tensors, sizes):
            m = min(n, mib * 2**20 // w)
            x = t[:m].cpu().numpy()
            xs.append(x.view(np.uint32) if w == 4 else x.view(np.uint16))
            tot += m * w
        return xs, tot

    def timed(xs, threads):
        secs = 0.0
        by_codec = {}
        for x, c in zip(xs, decisions):
            by_codec.setdefault(c, []).append(x)
        for c, group in by_codec.items():
            secs += _oracle_seconds(group, c, dtype, threads)
        return secs

    xs1, b1 = sample(16)
    s1 = timed(xs1, 1)
    xsn, bn = sample(64)
    sn = timed(xsn, cores)
    return {"value": round(bn / sn / 1e9, 4), "unit": "GB/s", "cores": cores, "kind": "oracle",
            "sample": f"first 64 MiB of each of the {len(sizes)} tensors ({bn / 2**20:.0f} MiB), oracle compress+"
                      f"decompress with the selector's codec, frames spread over {cores} threads, {sn:.1f} s",
            "single_thread": {"value": round(b1 / s1 / 1e9, 4), "cores": 1,
                              "sample": f"first 16 MiB of each tensor ({b1 / 2**20:.0f} MiB), {s1:.1f} s"},
            "cpu_model": _cpu_model(), "cpu_count": os.cpu_count()}


def cpu_plan(path: str) -> dict:
    """SURVEY §8(d) oracle-timing plan (`bench.py --cpu-plan OUT.json`, CPU only): per codec,
    single thread on config 1 and on the config-2 iid fp32 points up to 64 MiB at s = 0.2 / 0.5 /
    0.8 and 1 GiB at the same sparsities; all host cores for the points >= 16 MiB."""
    import synth
    cores = len(os.sched_getaffinity(0)) if hasattr(os, "sched_getaffinity") else (os.cpu_count() or 1)
    rows = []
    cfg1 = synth.relu_iid(1 << 20, 0.5, seed=synth.seed_of(1), exact=True)
    points = [("config1_4MiB", cfg1, 0.5)]
    for si, s in enumerate((0.2, 0.5, 0.8)):
        for zi, mib in enumerate((0.0625, 0.25, 1, 4, 16, 64, 1024)):
            n = int(mib * 2**18)
            points.append((f"iid_{mib}MiB", synth.relu_iid(n, s, seed=synth.seed_of(2, zi, si)), s))
    for name, x, s in points:
        for codec in (1, 2, 3, 4):
            for threads in ((1, cores) if x.nbytes >= 16 << 20 else (1,)):
                secs = _oracle_seconds([x], codec, 0, threads)
                rows.append({"point": name, "sparsity": s, "MiB": x.nbytes / 2**20, "codec": codec,
                             "threads": threads, "s": round(secs, 4), "GBps": round(x.nbytes / secs / 1e9, 4)})
                log(json.dumps(rows[-1]))
    out = {"cpu_model": _cpu_model(), "cpu_count": os.cpu_count(), "threads_all": cores,
           "how": "oracle compress + decompress per frame (F = 2^22), scalar C -O2; threads > 1 spread frames "
                  "over a host thread pool", "rows": rows}
    with open(path, "w") as f:
        json.dump(out, f, indent=1)
    return out


# ------------------------------------------------------------------------------------ reference arm
def run_reference(args, rank: int, world: int) -> dict | None:
    """The oracle as it stands on the host cores, same workload / metric / unit: each step is a
    bounded sample (the first 4 MiB of every tensor of the set): probe + select + compress +
    decompress on the CPU (there is no link to cross)."""
    if rank != 0:
        return None
    import numpy as np

    import synth
    from oracle import oracle as O
    wname, spec, dtype = workload(args.workload)
    w = synth.WIDTH[dtype]
    sample = 4 << 20
    xs = [synth.relu_iid(min(synth.numel(s), sample // w), sp, seed=synth.seed_of(3, 0, 0, i), dtype=dtype)
          for i, (_, s, sp) in enumerate(spec)]
    cal = O.make_calib(bw_d2h=50e9, bw_h2d=50e9, alpha_d2h=10e-6, alpha_h2d=10e-6)
    if os.path.exists(CALIB_PATH):
        with open(CALIB_PATH) as f:
            d = json.load(f)["calib"]
        cal = O.make_calib(alpha_d2h=d["alpha_d2h"], bw_d2h=d["bw_d2h"], alpha_h2d=d["alpha_h2d"],
                           bw_h2d=d["bw_h2d"], beta=d["beta"], lz4_gamma1=d["lz4_gamma1"],
                           lz4_gamma2=d["lz4_gamma2"], margin=d["margin"], mode=d["mode"])

    def step():
        for x in xs:
            counts = O.probe(x, dtype)
            codec = O.select(x.size, dtype, counts, 0.0, 0.0, cal)["codec"]
            blob = O.compress(x, codec, dtype)
            O.decompress(blob, x.size, dtype)

    for _ in range(args.warmup):
        step()
    t0 = time.perf_counter()
    for _ in range(args.steps):
        step()
    dt = (time.perf_counter() - t0) / args.steps
    nbytes = sum(x.nbytes for x in xs)
    value = nbytes / dt / 1e9
    return {"impl": "reference", "metric": METRIC, "value": round(value, 4), "unit": "GB/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(dt * 1e3, 3), "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "u32" if w == 4 else "u16", "data": "synthetic",
            "config": {"workload": wname, "sample": f"first {sample >> 20} MiB of each of {len(xs)} tensors"},
            "cpu_baseline": {"value": round(value, 4), "unit": "GB/s", "cores": 1, "kind": "oracle",
                             "sample": f"{nbytes >> 20} MiB per step: probe+select+compress+decompress, 1 thread"},
            "e2e": {"value": round(value, 4), "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}


def _free_port() -> int:
    import socket
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        return so.getsockname()[1]


def spawn_replicas(args, argv) -> int:
    """`python bench.py --gpus N` outside torchrun: start one rank process per GPU (same argv,
    RANK / LOCAL_RANK / WORLD_SIZE / MASTER_* in the environment) and wait for all of them.  Rank
    0 prints the one JSON line (stdout is inherited).  Asking for more GPUs than are visible is an
    error, never a silent N = 1."""
    if not args.stub and not os.environ.get("BENCH_SHARE_GPU"):
        import torch
        visible = torch.cuda.device_count()
        if args.gpus > visible:
            print(f"bench.py: --gpus {args.gpus} but only {visible} CUDA device(s) are visible", file=sys.stderr)
            return 2
    port = _free_port()
    procs = []
    for r in range(args.gpus):
        env = dict(os.environ, RANK=str(r), LOCAL_RANK=str(r), WORLD_SIZE=str(args.gpus),
                   LOCAL_WORLD_SIZE=str(args.gpus), MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        procs.append(subprocess.Popen([sys.executable, os.path.abspath(__file__), *argv], env=env))
    rcs = [p.wait() for p in procs]
    return max(rcs, key=abs)


def run_stub(args, rank: int, world: int, dist) -> dict | None:
    """CPU-only stand-in for run_ours (tests/test_multirank_cpu.py): exercises the launcher, the
    CPU barrier and the aggregation with a fake per-rank device time (rank r: 10 (r + 1) ms per
    step) and 1 MiB of 'swapped' bytes per rank."""
    raw = 1 << 20
    ms_rank = 10.0 * (rank + 1)
    if dist is not None:
        dist.barrier()
    ms_max = _max_over_ranks(ms_rank * args.steps, dist) / args.steps
    per_rank = _gather(dist, {"rank": rank, "ms_per_step": ms_rank, "pid": os.getpid(),
                              "every_compressed_tensor_faster": True})
    return {"metric": METRIC, "value": round(job_throughput(world, raw, ms_max), 6), "unit": "GB/s",
            "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_max,
            "higher_is_better": True, "scaling": "weak", "data": "stub", "per_rank": per_rank,
            "every_compressed_tensor_faster_all_ranks": all(p["every_compressed_tensor_faster"] for p in per_rank)}


def _gather(dist, obj) -> list:
    """Every rank's `obj`, in rank order (rank 0 alone: [obj])."""
    if dist is None or not dist.is_initialized():
        return [obj]
    out = [None] * dist.get_world_size()
    dist.all_gather_object(out, obj)
    return out


def main(argv=None):
    argv = sys.argv[1:] if argv is None else argv
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default="vgg16", choices=["vgg16", "resnet50", "resnet50_f16", "bert"])
    ap.add_argument("--calibrate", action="store_true", help="full calibration sweep, writes calib/b200.json")
    ap.add_argument("--no-extras", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--stub", action="store_true", help=argparse.SUPPRESS)  # CPU test of the launcher
    ap.add_argument("--swap-target", default="host", choices=["host", "peer", "self"],
                    help="where containers go (NEXT-4b): pinned host memory, the next GPU's HBM over NVLink "
                         "(rank r -> (r + 1) mod N), or this GPU's HBM")
    ap.add_argument("--cpu-plan", metavar="OUT_JSON", help="oracle timing plan of SURVEY §8(d) (CPU only)")
    args = ap.parse_args(argv)
    if args.cpu_plan:
        cpu_plan(args.cpu_plan)
        return 0
    if args.warmup < 3:
        args.warmup = 3
    if args.gpus < 1:
        print("bench.py: --gpus must be >= 1", file=sys.stderr)
        return 2
    under_launcher = "WORLD_SIZE" in os.environ
    if not under_launcher and args.gpus > 1 and args.impl == "ours":
        return spawn_replicas(args, argv)
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if os.environ.get("BENCH_SHARE_GPU"):
        # functional test of the N-rank path on a box with fewer GPUs: every rank on GPU 0
        # (the numbers are then not a scaling measurement)
        local_rank = 0
    if args.impl == "reference":
        res = run_reference(args, rank, world)
        if res is not None:
            print(json.dumps(res), flush=True)
        return 0
    if world != args.gpus:
        print(f"bench.py: --gpus {args.gpus} but the launcher started {world} rank(s)", file=sys.stderr)
        return 2
    dist = None
    if world > 1:
        import torch.distributed as tdist
        # replicas only: a CPU (gloo) group for the barrier and the MAX / gather of per-rank
        # numbers; nothing on the data path crosses GPUs (no NCCL)
        tdist.init_process_group("gloo")
        dist = tdist
    res = run_stub(args, rank, world, dist) if args.stub else run_ours(args, rank, world, local_rank, dist)
    if rank == 0 and res is not None:
        print(json.dumps(res), flush=True)
    if dist is not None:
        dist.barrier()
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
