"""How much of a small codec call's event time is host-side launch work?

For each size: the host time of one cswap_compress / cswap_decompress call (perf_counter around
the call, the device idle before it), the CUDA-event time around the call as tools/codec_bench.py
measures it, the same with the device kept busy by a queued 200 us spin kernel before the
events (host enqueue work then overlaps device time and drops out of the event time), and the
kernel-timing records of the library (events right before the graph launch; stamp-kernel device
clock).  ZVC f32 / f16 at s = 0.5.
"""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch

    import synth
    from paper_conf_cluster_chenhzchysc21_b200 import cswap as C
    C.init(0)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    for dname, dtype in (("f32", C.F32), ("f16", C.F16)):
        w = C.WIDTH[dtype]
        for mib in (1, 16, 24, 96, 256):
            n = (mib << 20) // w
            x = synth.relu_iid_torch(n, 0.5, seed=123, dtype=dtype, device="cuda")
            y = torch.empty_like(x)
            cap = C.max_compressed_size(n, dtype, C.ZVC)
            buf = torch.empty(cap, dtype=torch.uint8, device="cuda")
            size = torch.zeros(1, dtype=torch.int64, device="cuda")
            err = torch.zeros(1, dtype=torch.int32, device="cuda")
            C.compress(x, n, dtype, C.ZVC, buf, cap, size)
            torch.cuda.synchronize()
            nb = int(size.item())
            calls = {"compress": lambda: C.compress(x, n, dtype, C.ZVC, buf, cap, size),
                     "decompress": lambda: C.decompress(buf, nb, y, n, dtype, C.ZVC, err=err)}
            row = {"dtype": dname, "MiB": mib}
            for name, fn in calls.items():
                for _ in range(3):
                    fn()
                host, ev_idle, ev_busy, rec_ev, rec_dev = [], [], [], [], []
                for rep in range(10):
                    flush.fill_(1)
                    torch.cuda.synchronize()
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record()
                    t0 = time.perf_counter()
                    fn()
                    host.append((time.perf_counter() - t0) * 1e6)
                    e1.record()
                    e1.synchronize()
                    ev_idle.append(e0.elapsed_time(e1) * 1e3)
                    # the device busy before the events: host work overlaps
                    flush.fill_(1)
                    torch.cuda.synchronize()
                    torch.cuda._sleep(400_000)  # ~200 us of device time
                    e0.record()
                    C.collect_kernel_timing()
                    C.set_kernel_timing(True)
                    fn()
                    C.set_kernel_timing(False)
                    e1.record()
                    e1.synchronize()
                    ev_busy.append(e0.elapsed_time(e1) * 1e3)
                    recs = C.collect_kernel_timing()
                    if recs:
                        rec_ev.append(recs[-1]["ms"] * 1e3)
                        rec_dev.append(recs[-1]["device_ms"] * 1e3)
                med = lambda v: round(sorted(v)[len(v) // 2], 1) if v else None  # noqa: E731
                row[name] = {"host_us": med(host), "events_device_idle_us": med(ev_idle),
                             "events_device_busy_us": med(ev_busy), "lib_events_us": med(rec_ev),
                             "lib_device_clock_us": med(rec_dev)}
            print(json.dumps(row), flush=True)


if __name__ == "__main__":
    main()
