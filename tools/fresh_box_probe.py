"""Does host-link throughput ramp up on a freshly acquired box?

The first bench.py run on a fresh box showed per-step times falling from 61 to 45.5 ms over its
20 timed steps, while later runs on the same box were flat at 45.5 ms.  This probe separates the
link from the library: it pins 2 x 1 GiB (torch pinned tensors, no libcswap), then alternates
784 MiB D2H and H2D copies for `--seconds`, printing the rate of every copy with its time since
start, plus the host's load average and free memory at the start and at the end.
"""
import argparse
import json
import os
import time

import torch


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--seconds", type=float, default=6.0)
    ap.add_argument("--mib", type=int, default=784)
    a = ap.parse_args()
    nb = a.mib << 20
    t_start = time.time()
    dev = torch.empty(nb, dtype=torch.uint8, device="cuda")
    dev.fill_(1)
    h1 = torch.empty(nb, dtype=torch.uint8, pin_memory=True)
    h2 = torch.empty(nb, dtype=torch.uint8, pin_memory=True)
    h2.fill_(2)
    print(json.dumps({"pin_s": round(time.time() - t_start, 3), "loadavg": os.getloadavg()}), flush=True)
    torch.cuda.synchronize()
    t0 = time.time()
    rows = []
    while time.time() - t0 < a.seconds:
        for name, fn in (("d2h", lambda: h1.copy_(dev, non_blocking=True)),
                         ("h2d", lambda: dev.copy_(h2, non_blocking=True))):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            fn()
            e1.record()
            e1.synchronize()
            ms = e0.elapsed_time(e1)
            rows.append({"t_s": round(time.time() - t0, 3), "dir": name, "GBps": round(nb / ms / 1e6, 2)})
    for r in rows:
        print(json.dumps(r))
    d2h = [r["GBps"] for r in rows if r["dir"] == "d2h"]
    h2d = [r["GBps"] for r in rows if r["dir"] == "h2d"]
    print(json.dumps({"d2h_first5": d2h[:5], "d2h_last5": d2h[-5:], "h2d_first5": h2d[:5], "h2d_last5": h2d[-5:],
                      "loadavg_end": os.getloadavg()}))


if __name__ == "__main__":
    main()
