"""Codec microbenchmark (BASELINE.json configs[1] points): device->device compress / decompress
GB/s of algorithmic bytes vs the measured HBM peak, L2 flushed between reps.

    python tools/codec_bench.py [--codecs zvc,rle,csr,lz4] [--mib 1024] [--s 0.5] [--reps 10]
                                [--dtype f32] [--ncu]   (ncu: 2 warm launches + 1 profiled each)
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--codecs", default="zvc")
    ap.add_argument("--mib", type=float, default=1024, help="tensor size in MiB (fractions allowed: 0.0625 = 64 KiB)")
    ap.add_argument("--s", default="0.5")
    ap.add_argument("--reps", type=int, default=10)
    ap.add_argument("--dtype", default="f32")
    ap.add_argument("--kind", default="iid", choices=["iid", "clustered", "clustered32", "dead", "zero", "dense"],
                    help="zero placement (DESIGN.md §5): iid, clustered runs (mean zero run 256 / 32), "
                         "channel-dead planes, all-zero, dense")
    ap.add_argument("--ncu", action="store_true")
    ap.add_argument("--check", action="store_true", help="verify round trip")
    ap.add_argument("--variant", type=int, default=-1, help="ZVC compress geometry (cswap_set_zvc_launch)")
    ap.add_argument("--grid", type=int, default=0, help="ZVC compress grid (0 = automatic)")
    a = ap.parse_args()
    import torch

    import synth
    from paper_conf_cluster_chenhzchysc21_b200 import cswap as C
    C.init(0)
    C.set_zvc_launch(a.grid, a.variant)
    sys.path.insert(0, ROOT)
    from bench import ClockSampler
    sampler = ClockSampler(0).__enter__()  # SM clock + throttle reasons under load (DESIGN §6 tables)
    names = {"none": C.NONE, "zvc": C.ZVC, "rle": C.RLE, "csr": C.CSR, "lz4": C.LZ4}
    dtype = {"f32": C.F32, "f16": C.F16, "bf16": C.BF16}[a.dtype]
    w = C.WIDTH[dtype]
    n = int(a.mib * 2**20) // w
    peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"] if os.path.exists(
        os.path.join(ROOT, "MEASURED_PEAKS.json")) else 6650.0
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    out = []
    for s in [float(v) for v in a.s.split(",")]:
        import numpy as np
        if a.kind == "iid":
            x = synth.relu_iid_torch(n, s, seed=123, dtype=dtype, device="cuda")
        elif a.kind == "dense":
            x = synth.relu_iid_torch(n, 0.0, seed=123, dtype=dtype, device="cuda")
        elif a.kind == "zero":
            x = torch.zeros(n, dtype=torch.int32 if w == 4 else torch.int16, device="cuda")
        elif a.kind == "dead":  # whole 56x56 planes of 64-channel images zero for a fraction s of the channels
            hw = 56 * 56
            h = synth.channel_dead((n // (64 * hw) + 1, 64, 56, 56), s, seed=7, dtype=dtype).reshape(-1)[:n]
            x = torch.from_numpy(np.ascontiguousarray(h).view(np.int32 if w == 4 else np.int16)).cuda()
        else:
            h = synth.relu_clustered(n, s, 256 if a.kind == "clustered" else 32, seed=5, dtype=dtype)
            x = torch.from_numpy(h.view(np.int32 if w == 4 else np.int16)).cuda()
        y = torch.empty_like(x)
        size = torch.zeros(1, dtype=torch.int64, device="cuda")
        err = torch.zeros(1, dtype=torch.int32, device="cuda")
        for cname in a.codecs.split(","):
            codec = names[cname]
            cap = C.max_compressed_size(n, dtype, codec)
            buf = torch.empty(cap, dtype=torch.uint8, device="cuda")
            reps = 1 if a.ncu else a.reps
            warm = 2

            def comp():
                C.compress(x, n, dtype, codec, buf, cap, size)

            def decomp(nb):
                C.decompress(buf, nb, y, n, dtype, codec, err=err)

            res = {"codec": cname, "s": s, "MiB": a.mib, "dtype": a.dtype, "kind": a.kind,
                   "variant": a.variant, "grid": a.grid}
            for label, fn in (("compress", comp), ("decompress", None)):
                if fn is None:
                    nb = int(size.item())
                    fn = lambda: decomp(nb)  # noqa: E731
                for _ in range(warm):
                    fn()
                torch.cuda.synchronize()
                ts = []
                for _ in range(reps):
                    flush.fill_(1)
                    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    ev0.record()
                    fn()
                    ev1.record()
                    ev1.synchronize()
                    ts.append(ev0.elapsed_time(ev1))
                ts.sort()
                ms = ts[len(ts) // 2]
                nb = int(size.item())
                alg = n * w + nb
                res[label] = {"ms": round(ms, 4), "GBps": round(alg / (ms * 1e-3) / 1e9, 1),
                              "frac": round(alg / (ms * 1e-3) / 1e9 / peak, 4),
                              "raw_GBps": round(n * w / (ms * 1e-3) / 1e9, 1)}
            res["ratio"] = round(int(size.item()) / (n * w), 4)
            if a.check:
                torch.cuda.synchronize()
                res["roundtrip_ok"] = bool(torch.equal(x, y)) and int(err.item()) == 0
            out.append(res)
            print(json.dumps(res), flush=True)
            del buf
    sampler.__exit__(None, None, None)
    print(json.dumps({"clocks": sampler.summary()}), flush=True)
    return out


if __name__ == "__main__":
    main()
