"""On-box calibration of the cost model.

PAPER.md:118 (§IV-A): the profiler measures the *effective* PCIe bandwidth, "We did not use the
name-tag bandwidth number"; PAPER.md:164-168 (§IV-C): (de)compression time is modelled by linear
regression on tensor size and sparsity, with sub-models per sparsity band; PAPER.md:265 uses
NVIDIA bandwidthTest for the link.  This module only orchestrates microbenchmarks (CUDA events on
the launching stream) and calls the library's fits (cswap_fit_link / cswap_fit_time_model /
cswap_fit_linear, C++).  The result is a cswap_calib installed with cswap_set_calibration and
saved as JSON (calib/b200.json).
"""
from __future__ import annotations

import json
import os
import time

from . import cswap as C

BANDS = [(0.0, 0.2), (0.2, 0.35), (0.35, 0.5), (0.5, 0.65), (0.65, 0.8), (0.8, 1.0)]
BAND_POINTS = [(0.05, 0.15), (0.22, 0.32), (0.38, 0.47), (0.52, 0.62), (0.68, 0.77), (0.85, 0.97)]
MIB = 1 << 20


def _events():
    import torch
    return torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)


def time_ms(fn, reps: int) -> float:
    """Median CUDA-event time of fn() on the current stream (after one warm-up)."""
    import torch
    fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        a, b = _events()
        a.record()
        fn()
        b.record()
        b.synchronize()
        ts.append(a.elapsed_time(b))
    ts.sort()
    return ts[len(ts) // 2]


def link_sweep(sizes=None, reps: int = 5) -> dict:
    """Pinned-host <-> device cudaMemcpyAsync per direction (bandwidthTest-style)."""
    import torch
    sizes = sizes or [1 << k for k in range(16, 31, 2)]  # 64 KiB .. 1 GiB
    host = torch.empty(max(sizes), dtype=torch.uint8).pin_memory()
    dev = torch.empty(max(sizes), dtype=torch.uint8, device="cuda")
    out = {"sizes": sizes, "d2h_ms": [], "h2d_ms": []}
    for b in sizes:
        out["d2h_ms"].append(time_ms(lambda: host[:b].copy_(dev[:b], non_blocking=True), reps))
        out["h2d_ms"].append(time_ms(lambda: dev[:b].copy_(host[:b], non_blocking=True), reps))
    for d in ("d2h", "h2d"):
        a, bw = C.fit_link([float(s) for s in sizes], [t * 1e-3 for t in out[d + "_ms"]])
        out[d] = {"alpha_s": a, "bw_Bps": bw, "peak_GBps": max(s / (t * 1e-3) for s, t in zip(sizes, out[d + "_ms"])) / 1e9}
    del host, dev
    return out


def codec_sweep(codecs, sizes_mib, dtype=C.F32, reps: int = 3, fmt=None, log=None) -> list:
    """Device->device compress / decompress times of synthetic iid ReLU tensors."""
    import torch
    import synth
    w = C.WIDTH[dtype]
    samples = []
    maxn = max(sizes_mib) * MIB // w
    src = torch.empty(maxn, dtype=torch.int32 if w == 4 else torch.int16, device="cuda")
    dst = torch.empty_like(src)
    size = torch.zeros(1, dtype=torch.int64, device="cuda")
    err = torch.zeros(1, dtype=torch.int32, device="cuda")
    for bi, pts in enumerate(BAND_POINTS):
        for si, s in enumerate(pts):
            x = synth.relu_iid_torch(maxn, s, seed=synth.seed_of(2, bi, si), dtype=dtype, device="cuda")
            src.copy_(x)
            del x
            for mib in sizes_mib:
                n = mib * MIB // w
                probe = C.probe(src, n, dtype)
                for codec in codecs:
                    cap = C.max_compressed_size(n, dtype, codec, fmt)
                    buf = torch.empty(cap, dtype=torch.uint8, device="cuda")
                    tc = time_ms(lambda: C.compress(src, n, dtype, codec, buf, cap, size, fmt=fmt), reps)
                    torch.cuda.synchronize()
                    nbytes = int(size.item())
                    tdc = time_ms(lambda: C.decompress(buf, nbytes, dst, n, dtype, codec, fmt=fmt, err=err), reps)
                    samples.append({"codec": codec, "S": n * w, "s": probe.zeros / probe.samples, "true_s": s,
                                    "band": bi, "t_c": tc * 1e-3, "t_dc": tdc * 1e-3, "bytes": nbytes,
                                    "probe": list(probe.tuple()), "n": n})
                    if log:
                        log(f"  codec={C.CODEC_NAMES[codec]} S={mib}MiB s={s:.2f} c={tc:.3f}ms dc={tdc:.3f}ms "
                            f"ratio={nbytes / (n * w):.3f}")
                    del buf
    return samples


def fit(link: dict, samples: list, codecs, frame_elems=1 << 22) -> tuple:
    """Returns (cswap.Calib, report)."""
    cal = C.get_calibration()
    cal.alpha_d2h, cal.bw_d2h = max(link["d2h"]["alpha_s"], 0.0), link["d2h"]["bw_Bps"]
    cal.alpha_h2d, cal.bw_h2d = max(link["h2d"]["alpha_s"], 0.0), link["h2d"]["bw_Bps"]
    report = {"rae": {}}
    for ci in range(4):
        codec = ci + 1
        for d, key in ((0, "t_c"), (1, "t_dc")):
            for b in range(6):
                base = ((ci * 2 + d) * 6 + b) * 3
                pts = [p for p in samples if p["codec"] == codec and p["band"] == b]
                if codec not in codecs or len(pts) < 3:
                    if codec not in codecs:  # not built: make it never win
                        cal.beta[base], cal.beta[base + 1], cal.beta[base + 2] = 1e3, 0.0, 0.0
                    continue
                try:
                    beta = C.fit_time_model([p["S"] for p in pts], [p["s"] for p in pts], [p[key] for p in pts])
                except C.CswapError:  # single sparsity in band: fall back to [1, S]
                    beta = C.fit_linear([[1.0, float(p["S"])] for p in pts], [p[key] for p in pts]) + [0.0]
                for i in range(3):
                    cal.beta[base + i] = beta[i]
            pts = [p for p in samples if p["codec"] == codec]
            if pts:
                pred = []
                for p in pts:
                    base = ((ci * 2 + d) * 6 + p["band"]) * 3
                    pred.append(cal.beta[base] + cal.beta[base + 1] * p["S"] + cal.beta[base + 2] * p["S"] * p["s"])
                y = [p[key] for p in pts]
                mean = sum(y) / len(y)
                rae = sum(abs(a - b) for a, b in zip(pred, y)) / max(sum(abs(mean - b) for b in y), 1e-30)
                report["rae"][f"{C.CODEC_NAMES[codec]}_{'c' if d == 0 else 'dc'}"] = rae
    # LZ4 size model: bytes - header - w*nnz_hat = g1 * zero_runs_hat + g2 * w * zeros_hat / 255
    lz = [p for p in samples if p["codec"] == C.LZ4]
    if len(lz) >= 3:
        rows, ys = [], []
        for p in lz:
            z, zr, bd, sm, pr = p["probe"]
            n, w = p["n"], p["S"] // p["n"]
            zeros_hat = (z * n + sm // 2) // sm
            zr_hat = (zr * n + sm // 2) // sm
            K = -(-n // frame_elems)
            hdr = (64 + 8 * K + 15) // 16 * 16 + K * 16
            rows.append([float(zr_hat), w * zeros_hat / 255.0])
            ys.append(p["bytes"] - hdr - w * (n - zeros_hat))
        try:
            g = C.fit_linear(rows, ys)
            cal.lz4_gamma1, cal.lz4_gamma2 = g
        except C.CswapError:
            pass
    report["link"] = {k: link[k] for k in ("d2h", "h2d")}
    return cal, report


def calib_to_json(cal) -> dict:
    d = {}
    for f, _ in C.Calib._fields_:
        v = getattr(cal, f)
        d[f] = list(v) if f == "beta" else v
    return d


def calib_from_json(d: dict):
    cal = C.Calib()
    for f, _ in C.Calib._fields_:
        if f == "beta":
            for i, v in enumerate(d["beta"]):
                cal.beta[i] = v
        elif f in d:
            setattr(cal, f, d[f])
    if "group_bytes" not in d:  # calibrations written before the swap-in group size existed
        cal.group_bytes = float(32 << 20)
    return cal


def run(codecs, quick: bool = False, path: str | None = None, log=print) -> dict:
    t0 = time.time()
    link = link_sweep(reps=3 if quick else 5)
    log(f"link d2h {link['d2h']['bw_Bps'] / 1e9:.1f} GB/s alpha {link['d2h']['alpha_s'] * 1e6:.1f} us; "
        f"h2d {link['h2d']['bw_Bps'] / 1e9:.1f} GB/s alpha {link['h2d']['alpha_s'] * 1e6:.1f} us")
    sizes = [1, 8, 64] if quick else [1, 4, 16, 64, 256]
    samples = codec_sweep(codecs, sizes, reps=3, log=log if not quick else None)
    cal, report = fit(link, samples, codecs)
    C.set_calibration(cal)
    out = {"calib": calib_to_json(cal), "report": report, "samples": samples, "codecs": list(codecs),
           "seconds": time.time() - t0, "when": time.strftime("%Y-%m-%dT%H:%M:%SZ", time.gmtime())}
    if path:
        os.makedirs(os.path.dirname(path), exist_ok=True)
        with open(path, "w") as f:
            json.dump(out, f, indent=1)
    return out


def load(path: str) -> bool:
    if not os.path.exists(path):
        return False
    with open(path) as f:
        d = json.load(f)
    C.set_calibration(calib_from_json(d["calib"]))
    return True
