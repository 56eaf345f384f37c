"""Per-tensor selector diagnosis at one drift point (tools/drift.py): for each activation VGG16
saves at a target sparsity, the probe's sparsity / run fraction, the selector's predicted
t_c / t_dc / size per codec, and the measured device times and sizes per codec."""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    import torchvision

    from paper_conf_cluster_chenhzchysc21_b200 import calibrate, cswap as C
    target = float(sys.argv[1]) if len(sys.argv) > 1 else 0.65
    C.init(0)
    calibrate.load(os.path.join(ROOT, "calib", "b200.json"))
    torch.manual_seed(0)
    model = torchvision.models.vgg16(weights=None).cuda()
    x = torch.randn(64, 3, 224, 224, device="cuda")
    convs = [m for m in model.features if isinstance(m, torch.nn.Conv2d)]
    sig = {}
    for c in convs:
        c.bias.data.zero_()
    hs = [c.register_forward_hook(lambda m, i, o: sig.__setitem__(m, float(o.float().std()))) for c in convs]
    with torch.no_grad():
        model(x)
    for h in hs:
        h.remove()
    q = statistics.NormalDist().inv_cdf(target)
    for c in convs:
        c.bias.data.fill_(-sig[c] * q)
    saved = []
    seen = set()

    def pack(t):
        if t.dtype == torch.float32 and t.numel() * 4 >= 1 << 20 and t.data_ptr() not in seen:
            seen.add(t.data_ptr())
            saved.append(t.detach().clone())
        return t
    with torch.autograd.graph.saved_tensors_hooks(pack, lambda t: t):
        model(x)
    size = torch.zeros(1, dtype=torch.int64, device="cuda")
    err = torch.zeros(1, dtype=torch.int32, device="cuda")
    for i, t in enumerate(saved):
        n = t.numel()
        p = C.probe(t, n, C.F32)
        d = C.select_from_probe(n, C.F32, p)
        row = {"i": i, "MiB": round(n * 4 / 2**20, 1), "s_probe": round(p.zeros / p.samples, 3),
               "s_true": round(float((t == 0).float().mean()), 3),
               "runs_frac_probe": round(p.boundaries / max(p.pairs, 1), 3), "chosen": d.codec,
               "pred_ms": {}, "meas_ms": {}, "pred_MiB": {}, "meas_MiB": {}}
        y = torch.empty_like(t)
        for codec in (1, 2, 3, 4):
            cap = C.max_compressed_size(n, C.F32, codec)
            buf = torch.empty(cap, dtype=torch.uint8, device="cuda")
            tc = calibrate.time_ms(lambda: C.compress(t, n, C.F32, codec, buf, cap, size), 3)
            torch.cuda.synchronize()
            nb = int(size.item())
            tdc = calibrate.time_ms(lambda: C.decompress(buf, nb, y, n, C.F32, codec, err=err), 3)
            row["pred_ms"][codec] = [round(d.t_c[codec - 1] * 1e3, 3), round(d.t_dc[codec - 1] * 1e3, 3)]
            row["meas_ms"][codec] = [round(tc, 3), round(tdc, 3)]
            row["pred_MiB"][codec] = round(d.size[codec - 1] / 2**20, 1)
            row["meas_MiB"][codec] = round(nb / 2**20, 1)
        print(json.dumps(row), flush=True)


if __name__ == "__main__":
    main()
