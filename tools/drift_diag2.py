"""Epoch-5 anomaly of tools/drift.py: time forward / backward of VGG16 steps at one drift point
replaying (a) the re-profiled plan, (b) it with RLE -> ZVC, (c) with RLE -> CSR, (d) all ZVC."""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    import torchvision

    from paper_conf_cluster_chenhzchysc21_b200.swap_hooks import SwapSaver
    target = float(sys.argv[1]) if len(sys.argv) > 1 else 0.65
    torch.manual_seed(0)
    model = torchvision.models.vgg16(weights=None).cuda()
    x = torch.randn(64, 3, 224, 224, device="cuda")
    y = torch.randint(0, 1000, (64,), device="cuda")
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

    def step(saver):
        e = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
        model.zero_grad(set_to_none=True)
        e[0].record()
        with saver:
            loss = torch.nn.functional.cross_entropy(model(x), y)
        e[1].record()
        loss.backward()
        e[2].record()
        e[2].synchronize()
        return e[0].elapsed_time(e[1]), e[1].elapsed_time(e[2])

    re = SwapSaver("auto", reprofile_every=10**9)
    step(re)
    plan = list(re.plan)
    sizes = []
    for alt in ("plan", "rle->zvc", "rle->csr", "all zvc"):
        p = list(plan)
        if alt == "rle->zvc":
            p = [1 if c == 2 else c for c in p]
        elif alt == "rle->csr":
            p = [3 if c == 2 else c for c in p]
        elif alt == "all zvc":
            p = [1 for _ in p]
        re.plan = p
        step(re)
        fb = [step(re) for _ in range(3)]
        print(json.dumps({"variant": alt, "plan": "".join(map(str, p)),
                          "fwd_ms": [round(a, 2) for a, _ in fb], "bwd_ms": [round(b, 2) for _, b in fb],
                          "host_MiB": round(re.stats["comp_bytes"] / 2**20, 1)}), flush=True)
        if alt == "plan":
            sizes = [(r.index, r.codec, round(r.nbytes / 2**20, 1), round(r.comp_bytes / 2**20, 2)) for r in re._order]
    print(json.dumps({"tensors": sizes}))


if __name__ == "__main__":
    main()
