"""Does a second saver interleaved with the first change its step time?  VGG16 at one drift
point: (A) re-profiling saver alone, (B) interleaved with a static-plan saver, (C) both plans
forced to the same RLE-heavy plan."""
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

    def setp(s):
        q = statistics.NormalDist().inv_cdf(s)
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
        return round(e[0].elapsed_time(e[1]), 2), round(e[1].elapsed_time(e[2]), 2)

    setp(0.02)
    st = SwapSaver("auto", reprofile_every=10**9)
    step(st)  # static plan from "epoch 0"
    setp(target)
    re = SwapSaver("auto", reprofile_every=10**9)
    step(re)
    print(json.dumps({"plan_re": "".join(map(str, re.plan)), "plan_st": "".join(map(str, st.plan))}))
    print(json.dumps({"A_re_alone": [step(re) for _ in range(4)]}), flush=True)
    print(json.dumps({"A_st_alone": [step(st) for _ in range(4)]}), flush=True)
    out = []
    for _ in range(3):
        out.append(("re", step(re)))
        out.append(("st", step(st)))
    print(json.dumps({"B_interleaved": out}), flush=True)
    print(json.dumps({"A_re_again": [step(re) for _ in range(4)]}), flush=True)


if __name__ == "__main__":
    main()
