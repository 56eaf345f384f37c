"""Online re-profiling under sparsity drift (analogue of PAPER.md Figs. 8-9,
:283-295): a torchvision VGG16 (random init, synthetic inputs, batch 64) whose conv biases are moved
each "epoch" so that every ReLU output reaches a target sparsity (bias = -sigma * Phi^-1(s) from the
layer's measured pre-activation std).  Two CSWAP savers run side by side on the same epochs:
  reprofiled  probes + decides on the first step of every epoch (reprofile_every = steps/epoch),
  static      keeps the plan decided in epoch 0.
Per epoch: target sparsity, codecs chosen, compressed-tensor count, ms per step of each saver.

    python tools/drift.py [--batch 64] [--steps 4] [--targets 0.02,0.1,0.2,0.35,0.5,0.65,0.8]

Each epoch: one profiling step of the re-profiling saver, one untimed replay step of each saver
(first use of a codec at a size grows scratch / instantiates graphs), then `--steps` timed steps
of each.  The bias recipe drives deep layers harder than the target (their inputs shift too), so
the measured mean sparsity of the ReLU outputs and the count of all-zero ones are reported.
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--batch", type=int, default=64)
    ap.add_argument("--steps", type=int, default=4)
    ap.add_argument("--targets", default="0.02,0.1,0.2,0.35,0.5,0.65,0.8")
    a = ap.parse_args()
    import torch
    import torchvision

    from paper_conf_cluster_chenhzchysc21_b200.swap_hooks import SwapSaver
    torch.manual_seed(0)
    model = torchvision.models.vgg16(weights=None).cuda()
    x = torch.randn(a.batch, 3, 224, 224, device="cuda")
    y = torch.randint(0, 1000, (a.batch,), device="cuda")
    convs = [m for m in model.features if isinstance(m, torch.nn.Conv2d)]
    # pre-activation std of every conv with zero bias (one forward)
    sig = {}
    for c in convs:
        c.bias.data.zero_()
    hooks = [c.register_forward_hook(lambda m, i, o: sig.__setitem__(m, float(o.float().std()))) for c in convs]
    with torch.no_grad():
        model(x)
    for h in hooks:
        h.remove()

    def set_sparsity(s):
        q = statistics.NormalDist().inv_cdf(s)
        for c in convs:
            c.bias.data.fill_(-sig[c] * q)

    def step(saver):
        model.zero_grad(set_to_none=True)
        with saver:
            loss = torch.nn.functional.cross_entropy(model(x), y)
        loss.backward()

    def timed(saver, n):
        per = []
        for _ in range(n):
            e = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
            model.zero_grad(set_to_none=True)
            e[0].record()
            with saver:
                loss = torch.nn.functional.cross_entropy(model(x), y)
            e[1].record()
            loss.backward()
            e[2].record()
            e[2].synchronize()
            per.append((round(e[0].elapsed_time(e[1]), 2), round(e[1].elapsed_time(e[2]), 2)))
        timed.last = per
        return sum(a + b for a, b in per) / n

    relus = [m for m in model.features if isinstance(m, torch.nn.ReLU)]
    zf = []

    def measured_sparsity():
        zf.clear()
        hk = [r.register_forward_hook(lambda m, i, o: zf.append(float((o == 0).float().mean()))) for r in relus]
        with torch.no_grad():
            model(x)
        for h in hk:
            h.remove()
        return round(sum(zf) / len(zf), 3), sum(1 for z in zf if z == 1.0)

    re = SwapSaver("auto", reprofile_every=10**9)
    st = SwapSaver("auto", reprofile_every=10**9)
    rows = []
    for e, s in enumerate(float(v) for v in a.targets.split(",")):
        set_sparsity(s)
        sp, dead = measured_sparsity()
        torch.cuda.synchronize()
        re.plan = None    # the first step of every epoch re-profiles (probe + decide per tensor)
        step(re)
        step(re)          # untimed replay
        step(st)          # st: profiles once (epoch 0), then replays that plan
        step(st)
        ms_re = timed(re, a.steps)
        per_re = timed.last
        ms_st = timed(st, a.steps)
        per_st = timed.last
        plan = re.plan or []
        row = {"epoch": e, "target_sparsity": s, "relu_sparsity_mean": sp, "relu_all_zero": dead,
               "codecs_reprofiled": plan,
               "compressed_reprofiled": sum(1 for c in plan if c != 0),
               "compressed_static": sum(1 for c in (st.plan or []) if c != 0), "tensors": len(plan),
               "ms_step_reprofiled": round(ms_re, 2), "ms_step_static": round(ms_st, 2),
               "host_MiB_reprofiled": round(re.stats["comp_bytes"] / 2**20, 1),
               "host_MiB_static": round(st.stats["comp_bytes"] / 2**20, 1),
               "fwd_bwd_ms_reprofiled": per_re, "fwd_bwd_ms_static": per_st}
        rows.append(row)
        print(json.dumps(row), flush=True)


if __name__ == "__main__":
    main()
