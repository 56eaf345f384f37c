"""Training-step analogue of PAPER.md Fig. 6 / Fig. 7 (§V-A/B) on one B200: a torchvision VGG16
(random init, synthetic 224x224 inputs, SGD) whose saved activations are swapped through libcswap
under each policy — resident (no swapping), vDNN (raw offload), SC (always ZVC), CSWAP (AUTO with
profiled Hidden_f / Hidden_b) — reporting ms per iteration, peak HBM and swapped bytes.  Gradients
of the swapped runs are checked bitwise against the resident run (deterministic cuDNN).

    python tools/train_step.py [--model vgg16|resnet50] [--batch 64] [--iters 5] [--dtype f32|bf16]
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--model", default="vgg16")
    ap.add_argument("--batch", type=int, default=64)
    ap.add_argument("--iters", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=2)
    ap.add_argument("--dtype", default="f32")
    ap.add_argument("--min-mib", type=float, default=1.0)
    ap.add_argument("--policies", default="resident,none,zvc,auto")
    a = ap.parse_args()
    import torch
    import torchvision

    from paper_conf_cluster_chenhzchysc21_b200.swap_hooks import SwapSaver
    torch.backends.cudnn.deterministic = True
    torch.backends.cudnn.benchmark = False
    dtype = {"f32": torch.float32, "bf16": torch.bfloat16, "f16": torch.float16}[a.dtype]
    torch.manual_seed(0)
    model = getattr(torchvision.models, a.model)(weights=None).cuda().to(dtype)
    opt = torch.optim.SGD(model.parameters(), lr=1e-3)
    x = torch.randn(a.batch, 3, 224, 224, device="cuda", dtype=dtype)
    y = torch.randint(0, 1000, (a.batch,), device="cuda")
    init = {k: v.clone() for k, v in model.state_dict().items()}

    after_fwd, fwd_peak = [], []

    def fwd_bwd(saver, mark=None):
        torch.manual_seed(1)  # same dropout masks in every run (bitwise gradient comparison)
        opt.zero_grad(set_to_none=True)
        if saver is None:
            loss = torch.nn.functional.cross_entropy(model(x).float(), y)
        else:
            with saver:
                loss = torch.nn.functional.cross_entropy(model(x).float(), y)
        if mark:
            mark()
        after_fwd.append(torch.cuda.memory_allocated())
        fwd_peak.append(torch.cuda.max_memory_allocated())
        loss.backward()
        return loss

    def grads_of(saver):
        model.load_state_dict(init)
        fwd_bwd(saver)
        torch.cuda.synchronize()
        return [p.grad.clone() for p in model.parameters()]

    ref = grads_of(None)
    rows = []
    for pol in a.policies.split(","):
        saver = None if pol == "resident" else SwapSaver(pol, min_bytes=int(a.min_mib * 2**20))
        if saver is not None and pol == "auto":
            model.load_state_dict(init)
            saver.profile(lambda mark: fwd_bwd(None, mark))
        got = grads_of(saver)
        exact = all(torch.equal(g, r) for g, r in zip(got, ref))
        model.load_state_dict(init)
        for _ in range(a.warmup):
            fwd_bwd(saver)
            opt.step()
        torch.cuda.synchronize()
        torch.cuda.reset_peak_memory_stats()
        after_fwd.clear()
        fwd_peak.clear()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        t0 = time.perf_counter()
        e0.record()
        for _ in range(a.iters):
            fwd_bwd(saver)
            opt.step()
        e1.record()
        e1.synchronize()
        wall = (time.perf_counter() - t0) / a.iters * 1e3
        ms = e0.elapsed_time(e1) / a.iters
        row = {"policy": pol, "ms_per_iter": round(ms, 2), "wall_ms_per_iter": round(wall, 2),
               "peak_GiB": round(torch.cuda.max_memory_allocated() / 2**30, 2),
               "after_fwd_GiB": round(max(after_fwd) / 2**30, 2),
               "fwd_peak_GiB": round(fwd_peak[0] / 2**30, 2), "grads_bitwise_equal": exact}
        if saver is not None:
            st = saver.stats
            row.update({"swapped_tensors": st["swapped"], "raw_MiB": round(st["raw_bytes"] / 2**20, 1),
                        "host_MiB": round(st["comp_bytes"] / 2**20, 1),
                        "codecs": {c: st["codecs"].count(c) for c in sorted(set(st["codecs"]))}})
            if saver.hidden:
                row["hidden_ms_sum"] = [round(sum(h[0] for h in saver.hidden) * 1e3, 2),
                                        round(sum(h[1] for h in saver.hidden) * 1e3, 2)]
        rows.append(row)
        print(json.dumps(row), flush=True)
    base = {r["policy"]: r["ms_per_iter"] for r in rows}
    if "none" in base and "auto" in base:
        print(json.dumps({"model": a.model, "batch": a.batch, "dtype": a.dtype,
                          "auto_vs_vdnn_time_reduction": round(1 - base["auto"] / base["none"], 4),
                          "auto_overhead_vs_resident": round(base["auto"] / base.get("resident", base["auto"]) - 1, 4)
                          if "resident" in base else None}))


if __name__ == "__main__":
    main()
