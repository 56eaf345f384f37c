"""Training integration on the GPU: a small conv net's loss and every
parameter gradient are bitwise identical with activations swapped through libcswap — for each
forced codec, the vDNN / SC / CSWAP policies, with and without prefetch — to the run that keeps
every activation resident (the swap path is lossless; deterministic cuDNN)."""
import pytest

pytestmark = pytest.mark.gpu


def _net(torch, dtype):
    torch.manual_seed(0)
    m = torch.nn.Sequential(
        torch.nn.Conv2d(3, 32, 3, padding=1), torch.nn.ReLU(inplace=True), torch.nn.MaxPool2d(2),
        torch.nn.Conv2d(32, 64, 3, padding=1), torch.nn.ReLU(inplace=True),
        torch.nn.Conv2d(64, 64, 3, padding=1), torch.nn.ReLU(inplace=True), torch.nn.MaxPool2d(2),
        torch.nn.Flatten(), torch.nn.Linear(64 * 16 * 16, 10))
    return m.cuda().to(dtype)


def _step(torch, m, x, saver):
    m.zero_grad(set_to_none=True)
    if saver is None:
        loss = m(x).float().square().sum()
    else:
        with saver:
            loss = m(x).float().square().sum()
    loss.backward()
    torch.cuda.synchronize()
    return loss.detach().clone(), [p.grad.clone() for p in m.parameters()]


@pytest.mark.parametrize("dtype_name", ["float32", "float16"])
def test_grads_bitwise_equal_under_swapping(dtype_name):
    import torch

    from paper_conf_cluster_chenhzchysc21_b200.swap_hooks import SwapSaver
    torch.backends.cudnn.deterministic = True
    torch.backends.cudnn.benchmark = False
    dtype = getattr(torch, dtype_name)
    m = _net(torch, dtype)
    torch.manual_seed(1)
    x = torch.randn(16, 3, 64, 64, device="cuda", dtype=dtype)
    ref_loss, ref = _step(torch, m, x, None)
    for policy in ["none", "zvc", "auto", 2, 3, 4]:
        for prefetch in (True, False):
            saver = SwapSaver(policy, min_bytes=1 << 16, prefetch=prefetch)
            loss, got = _step(torch, m, x, saver)
            assert saver.stats["swapped"] >= 5, saver.stats
            assert torch.equal(loss, ref_loss), (policy, prefetch)
            for a, b in zip(got, ref):
                assert torch.equal(a, b), (policy, prefetch)
            assert not saver._live


def test_profiler_hidden_times_and_auto():
    import torch

    from paper_conf_cluster_chenhzchysc21_b200.swap_hooks import SwapSaver
    torch.backends.cudnn.deterministic = True
    m = _net(torch, torch.float32)
    x = torch.randn(16, 3, 64, 64, device="cuda")
    saver = SwapSaver("auto", min_bytes=1 << 16)

    def step(mark_fwd_end):
        m.zero_grad(set_to_none=True)
        loss = m(x).square().sum()
        mark_fwd_end()
        loss.backward()

    hidden = saver.profile(step)
    assert len(hidden) >= 5 and all(hf >= 0 and hb >= 0 for hf, hb in hidden)
    assert any(hf > 0 for hf, _ in hidden)
    ref_loss, ref = _step(torch, m, x, None)
    loss, got = _step(torch, m, x, saver)
    assert torch.equal(loss, ref_loss) and all(torch.equal(a, b) for a, b in zip(got, ref))


def test_online_reprofiling_replays_plan_and_follows_drift():
    """NEXT-2 (PAPER.md:118 sparsity profiled per epoch; :156-162 the advisor re-decides):
    SwapSaver("auto", reprofile_every=2) over 4 steps whose ReLU sparsity drifts (the conv biases
    move so every activation becomes zero from step 2 on).  Every step's loss and gradients are
    bitwise equal to the resident run; the probe runs only on the profiling steps 0 and 2 (one
    per swapped tensor, none on the replay steps 1 and 3); the plan changes with the drift and
    step 3 replays step 2's plan."""
    import torch

    from paper_conf_cluster_chenhzchysc21_b200 import cswap as C
    from paper_conf_cluster_chenhzchysc21_b200.swap_hooks import SwapSaver
    C.init(0)
    torch.backends.cudnn.deterministic = True
    torch.backends.cudnn.benchmark = False
    m = _net(torch, torch.float32)
    torch.manual_seed(1)
    x = torch.randn(16, 3, 64, 64, device="cuda")
    convs = [mod for mod in m if isinstance(mod, torch.nn.Conv2d)]
    base = [c.bias.detach().clone() for c in convs]
    saver = SwapSaver("auto", min_bytes=1 << 16, reprofile_every=2)
    probes = []
    for step in range(4):
        with torch.no_grad():
            for c, b in zip(convs, base):
                c.bias.copy_(b - (100.0 if step >= 2 else 0.0))  # step >= 2: every ReLU output is zero
        ref_loss, ref = _step(torch, m, x, None)
        C.collect_kernel_timing()
        C.set_kernel_timing(True)
        loss, got = _step(torch, m, x, saver)
        C.set_kernel_timing(False)
        recs = C.collect_kernel_timing()
        probes.append(sum(1 for r in recs if r["direction"] == 2))
        assert torch.equal(loss, ref_loss), step
        assert all(torch.equal(a, b) for a, b in zip(got, ref)), step
        assert not saver._live
    n = saver.stats["swapped"]
    assert n >= 5
    assert probes[1] == 0 and probes[3] == 0, probes
    assert probes[0] >= n and probes[2] >= n, probes
    (s0, plan0), (s2, plan2) = saver.plan_history
    assert (s0, s2) == (0, 2) and plan0 != plan2
    assert C.RLE in plan2  # all-zero activations: run-length coding wins
    assert saver.stats["codecs"] == plan2  # step 3 replayed the plan of step 2
