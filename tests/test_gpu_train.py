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
