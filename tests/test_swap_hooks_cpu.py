"""Host logic of the training integration (swap_hooks.SwapSaver) on CPU with a stand-in backend
that keeps a host copy: deduplication of an activation saved by two ops, restore on use, prefetch
in reverse save order, reference counting, the profiler's Hidden_f/Hidden_b bookkeeping order.
Gradients must equal a run without hooks exactly (the swap is lossless)."""
import torch

from paper_conf_cluster_chenhzchysc21_b200.swap_hooks import SwapSaver


class HostCopy:
    def __init__(self):
        self.out, self.inn, self.freed = [], [], 0

    @staticmethod
    def accepts(t):
        return True

    def swap_out(self, t, codec, hf, hb):
        self.out.append((tuple(t.shape), codec, hf, hb))
        return t.detach().clone()

    def swap_in(self, h, out, stream):
        self.inn.append(tuple(out.shape))
        out.copy_(h)

    @staticmethod
    def info(h):
        return 1, h.numel() * h.element_size()

    def free(self, h):
        self.freed += 1


def net():
    torch.manual_seed(0)
    return torch.nn.Sequential(
        torch.nn.Conv2d(3, 8, 3, padding=1), torch.nn.ReLU(), torch.nn.MaxPool2d(2),
        torch.nn.Conv2d(8, 16, 3, padding=1), torch.nn.ReLU(), torch.nn.MaxPool2d(2),
        torch.nn.Flatten(), torch.nn.Linear(16 * 8 * 8, 10))


def grads(model, x, saver=None):
    model.zero_grad()
    if saver is None:
        loss = model(x).square().sum()
    else:
        with saver:
            loss = model(x).square().sum()
    loss.backward()
    return loss.detach(), [p.grad.clone() for p in model.parameters()]


def test_hooks_lossless_and_bookkeeping():
    x = torch.randn(4, 3, 32, 32)
    m = net()
    ref_loss, ref = grads(m, x)
    be = HostCopy()
    saver = SwapSaver(policy=1, min_bytes=1024, backend=be)
    loss, got = grads(m, x, saver)
    assert torch.equal(loss, ref_loss)
    assert all(torch.equal(a, b) for a, b in zip(got, ref))
    n = saver.stats["swapped"]
    # conv1 input (x), relu1 out (saved by relu and pool), pool1 out (conv2 input), relu2 out,
    # pool2 out / flatten -> linear input: every distinct activation once
    assert n == len(be.out) and n >= 4
    assert be.freed == n and not saver._live  # every handle released after backward
    assert len(be.inn) == n  # each restored exactly once (prefetched or on demand)
    # restores run in reverse save order (prefetch of i-1 is issued when i is used)
    saved = [s for s, *_ in be.out]
    assert be.inn == list(reversed(saved))


def test_dedup_of_tensor_saved_twice():
    be = HostCopy()
    saver = SwapSaver(policy=1, min_bytes=0, backend=be)
    x = torch.randn(1000, requires_grad=True)
    with saver:
        y = torch.relu(x * 2.0)      # relu saves its output y
        z = (y * y).sum()            # mul saves y twice (both operands)
    z.backward()
    assert saver.stats["swapped"] == len(be.out)
    shapes = [s for s, *_ in be.out]
    assert shapes.count((1000,)) == len(shapes)
    assert be.freed == len(shapes)
    xr = x.detach().clone().requires_grad_(True)
    (torch.relu(xr * 2.0).square().sum()).backward()
    assert torch.equal(x.grad, xr.grad)


def test_small_and_parameter_tensors_stay_resident():
    be = HostCopy()
    saver = SwapSaver(policy=1, min_bytes=1 << 30, backend=be)
    x = torch.randn(4, 3, 32, 32)
    m = net()
    _, got = grads(m, x, saver)
    _, ref = grads(m, x)
    assert saver.stats["swapped"] == 0 and not be.out
    assert all(torch.equal(a, b) for a, b in zip(got, ref))


def test_hidden_times_reach_swap_out_in_save_order():
    be = HostCopy()
    saver = SwapSaver(policy=255, min_bytes=1024, backend=be)
    saver.hidden = [(0.001 * (i + 1), 0.002 * (i + 1)) for i in range(16)]
    grads(net(), torch.randn(4, 3, 32, 32), saver)
    for i, (_, codec, hf, hb) in enumerate(be.out):
        assert codec == 255 and hf == 0.001 * (i + 1) and hb == 0.002 * (i + 1)


def test_reused_address_is_not_deduplicated():
    """A swapped-out activation's memory is freed; the allocator may place the next activation of
    the same size at the same address (same data_ptr, numel, dtype, version).  That is a new
    tensor and must get its own swap record."""
    torch.manual_seed(0)
    layers = [torch.nn.Linear(128, 128) for _ in range(8)]
    x = torch.randn(64, 128)  # 32 KiB activations: below malloc's mmap threshold, so reused

    def fwd():
        h = x
        for lin in layers:
            h = torch.relu(lin(h))
        return h.square().sum()

    for p in (q for lin in layers for q in lin.parameters()):
        p.grad = None
    fwd().backward()
    ref = [p.grad.clone() for lin in layers for p in lin.parameters()]
    for p in (q for lin in layers for q in lin.parameters()):
        p.grad = None
    be = HostCopy()
    saver = SwapSaver(policy=1, min_bytes=1024, backend=be)
    with saver:
        loss = fwd()
    loss.backward()
    got = [p.grad.clone() for lin in layers for p in lin.parameters()]
    assert all(torch.equal(a, b) for a, b in zip(got, ref))
    # x and the 8 relu outputs: each its own record, however the allocator reused addresses
    assert saver.stats["swapped"] == len(be.out) == 9


class Deciding(HostCopy):
    """AUTO stand-in: 'compresses' (codec 1) iff the tensor has any zero, else NONE."""

    def swap_out(self, t, codec, hf, hb):
        h = super().swap_out(t, codec, hf, hb)
        self.decided = getattr(self, "decided", 0) + (codec == 255)
        return (h, 1 if codec == 1 or (codec == 255 and bool((t == 0).any())) else 0)

    def swap_in(self, h, out, stream):
        super().swap_in(h[0], out, stream)

    @staticmethod
    def info(h):
        return h[1], h[0].numel() * h[0].element_size()


def test_reprofiling_replays_plan_between_profiling_steps():
    be = Deciding()
    saver = SwapSaver(policy="auto", min_bytes=0, backend=be, reprofile_every=3)
    w = torch.randn(64, 64, requires_grad=True)
    shift = 1000.0  # large positive bias: no zeros -> NONE
    plans = []
    for step in range(7):
        if step == 3:
            shift = -1000.0  # drift: every relu output becomes all zero -> compress
        x = torch.randn(32, 64)
        with saver:
            y = torch.relu(x @ w + shift)
            loss = (y * y).sum()
        loss.backward()
        plans.append(list(saver.stats["codecs"]))
    # steps 0, 3, 6 are profiling steps (AUTO asked per tensor); the others replay the plan
    assert [s for s, _ in saver.plan_history] == [0, 3, 6]
    # saved: x (the matmul input, never zero) and the relu output y
    assert plans[0] == plans[1] == plans[2] == [0, 0]
    assert plans[3] == plans[4] == plans[5] == [0, 1]
    assert be.decided == sum(len(plans[i]) for i in (0, 3, 6))
