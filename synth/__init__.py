"""Seeded synthetic input generators shared by the oracle tests, the GPU parity tests and
bench.py.  This module holds NONE of the method's arithmetic (no codec, probe or selector
logic): it only draws tensors with the shapes, sparsities and zero-placement structure of
the paper's workloads (the paper's "synthetic tensor generator"), and
names the workload sets of DESIGN.md §5.

Values are returned as RAW WORDS (np.uint32 for f32, np.uint16 for f16/bf16) so every
consumer compares bits, never floats.  Non-zeros are |N(0,1)| (ReLU-like); exact zeros
from rounding are re-drawn, so the zero pattern is exactly the drawn mask.
"""
from __future__ import annotations

import numpy as np

F32, F16, BF16 = 0, 1, 2
WIDTH = {F32: 4, F16: 2, BF16: 2}
NAMES = {F32: "f32", F16: "f16", BF16: "bf16"}
WORD = {F32: np.uint32, F16: np.uint16, BF16: np.uint16}


def seed_of(config: int, size_idx: int = 0, sparsity_idx: int = 0, layer_idx: int = 0) -> int:
    """seed = (config << 24) | (size_idx << 16) | (sparsity_idx << 8) | layer_idx."""
    return (config << 24) | (size_idx << 16) | (sparsity_idx << 8) | layer_idx


def _positive_words(rng: np.random.Generator, m: int, dtype: int) -> np.ndarray:
    """m words of |N(0,1)| in dtype, none bitwise zero."""
    v = np.abs(rng.standard_normal(m, dtype=np.float32))
    if dtype == F32:
        w = v.view(np.uint32).copy()
    elif dtype == F16:
        w = v.astype(np.float16).view(np.uint16).copy()
    else:  # bf16: round-to-nearest-even on the upper 16 bits of the fp32 pattern
        b = v.view(np.uint32).astype(np.uint64)
        w = ((b + 0x7FFF + ((b >> 16) & 1)) >> 16).astype(np.uint16)
    bad = w == 0
    while bad.any():  # re-draw exact zeros (rounding underflow)
        w[bad] = _positive_words(rng, int(bad.sum()), dtype)
        bad = w == 0
    return w


def relu_iid(n: int, sparsity: float, seed: int, dtype: int = F32, exact: bool = False) -> np.ndarray:
    """iid Bernoulli(sparsity) zero mask; exact=True places exactly round(sparsity*n) zeros
    by a random permutation (config 1)."""
    rng = np.random.Generator(np.random.PCG64(seed))
    x = _positive_words(rng, n, dtype)
    if exact:
        nz = int(round(sparsity * n))
        zero_idx = rng.permutation(n)[:nz]
        x[zero_idx] = 0
    else:
        x[rng.random(n) < sparsity] = 0
    return x


def relu_clustered(n: int, sparsity: float, mean_zero_run: float, seed: int, dtype: int = F32) -> np.ndarray:
    """Two-state Markov zero placement: zero runs ~ Geometric(mean L0), non-zero runs
    ~ Geometric(mean L0 (1-s)/s)."""
    rng = np.random.Generator(np.random.PCG64(seed))
    x = _positive_words(rng, n, dtype)
    if sparsity <= 0:
        return x
    if sparsity >= 1:
        x[:] = 0
        return x
    L0 = float(mean_zero_run)
    L1 = max(L0 * (1 - sparsity) / sparsity, 1.0)
    mask = np.zeros(n, dtype=bool)
    pos = 0
    state = rng.random() < sparsity
    while pos < n:
        m = L0 if state else L1
        run = int(rng.geometric(1.0 / m))
        if state:
            mask[pos:pos + run] = True
        pos += run
        state = not state
    x[mask] = 0
    return x


def channel_dead(shape, sparsity: float, seed: int, dtype: int = F32) -> np.ndarray:
    """NCHW tensor where a fraction `sparsity` of the (n, c) planes are entirely zero."""
    N, C, H, W = shape
    rng = np.random.Generator(np.random.PCG64(seed))
    x = _positive_words(rng, N * C * H * W, dtype).reshape(N * C, H * W)
    dead = rng.random(N * C) < sparsity
    x[dead] = 0
    return x.reshape(-1)


def constant(n: int, word: int, dtype: int = F32) -> np.ndarray:
    return np.full(n, word, dtype=WORD[dtype])


# --------------------------------------------------------------------------------------
# Device-side generation for the big workloads (torch is plumbing here: Philox draws).
# --------------------------------------------------------------------------------------
def relu_iid_torch(n: int, sparsity: float, seed: int, dtype: int, device):
    """Same recipe as relu_iid (Bernoulli mask, |N(0,1)| non-zeros) drawn on `device`;
    returns a tensor of raw words (int32 for f32, int16 for f16/bf16)."""
    import torch
    g = torch.Generator(device=device)
    g.manual_seed(seed)
    tdt = {F32: torch.float32, F16: torch.float16, BF16: torch.bfloat16}[dtype]
    v = torch.randn(n, generator=g, device=device, dtype=torch.float32).abs_().to(tdt)
    v[v == 0] = 1.0  # rounding underflow -> a fixed non-zero
    keep = torch.rand(n, generator=g, device=device) >= sparsity
    v.mul_(keep.to(tdt))
    return v.view(torch.int32 if dtype == F32 else torch.int16)


# --------------------------------------------------------------------------------------
# Workload sets (BASELINE.json configs 3-4)
# --------------------------------------------------------------------------------------
def vgg16_b64():
    """The 12 conv-input ReLU/MAX outputs of VGG16 at batch 64 (vDNN conv-input policy,
    PAPER.md:251), with a synthetic per-layer sparsity profile inside the paper's 20-80 %
    range and MAX4 < 45 %.  Returns [(name, shape, s)]."""
    B = 64
    return [
        ("relu1_1", (B, 64, 224, 224), 0.45),
        ("pool1", (B, 64, 112, 112), 0.30),
        ("relu2_1", (B, 128, 112, 112), 0.50),
        ("pool2", (B, 128, 56, 56), 0.30),
        ("relu3_1", (B, 256, 56, 56), 0.55),
        ("relu3_2", (B, 256, 56, 56), 0.65),
        ("pool3", (B, 256, 28, 28), 0.35),
        ("relu4_1", (B, 512, 28, 28), 0.70),
        ("relu4_2", (B, 512, 28, 28), 0.75),
        ("pool4", (B, 512, 14, 14), 0.40),
        ("relu5_1", (B, 512, 14, 14), 0.80),
        ("relu5_2", (B, 512, 14, 14), 0.80),
    ]


def resnet50_b64(seed: int = 4 << 24):
    """The 49 ReLU outputs + the maxpool output of torchvision ResNet-50 v1.5 at batch 64,
    224x224 (stride on the 3x3 conv).  Sparsity ~ U[0.3, 0.7], seeded."""
    B = 64
    shapes = [("stem_relu", (B, 64, 112, 112)), ("maxpool", (B, 64, 56, 56))]
    hw = 56
    for li, (width, blocks) in enumerate([(64, 3), (128, 4), (256, 6), (512, 3)]):
        for b in range(blocks):
            stride = 2 if (b == 0 and li > 0) else 1
            hw_in = hw
            hw_out = hw // stride
            shapes.append((f"l{li+1}b{b}_relu1", (B, width, hw_in, hw_in)))
            shapes.append((f"l{li+1}b{b}_relu2", (B, width, hw_out, hw_out)))
            shapes.append((f"l{li+1}b{b}_relu3", (B, width * 4, hw_out, hw_out)))
            hw = hw_out
    rng = np.random.Generator(np.random.PCG64(seed))
    return [(name, shp, float(rng.uniform(0.3, 0.7))) for name, shp in shapes]


def bert_large_b8():
    """Per layer of BERT-large (24 layers), batch 8, seq 512, fp16: attention-prob dropout
    [8,16,512,512] (s=0.10), GELU output [8,512,4096] (s~0), two hidden dropouts
    [8,512,1024] (s=0.10)."""
    out = []
    for l in range(24):
        out.append((f"L{l}_attn_drop", (8, 16, 512, 512), 0.10))
        out.append((f"L{l}_gelu", (8, 512, 4096), 0.0))
        out.append((f"L{l}_hid_drop1", (8, 512, 1024), 0.10))
        out.append((f"L{l}_hid_drop2", (8, 512, 1024), 0.10))
    return out


def numel(shape) -> int:
    n = 1
    for d in shape:
        n *= int(d)
    return n
