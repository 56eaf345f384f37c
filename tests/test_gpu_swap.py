"""GPU swap pipeline: the pinned host container equals the oracle's bytes and the restored
tensor is bitwise equal (DESIGN.md §1 rows a11/a12), AUTO selection agrees with the oracle
selector on the same probe counts, and swaps at BASELINE sizes round-trip."""
import numpy as np
import pytest

import synth
from oracle import oracle as O
from tests import gpu_util as G

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def C():
    return G.lib()


@pytest.mark.parametrize("codec", list(G.IMPLEMENTED))
@pytest.mark.parametrize("n", [0, 1000, (1 << 22) + 12345])
def test_swap_container_equals_oracle(C, codec, n):
    import torch
    C.set_format(1 << 20, 1024, 65536)
    x = synth.relu_iid(n, 0.5, seed=n + 1)
    d = G.to_dev(x) if n else G.empty_like_words(0, 0)
    h = C.swap_out(d, n, C.F32, codec)
    h.wait()
    ref = O.compress(x, codec, O.F32, F=1 << 20, param={3: 1024, 4: 65536}.get(codec, 0))
    assert h.host_bytes() == ref
    out = G.poisoned_words(n, 0)
    h.swap_in(out)
    h.wait()
    torch.cuda.synchronize()
    assert np.array_equal(G.from_dev(out)[:n], x)
    h.close()
    C.set_format(1 << 22, 1024, 65536)


def test_auto_matches_oracle_selector(C):
    cal = C.get_calibration()
    for n, s in [(1 << 10, 0.5), (1 << 20, 0.05), (1 << 22, 0.5), (1 << 22, 0.0), (1 << 22, 1.0)]:
        x = synth.relu_iid(n, s, seed=7)
        d = G.to_dev(x)
        counts = O.probe(x, O.F32)
        if n == 1 << 22 and s == 1.0 and O.RLE not in G.IMPLEMENTED:
            continue  # all-zero tensors select RLE
        h = C.swap_out(d, n, C.F32, C.AUTO)
        h.wait()
        q = h.query()
        counts = O.probe(x, O.F32)
        oc = O.Calib()
        for f, _ in C.Calib._fields_:
            v = getattr(cal, f)
            if f == "beta":
                for i in range(len(v)):
                    oc.beta[i] = v[i]
            elif f == "reserved":
                continue
            else:
                setattr(oc, f, v)
        ref = O.select(n, O.F32, counts, 0.0, 0.0, oc)
        expect = ref["codec"] if ref["codec"] in G.IMPLEMENTED else None
        assert q["decision"].codec == ref["codec"]
        if expect is not None:
            assert q["codec"] == expect
        h.close()


def test_vgg_sized_tensor_roundtrip_sampled_frames(C):
    """Full BASELINE size (VGG16 b64 relu1_1, 784 MiB fp32, F = 2^22) in the bench launch
    configuration: the oracle checks sampled frames one by one; the round trip is checked in full."""
    import torch
    name, shape, s = synth.vgg16_b64()[0]
    n = synth.numel(shape)
    d = synth.relu_iid_torch(n, s, seed=synth.seed_of(3, 0, 0, 0), dtype=0, device="cuda")
    h = C.swap_out(d, n, C.F32, C.ZVC)
    h.wait()
    blob = h.host_bytes()
    x = G.from_dev(d)
    F = 1 << 22
    K = -(-n // F)
    import struct
    fb = struct.unpack_from(f"<{K}Q", blob, 64)
    starts = np.concatenate([[(64 + 8 * K + 15) // 16 * 16], np.cumsum(fb)[:-1] + (64 + 8 * K + 15) // 16 * 16])
    for k in [0, 1, K // 2, K - 1]:
        xf = x[k * F:(k + 1) * F]
        ref = O.compress(xf, O.ZVC, O.F32, F=F)
        ds = (64 + 8 + 15) // 16 * 16
        assert blob[starts[k]:starts[k] + fb[k]] == ref[ds:]
    for k in range(K):  # closed form per frame at full size: align16(Fk/8) + align16(4 nnz_k)
        Fk = min(F, n - k * F)
        nnz_k = int(torch.count_nonzero(d[k * F:k * F + Fk]).item())
        assert fb[k] == ((Fk + 31) // 32 * 4 + 15) // 16 * 16 + (4 * nnz_k + 15) // 16 * 16
    out = G.poison_like(d)
    h.swap_in(out)
    h.wait()
    assert torch.equal(out, d)
    h.close()
