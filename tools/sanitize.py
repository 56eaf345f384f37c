"""Small-size workload for compute-sanitizer (memcheck / racecheck / synccheck / initcheck):
every codec x f32/f16 x ragged sizes and multi-frame formats, compress -> decompress through the
C ABI with the round trip checked, corrupted containers (must flag an error, never fault), and
one AUTO swap-out / swap-in.  The persistent ZVC compress runs on a small grid (8 CTAs) so that
co-residency, which its cross-CTA offset protocol needs, holds under the sanitizer's reduced
occupancy.

    compute-sanitizer --tool memcheck python tools/sanitize.py
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import numpy as np
    import torch

    import synth
    from paper_conf_cluster_chenhzchysc21_b200 import cswap as C
    C.init(0)
    C.set_zvc_launch(8, -1)
    names = {C.NONE: "none", C.ZVC: "zvc", C.RLE: "rle", C.CSR: "csr", C.LZ4: "lz4"}
    n_ok = 0
    for dtype in (C.F32, C.F16):
        for n, F in ((1, 1024), (1000, 1024), (70001, 16384), (300000, 1 << 22)):
            x = synth.relu_iid_torch(n, 0.55, seed=n, dtype=dtype, device="cuda")
            for codec in names:
                fmt = (F, 1024 if F % 1024 == 0 else F, 65536)
                cap = C.max_compressed_size(n, dtype, codec, fmt)
                buf = torch.empty(cap, dtype=torch.uint8, device="cuda")
                size = torch.zeros(1, dtype=torch.int64, device="cuda")
                err = torch.zeros(1, dtype=torch.int32, device="cuda")
                y = torch.empty_like(x)
                C.compress(x, n, dtype, codec, buf, cap, size, fmt=fmt)
                nb = int(size.item())
                C.decompress(buf, nb, y, n, dtype, codec, fmt=fmt, err=err)
                torch.cuda.synchronize()
                assert int(err.item()) == 0 and torch.equal(x, y), (names[codec], dtype, n, F)
                # corrupted payload bytes: an error flag, no fault
                if codec != C.NONE and nb > 200:
                    bad = buf[:nb].clone()  # only the written bytes (initcheck)
                    rng = np.random.default_rng(n + codec)
                    for pos in rng.integers(64 + 8, nb, size=8):
                        bad[int(pos)] ^= 0x5A
                    err.zero_()
                    C.decompress(bad, nb, y, n, dtype, codec, fmt=fmt, err=err)
                    torch.cuda.synchronize()
                n_ok += 1
    x = synth.relu_iid_torch(1 << 20, 0.5, seed=7, dtype=C.F32, device="cuda")
    y = torch.empty_like(x)
    h = C.swap_out(x, 1 << 20, C.F32, C.AUTO)
    h.swap_in(y)
    h.wait()
    h.close()
    torch.cuda.synchronize()
    assert torch.equal(x, y)
    print(f"sanitize workload ok: {n_ok} codec round trips + corrupt decodes + 1 swap")


if __name__ == "__main__":
    main()
