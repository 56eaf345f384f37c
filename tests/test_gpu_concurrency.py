"""The persistent ZVC compress under concurrency: its CTAs wait
for the published counts of other CTAs, so every CTA must be resident; the cooperative launch
guarantees that.  Each scenario runs in a subprocess with a timeout, so a stall fails the test
instead of hanging the GPU: (a) a hog kernel holds half the SMs for 50 ms while a compress is
launched on another stream; (b) two host threads compress on two streams at once; (c) both.
Outputs must equal the serial result, which equals the oracle on sampled frames."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

SCRIPT = r'''
import ctypes, hashlib, json, sys, threading
import numpy as np, torch
sys.path.insert(0, ROOT)
import synth
from oracle import oracle as O
from tests import gpu_util as G
C = G.lib()
hog = ctypes.CDLL(HOG)
hog.hog_launch.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_uint64, ctypes.c_void_p, ctypes.c_void_p]
sink = torch.zeros(1, dtype=torch.int32, device="cuda")
sms = torch.cuda.get_device_properties(0).multi_processor_count
n = 64 << 20  # 256 MiB f32
dtype = C.F32
xs = [synth.relu_iid_torch(n, s, seed=synth.seed_of(9, 0, i), dtype=0, device="cuda") for i, s in enumerate((0.5, 0.8))]
cap = C.max_compressed_size(n, dtype, C.ZVC)

def compress(x, stream):
    out = torch.full((cap,), 0xA5, dtype=torch.uint8, device="cuda")
    size = torch.zeros(1, dtype=torch.int64, device="cuda")
    with torch.cuda.stream(stream):
        C.compress(x, n, dtype, C.ZVC, out, cap, size, stream=stream)
    stream.synchronize()
    return hashlib.sha256(out[:int(size.item())].cpu().numpy().tobytes()).hexdigest(), out, int(size.item())

s0 = torch.cuda.current_stream()
ref = []
for x in xs:
    digest, out, size = compress(x, s0)
    ref.append(digest)
    # the serial result equals the oracle on the first and the last frame
    blob = out[:size].cpu().numpy().tobytes()
    words = G.from_dev(x)
    F = 1 << 22
    K = n // F
    fb = np.frombuffer(blob, dtype=np.uint64, count=K, offset=64)
    ds = (64 + 8 * K + 15) // 16 * 16
    starts = [int(v) for v in np.concatenate([[ds], ds + np.cumsum(fb)[:-1]])]
    for k in (0, K - 1):
        r = O.compress(words[k * F:(k + 1) * F], O.ZVC, O.F32)
        assert blob[starts[k]:starts[k] + fb[k]] == r[(64 + 8 + 15) // 16 * 16:], k
res = {}
# (a) a hog holds half the SMs (one 1024-thread CTA with 150 KiB smem per SM) for 50 ms
side = torch.cuda.Stream()
hog.hog_launch(sms // 2, 150 * 1024, 50_000_000, ctypes.c_void_p(sink.data_ptr()), ctypes.c_void_p(side.cuda_stream))
st = torch.cuda.Stream()
res["hog"] = compress(xs[0], st)[0] == ref[0]
torch.cuda.synchronize()
# (b) two host threads, two streams, 5 compresses each, all at once
ok = []
def worker(i):
    stream = torch.cuda.Stream()
    for _ in range(5):
        ok.append(compress(xs[i], stream)[0] == ref[i])
th = [threading.Thread(target=worker, args=(i,)) for i in range(2)]
[t.start() for t in th]
[t.join() for t in th]
res["two_streams"] = len(ok) == 10 and all(ok)
# (c) both: hog + two threads
hog.hog_launch(sms // 2, 150 * 1024, 50_000_000, ctypes.c_void_p(sink.data_ptr()), ctypes.c_void_p(side.cuda_stream))
ok.clear()
th = [threading.Thread(target=worker, args=(i,)) for i in range(2)]
[t.start() for t in th]
[t.join() for t in th]
res["hog_two_streams"] = len(ok) == 10 and all(ok)
torch.cuda.synchronize()
print(json.dumps(res))
'''


@pytest.fixture(scope="module")
def hog_so(tmp_path_factory):
    out = str(tmp_path_factory.mktemp("hog") / "libhog.so")
    subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-shared", "-Xcompiler", "-fPIC", "-O2",
                           "-gencode", "arch=compute_100a,code=sm_100a",
                           os.path.join(ROOT, "tests", "native", "hog.cu"), "-o", out])
    return out


def test_persistent_compress_progresses_beside_other_kernels(hog_so):
    code = f"ROOT = {ROOT!r}\nHOG = {hog_so!r}\n" + SCRIPT
    p = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, timeout=300, cwd=ROOT)
    assert p.returncode == 0, p.stderr[-3000:]
    res = json.loads(p.stdout.strip().splitlines()[-1])
    assert res == {"hog": True, "two_streams": True, "hog_two_streams": True}
