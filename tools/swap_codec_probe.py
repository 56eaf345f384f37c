"""Swap-level latency (swap_out + swap_in, CUDA events and host wall) per codec for a few tensor
kinds — isolates per-codec pipeline costs that device-only codec timings do not show."""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch

    import synth
    from paper_conf_cluster_chenhzchysc21_b200 import cswap as C
    C.init(0)
    n = 49 << 20  # 196 MiB fp32
    kinds = {"zeros": torch.zeros(n, dtype=torch.int32, device="cuda"),
             "iid_0.65": synth.relu_iid_torch(n, 0.65, seed=1, dtype=C.F32, device="cuda")}
    out = torch.empty(n, dtype=torch.int32, device="cuda")
    side = torch.cuda.Stream()
    for name, x in kinds.items():
        for codec in (0, 1, 2, 3):
            for stream_name, st in (("cur", torch.cuda.current_stream()), ("side", side)):
                ts, ws = [], []
                for r in range(6):
                    torch.cuda.synchronize()
                    e0, e1, e2 = (torch.cuda.Event(enable_timing=True) for _ in range(3))
                    w0 = time.perf_counter()
                    e0.record()
                    h = C.swap_out(x, n, C.F32, codec)
                    e1.record()
                    st.wait_stream(torch.cuda.current_stream())
                    h.swap_in(out, stream=st)
                    e2.record(st)
                    e2.synchronize()
                    w1 = time.perf_counter()
                    h.close()
                    if r:
                        ts.append((e0.elapsed_time(e1), e1.elapsed_time(e2)))
                        ws.append((w1 - w0) * 1e3)
                assert torch.equal(out, x)
                print(json.dumps({"kind": name, "codec": codec, "stream": stream_name,
                                  "out_ms": round(sorted(t[0] for t in ts)[2], 3),
                                  "in_ms": round(sorted(t[1] for t in ts)[2], 3),
                                  "wall_ms": round(sorted(ws)[2], 3)}), flush=True)


if __name__ == "__main__":
    main()
