"""Markdown tables from a codec_bench JSONL sweep (tools/gpu_tasks.sh sweep / zvc):
per (kind, dtype, codec) rows of size x sparsity with compress / decompress fraction of the
measured HBM peak (algorithmic bytes) and the compression ratio.

    python tools/sweep_table.py gpurun_out/sweep.jsonl > profiles/codec_sweep_r01.md
"""
import json
import sys
from collections import defaultdict


def main():
    lines = [json.loads(l) for l in open(sys.argv[1]) if l.strip().startswith("{")]
    rows = [r for r in lines if "codec" in r]
    clocks = [r["clocks"] for r in lines if "clocks" in r]
    bad = [r for r in rows if r.get("roundtrip_ok") is False]
    groups = defaultdict(list)
    for r in rows:
        groups[(r.get("kind", "iid"), r["dtype"], r["codec"])].append(r)
    print(f"# Codec sweep ({len(rows)} points, round trips checked: "
          f"{sum(1 for r in rows if r.get('roundtrip_ok'))} ok, {len(bad)} failed)\n")
    if clocks:
        mhz = sorted(c["sm_mhz"] for c in clocks if c.get("sm_mhz"))
        reasons = sorted({x for c in clocks for x in c.get("reasons", [])})
        print(f"SM clock under load (nvidia-smi, {len(clocks)} runs): median {mhz[len(mhz) // 2] if mhz else None} MHz, "
              f"max {clocks[0].get('sm_max_mhz')} MHz, throttle reasons {reasons or 'none'}\n")
    print("Cells: compress / decompress fraction of the measured HBM peak in algorithmic bytes "
          "(raw + container), ms in parentheses; ratio = container / raw.  tools/codec_bench.py, "
          "L2 flushed between reps, median.\n")
    for (kind, dt, codec), rs in sorted(groups.items()):
        sps = sorted({r["s"] for r in rs})
        sizes = sorted({r["MiB"] for r in rs})
        print(f"## {codec.upper()} {dt} {kind}\n")
        print("| size | " + " | ".join(f"s = {s}" for s in sps) + " |")
        print("|---|" + "---|" * len(sps))
        for m in sizes:
            cells = []
            for s in sps:
                r = next((x for x in rs if x["MiB"] == m and x["s"] == s), None)
                if r is None:
                    cells.append("")
                    continue
                c, d = r["compress"], r["decompress"]
                cells.append(f"{c['frac']:.2f} / {d['frac']:.2f} ({c['ms']:.3g} / {d['ms']:.3g} ms), r {r['ratio']:.3f}")
            label = f"{m * 1024:g} KiB" if m < 1 else f"{m:g} MiB"
            print(f"| {label} | " + " | ".join(cells) + " |")
        print()


if __name__ == "__main__":
    main()
