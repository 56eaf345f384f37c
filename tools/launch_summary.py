"""Summarise an `ncu --metrics gpu__time_duration.sum --csv` launch list into a short text table:
per kernel (library kernels only, namespace cswap::) launches, total / mean duration and share
of the library's kernel time.  Launch times under ncu are serialised and cold-cache, so shares,
not absolute times, are what bench.py's roofline object is checked against.

    python tools/launch_summary.py gpurun_out/launches_r01.csv "command line" > profiles/launches_r01.txt
"""
import csv
import io
import re
import sys


def main():
    path, cmd = sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else ""
    text = open(path).read()
    start = text.index('"ID"')
    rows = list(csv.DictReader(io.StringIO(text[start:])))
    per = {}
    order = []
    for r in rows:
        if r["Metric Name"] != "gpu__time_duration.sum":
            continue
        name = r["Kernel Name"]
        if "cswap::" not in name:
            continue
        short = re.sub(r"^void ", "", name.split("(")[0]).replace("cswap::", "")
        ns = float(r["Metric Value"].replace(",", ""))
        p = per.setdefault(short, [0, 0.0])
        p[0] += 1
        p[1] += ns
        order.append((short, ns))
    tot = sum(v[1] for v in per.values())
    print(f"# ncu launch list (gpu__time_duration.sum, --clock-control none): {cmd}")
    print(f"# library kernels: {len(order)} launches, {tot / 1e6:.3f} ms total (serialised, cold cache)")
    print(f"# {'kernel':58s} {'launches':>8s} {'total_ms':>10s} {'mean_us':>9s} {'share':>7s}")
    for k, (n, ns) in sorted(per.items(), key=lambda kv: -kv[1][1]):
        print(f"  {k:58s} {n:8d} {ns / 1e6:10.3f} {ns / n / 1e3:9.1f} {ns / tot:7.1%}")


if __name__ == "__main__":
    main()
