"""Summarise ncu reports (.ncu-rep) into a small JSON kept under profiles/.

    python tools/ncu_summary.py OUT.json name=path.ncu-rep [name=path.ncu-rep ...]

Per kernel: launches, mean duration, DRAM read+write bytes per launch, DRAM throughput %,
issue-active %, registers, achieved occupancy.  Traffic is what the roofline object's `traffic`
field reports (bench.py scales the measured DRAM-bytes/algorithmic-bytes ratio to its launches).
"""
import csv
import io
import json
import subprocess
import sys

METRICS = {
    "gpu__time_duration.sum": "duration_ns",
    "dram__bytes_read.sum": "dram_read",
    "dram__bytes_write.sum": "dram_write",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed": "dram_pct",
    "smsp__issue_active.avg.pct_of_peak_sustained_active": "issue_active_pct",
    "sm__warps_active.avg.pct_of_peak_sustained_active": "achieved_occupancy_pct",
    "launch__registers_per_thread": "registers",
    "launch__grid_size": "grid",
    "launch__block_size": "block",
}
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1, "us": 1e3, "ms": 1e6, "usecond": 1e3,
         "msecond": 1e6, "nsecond": 1}


def read(path):
    raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units = rows[0], rows[1]
    out = []
    for r in rows[2:]:
        d = {"kernel": r[hdr.index("Kernel Name")].split("(")[0].replace("void ", "")}
        for m, key in METRICS.items():
            if m in hdr:
                i = hdr.index(m)
                v = r[i].replace(",", "")
                try:
                    d[key] = float(v) * SCALE.get(units[i], 1)
                except ValueError:
                    d[key] = v
        out.append(d)
    return out


def summarise(launches):
    by = {}
    for d in launches:
        by.setdefault(d["kernel"], []).append(d)
    res = {}
    for k, ls in by.items():
        n = len(ls)
        avg = lambda key: sum(x.get(key, 0) for x in ls) / n  # noqa: E731
        res[k] = {"launches": n, "duration_us": avg("duration_ns") / 1e3,
                  "dram_bytes_per_launch": avg("dram_read") + avg("dram_write"),
                  "dram_read_per_launch": avg("dram_read"), "dram_write_per_launch": avg("dram_write"),
                  "dram_pct": avg("dram_pct"), "issue_active_pct": avg("issue_active_pct"),
                  "achieved_occupancy_pct": avg("achieved_occupancy_pct"), "registers": ls[0].get("registers"),
                  "grid": ls[0].get("grid"), "block": ls[0].get("block")}
    return res


if __name__ == "__main__":
    out = {}
    for arg in sys.argv[2:]:
        name, path = arg.split("=", 1)
        out[name] = summarise(read(path))
    with open(sys.argv[1], "w") as f:
        json.dump(out, f, indent=1)
    print(json.dumps(out, indent=1))
