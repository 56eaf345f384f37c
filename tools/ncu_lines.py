"""Instructions executed and stall samples per CUDA source line of one kernel in an ncu report
(needs -lineinfo and --import-source on).  python tools/ncu_lines.py REPORT KERNEL_REGEX [N]"""
import csv
import subprocess
import sys
from collections import Counter


def main():
    rep, kre = sys.argv[1], sys.argv[2]
    top = int(sys.argv[3]) if len(sys.argv) > 3 else 30
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=sass,cuda", "-k",
                          "regex:" + kre], capture_output=True, text=True).stdout
    fname, hdr = "?", None
    ins, smp, src = Counter(), Counter(), {}
    for r in csv.reader(out.splitlines()):
        if not r:
            continue
        if r[0] == "File Path":
            fname = r[1].split("/")[-1]
            continue
        if r[0] == "Line No":
            hdr = r
            continue
        if hdr is None or len(r) != len(hdr) or not r[0].isdigit():
            continue
        key = (fname, int(r[0]))
        src.setdefault(key, r[1].strip()[:90])
        ie, sp = hdr.index("Instructions Executed"), hdr.index("Warp Stall Sampling (All Samples)")
        ins[key] += int(r[ie] or 0)
        smp[key] += int(r[sp] or 0)
    tot, ts = sum(ins.values()) or 1, sum(smp.values()) or 1
    print(f"warp instructions {tot}, stall samples {ts}")
    for key, v in ins.most_common(top):
        print(f"{key[0]}:{key[1]:<5d} {100 * v / tot:5.1f}% ins {100 * smp[key] / ts:5.1f}% stall | {src[key]}")


if __name__ == "__main__":
    main()
