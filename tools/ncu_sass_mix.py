"""Instruction mix and stall samples per SASS opcode of one kernel in an ncu report
(ncu --page source --print-source=sass).  python tools/ncu_sass_mix.py REPORT KERNEL_REGEX [N]"""
import csv
import subprocess
import sys
from collections import Counter


def main():
    rep, kre = sys.argv[1], sys.argv[2]
    top = int(sys.argv[3]) if len(sys.argv) > 3 else 20
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=sass", "-k", "regex:" + kre],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    blk, started = [], False
    rows = [r for r in rows if r]
    for r in rows:
        if r and r[0] == "Kernel Name":
            if started:
                break
            started = True
            print(r[1][:100])
            continue
        blk.append(r)
    h = blk[0]
    data = [r for r in blk[1:] if len(r) == len(h)]
    ie, sp = h.index("Instructions Executed"), h.index("Warp Stall Sampling (All Samples)")
    tot = sum(int(r[ie] or 0) for r in data)
    ts = sum(int(r[sp] or 0) for r in data) or 1
    c, s = Counter(), Counter()
    for r in data:
        toks = r[1].split()
        if not toks:
            continue
        op = (toks[1] if toks[0].startswith("@") else toks[0]).split(".")[0]
        c[op] += int(r[ie] or 0)
        s[op] += int(r[sp] or 0)
    print(f"warp instructions {tot}, stall samples {ts}")
    for k, v in c.most_common(top):
        print(f"  {k:10s} {v:12d} {100 * v / tot:5.1f}%  stall {100 * s[k] / ts:5.1f}%")


if __name__ == "__main__":
    main()
