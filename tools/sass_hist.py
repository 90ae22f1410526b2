"""Per-opcode executed-instruction histogram from an .ncu-rep source page (SASS)."""
import csv
import io
import re
import subprocess
import sys
from collections import Counter


def hist(path, top=25):
    raw = subprocess.run(["ncu", "-i", path, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    h = rows[1]
    ie = h.index("Instructions Executed")
    samp = h.index("Warp Stall Sampling (All Samples)")
    c, s = Counter(), Counter()
    for r in rows[2:]:
        if len(r) <= ie:
            continue
        m = re.match(r"\s*(@!?U?P\w+\s+)?([A-Z0-9_]+)(\.[A-Z0-9_.]+)?", r[1])
        if not m:
            continue
        op = m.group(2) + (m.group(3) or "")
        c[op] += int(r[ie] or 0)
        s[op] += int(r[samp] or 0)
    tot = sum(c.values())
    ts = sum(s.values()) or 1
    print(f"total warp-instructions executed: {tot}")
    for op, n in c.most_common(top):
        print(f"  {op:28s} {n:14d} {100 * n / tot:6.2f} %   stall-samples {100 * s[op] / ts:5.1f} %")


if __name__ == "__main__":
    hist(sys.argv[1])
