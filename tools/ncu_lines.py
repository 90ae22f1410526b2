"""Per-CUDA-source-line executed warp-instructions from an .ncu-rep (source page, cuda+sass):
python tools/ncu_lines.py report.ncu-rep [top]"""
import csv
import io
import subprocess
import sys


def main():
    raw = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
    path, hdr, acc, src = None, None, {}, {}
    for r in csv.reader(io.StringIO(raw)):
        if not r:
            continue
        if r[0] == "File Path":
            path = r[1].split("/")[-1]
            continue
        if r[0] == "Line No":
            hdr = r
            ie = hdr.index("Instructions Executed")
            continue
        if hdr is None or len(r) <= ie:
            continue
        if r[0]:                                   # a CUDA line row (its SASS rows follow with r[0] empty?)
            key = (path, r[0])
            src[key] = r[1][:80]
            try:
                acc[key] = acc.get(key, 0) + int(r[ie] or 0)
            except ValueError:
                pass
    tot = sum(acc.values()) or 1
    print("total", tot)
    for k, v in sorted(acc.items(), key=lambda t: -t[1])[:top]:
        print(f"{v:>11} {100 * v / tot:5.1f}% {k[0]}:{k[1]:>4} {src[k]}")


if __name__ == "__main__":
    main()
