"""Summarise an .ncu-rep (raw page) into the handful of numbers we track."""
import csv
import io
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "launch__registers_per_thread", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum",
        "dram__bytes_read.sum", "dram__bytes_write.sum", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "l1tex__throughput.avg.pct_of_peak_sustained_active", "lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "sm__cycles_elapsed.avg.per_second"]


def summarise(path, out=sys.stdout):
    raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    h = rows[0]
    for r in rows[2:]:
        d = {a: (u, v) for a, u, v in zip(h, rows[1], r)}
        print(f"== {d.get('Kernel Name', ('', '?'))[1][:60]}", file=out)
        for k in KEYS:
            if k in d:
                print(f"  {k:62s} {d[k][1]:>14s} {d[k][0]}", file=out)
        st = [(k, float(d[k][1])) for k in d if k.startswith("smsp__pcsamp_warps_issue_stalled_")
              and not k.endswith("not_issued") and d[k][1].replace(".", "", 1).isdigit()]
        tot = sum(v for _, v in st) or 1
        for k, v in sorted(st, key=lambda t: -t[1])[:8]:
            print(f"  stall {k[33:]:56s} {100 * v / tot:6.1f} %", file=out)


if __name__ == "__main__":
    for p in sys.argv[1:]:
        summarise(p)
