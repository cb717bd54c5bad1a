"""Print the headline ncu sections + stall breakdown + top source lines of a report."""
import csv
import subprocess
import sys

sys.path.insert(0, __import__("os").path.dirname(__file__))
from ncu_lines import lines  # noqa: E402

KEEP = ("Duration", "Elapsed Cycles", "DRAM Throughput", "Memory Throughput", "Compute (SM) Throughput",
        "Issue Slots Busy", "Executed Ipc Active", "Achieved Occupancy", "Theoretical Occupancy",
        "Registers Per Thread", "Dynamic Shared Memory Per Block", "Avg. Active Threads Per Warp",
        "Warp Cycles Per Issued Instruction", "L1/TEX Hit Rate", "L2 Hit Rate", "Block Limit Registers",
        "Block Limit Shared Mem", "Eligible Warps Per Scheduler", "Active Warps Per Scheduler")


def main(rep, n=25):
    txt = subprocess.run(["ncu", "-i", rep, "--page", "details", "--csv"], capture_output=True, text=True).stdout
    r = csv.reader(txt.splitlines())
    hdr = next(r)
    seen = set()
    for row in r:
        d = dict(zip(hdr, row))
        k = d.get("Metric Name", "")
        if k in KEEP and k not in seen:
            seen.add(k)
            print(f"{k:45s} {d.get('Metric Value', ''):>14s} {d.get('Metric Unit', '')}")
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rr = list(csv.reader(raw.splitlines()))
    h, v = rr[0], rr[2] if len(rr) > 2 else rr[1]
    for name in ("dram__bytes_read.sum", "dram__bytes_write.sum", "smsp__inst_executed.sum",
                 "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.pct_of_peak_sustained_active"):
        if name in h:
            print(f"{name:55s} {v[h.index(name)]}")
    rows = lines(rep)
    tot = sum(x[0] for x in rows) or 1
    print("top source lines (stall samples %, instructions %):")
    tex = sum(x[1] for x in rows) or 1
    for s, ex, f, ln, src in sorted(rows, reverse=True)[:n]:
        print(f"{100*s/tot:5.1f}% {100*ex/tex:5.1f}%i {f}:{ln:5s} {src}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 25)
