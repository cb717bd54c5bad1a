"""Per-kernel ncu summary of a --set full report: the details-page metrics that bound a kernel and
its top CUDA source lines by executed warp-instructions (with average active lanes per line).

  python tools/ncu_kernel_lines.py REPORT.ncu-rep KERNEL_REGEX [N]"""
import csv
import subprocess
import sys

WANT = ["Duration", "Registers Per Thread", "Achieved Occupancy", "Theoretical Occupancy", "Issue Slots Busy",
        "Eligible Warps Per Scheduler", "Warp Cycles Per Issued Instruction", "Avg. Active Threads Per Warp",
        "Executed Ipc Active", "DRAM Throughput", "L1/TEX Hit Rate", "L2 Hit Rate", "Block Limit Registers",
        "Block Limit Shared Mem", "Dynamic Shared Memory Per Block"]


def main(rep, kre, n=25):
    det = subprocess.run(["ncu", "-i", rep, "--page", "details", "--csv", "--kernel-name", f"regex:{kre}"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(det.splitlines()))
    if rows:
        h = rows[0]
        mi, vi, ui = h.index("Metric Name"), h.index("Metric Value"), h.index("Metric Unit")
        for r in rows[1:]:
            if r[mi] in WANT:
                print(f"{r[mi]:42s} {r[vi]} {r[ui]}")
    src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass",
                          "--kernel-name", f"regex:{kre}"], capture_output=True, text=True).stdout
    hdr, fname, agg = None, None, {}
    for row in csv.reader(src.splitlines()):
        if not row:
            continue
        if row[0] == "File Path":
            fname = row[1].split("/")[-1]
            continue
        if row[0] == "Line No":
            hdr = row
            continue
        if hdr and row[0] not in ("", "Function Name"):
            d = dict(zip(hdr[2:], row[2:]))
            try:
                ex = int(d.get("Instructions Executed", "0") or 0)
                th = int(d.get("Thread Instructions Executed", "0") or 0)
                st = int(d.get("Warp Stall Sampling (All Samples)", "0") or 0)
            except ValueError:
                continue
            k = (fname, int(row[0]))
            a = agg.get(k, [0, 0, 0, row[1][:90]])
            a[0] += ex
            a[1] += th
            a[2] += st
            agg[k] = a
    tot = sum(v[0] for v in agg.values()) or 1
    ts = sum(v[2] for v in agg.values()) or 1
    print(f"# top source lines by warp-instructions (total {tot}); % instr, % stall samples, avg active lanes")
    for (f, ln), v in sorted(agg.items(), key=lambda x: -x[1][0])[:n]:
        print(f"{100 * v[0] / tot:5.1f}% {100 * v[2] / ts:5.1f}%s {v[1] / max(v[0], 1):5.1f}  {f}:{ln}  {v[3]}")


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2], int(sys.argv[3]) if len(sys.argv) > 3 else 25)
