"""Summarise an ncu --set full capture of the partition passes (prepass, part_count, part_scan,
part_scatter) into one table: duration, DRAM bytes, achieved DRAM GB/s, issue-slot utilisation.
usage: python tools/part_summary.py <report.ncu-rep> <requests>"""
import csv
import io
import subprocess
import sys

M = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
     "smsp__issue_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum",
     "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread"]


def main(rep, n):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv", "--print-units", "base",
                          "--metrics", ",".join(M)], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h = rows[0]
    print(f"# ncu --set full, partition passes, {n} requests (tools/profile_run.py --replicas 1024 --seconds 600)")
    print(f"{'kernel':14s} {'ms':>7s} {'DRAM GB':>8s} {'GB/s':>7s} {'B/req':>6s} {'issue%':>7s} {'warps%':>7s} {'inst/req':>8s} regs")
    for r in rows[1:]:
        d = dict(zip(h, r))
        if not d.get("Kernel Name") or not d.get(M[0], "").replace(".", "").isdigit():
            continue
        ms = float(d[M[0]]) / 1e6
        b = float(d[M[1]]) + float(d[M[2]])
        print(f"{d['Kernel Name'].split('(')[0][:14]:14s} {ms:7.3f} {b / 1e9:8.2f} {b / ms / 1e6:7.0f} "
              f"{b / n:6.2f} {float(d[M[3]]):7.1f} {float(d[M[5]]):7.1f} {float(d[M[4]]) / n:8.3f} {d[M[6]]}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]))
