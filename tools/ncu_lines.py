"""Summarise an ncu report's source page: warp-stall samples per CUDA source line (top N)."""
import csv
import subprocess
import sys


def lines(rep):
    txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    rows, fname, hdr = [], None, None
    for row in csv.reader(txt.splitlines()):
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
                s = int(d.get("Warp Stall Sampling (All Samples)", "0") or 0)
                ex = int(d.get("Instructions Executed", "0") or 0)
            except ValueError:
                continue
            rows.append((s, ex, fname, row[0], row[1][:90]))
    return rows


if __name__ == "__main__":
    rep = sys.argv[1]
    n = int(sys.argv[2]) if len(sys.argv) > 2 else 40
    rows = lines(rep)
    tot = sum(r[0] for r in rows) or 1
    tex = sum(r[1] for r in rows) or 1
    print(f"total samples {tot}, warp instructions {tex}")
    for s, ex, f, ln, src in sorted(rows, reverse=True)[:n]:
        print(f"{100*s/tot:5.1f}% {100*ex/tex:5.1f}%i {f}:{ln:5s} {src}")
