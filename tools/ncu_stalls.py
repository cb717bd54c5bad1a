"""Stall-reason breakdown per kernel phase of an ncu report (source page, cuda,sass view)."""
import collections
import csv
import os
import subprocess
import sys

SRC = os.path.join(os.path.dirname(__file__), "..", "paper_conf_middleware_bhasisjgpkd24_b200", "csrc", "replay.cu")


def main(rep):
    src = open(SRC).read().split("\n")
    marks = [(i + 1, l.split("----")[-1].strip()[:28]) for i, l in enumerate(src)
             if "// ----------------------------------------------------------------" in l]
    txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    hdr, fname = None, None
    agg = collections.defaultdict(collections.Counter)
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
            k = fname
            if fname == "replay.cu":
                k = "helpers"
                for i, name in marks:
                    if int(row[0]) >= i:
                        k = name
            for col, v in d.items():
                if col.startswith("stall_") and "Not Issued" not in col and v.isdigit():
                    agg[k][col[6:]] += int(v)
    tot = sum(sum(c.values()) for c in agg.values()) or 1
    for k, c in sorted(agg.items(), key=lambda x: -sum(x[1].values())):
        s = sum(c.values())
        top = ", ".join(f"{n} {100 * v / tot:.1f}" for n, v in c.most_common(4))
        print(f"{100 * s / tot:5.1f}%  {k:28s} {top}")


if __name__ == "__main__":
    main(sys.argv[1])
