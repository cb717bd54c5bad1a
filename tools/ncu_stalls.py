"""Stall-reason breakdown per code region of replay.cu from an ncu report (source page, cuda,sass
view).  Regions are the kernel's '// ----' phase markers AND every device function definition
(tools/ncu_regions.regions_from the report's embedded source), so helper bodies above the kernel (place_group, candidate_unit_fast,
exchange_keys, ...) are attributed to themselves, not to the marker that precedes them."""
import collections
import csv
import os
import subprocess
import sys

sys.path.insert(0, os.path.dirname(__file__))
from ncu_lines import lines  # noqa: E402
from ncu_regions import region_of, regions_from, source_map  # noqa: E402


def main(rep):
    marks = regions_from(source_map(lines(rep)))
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
                k = region_of(marks, int(row[0]))
            for col, v in d.items():
                if col.startswith("stall_") and "Not Issued" not in col and v.isdigit():
                    agg[k][col[6:]] += int(v)
    tot = sum(sum(c.values()) for c in agg.values()) or 1
    for k, c in sorted(agg.items(), key=lambda x: -sum(x[1].values())):
        s = sum(c.values())
        top = ", ".join(f"{n} {100 * v / tot:.1f}" for n, v in c.most_common(4))
        print(f"{100 * s / tot:5.1f}%  {k:30s} {top}")


if __name__ == "__main__":
    main(sys.argv[1])
