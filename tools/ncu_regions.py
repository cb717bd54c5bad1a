"""Warp instructions per replica-epoch, per code region of replay.cu (regions = '// ----' phase
markers and the device functions above the kernel), from an ncu source page.  The region map is
built from the profiled source file ($PROTEAN_SRC, default: the tree's replay.cu)."""
import collections
import os
import re
import sys

sys.path.insert(0, os.path.dirname(__file__))
from ncu_lines import lines  # noqa: E402


def regions_from(src_lines):
    """src_lines: {line_no: text} of replay.cu -> [(first line, region name)] ascending."""
    marks = []
    for i in sorted(src_lines):
        l = src_lines[i]
        if "// ----------------------------------------------------------------" in l:
            marks.append((i, l.split("----")[-1].strip()[:30]))
        else:
            m = re.match(r"(?:template <[^>]*>\s*)?(?:static )?__(?:device|global)__.*?(\w+)\(", l)  # top-level only
            if m and not l.strip().startswith("//"):
                marks.append((i, m.group(1)))
    return marks


def region_of(marks, ln):
    k = "?"
    for i, name in marks:
        if ln >= i:
            k = name
    return k


def source_map(rows, fname="replay.cu"):
    """The profiled replay.cu: $PROTEAN_SRC (the file as built for the report, e.g. `git show
    <commit>:.../replay.cu`), else the tree's current file (valid when it is unchanged since)."""
    path = os.environ.get("PROTEAN_SRC") or os.path.join(os.path.dirname(__file__), "..",
                                                         "paper_conf_middleware_bhasisjgpkd24_b200", "csrc", fname)
    return {i + 1: l for i, l in enumerate(open(path).read().split("\n"))}


def main(rep, per_unit):
    rows = lines(rep)
    marks = regions_from(source_map(rows))
    agg = collections.Counter()
    for s, ex, f, ln, _ in rows:
        agg[region_of(marks, int(ln)) if f == "replay.cu" else f] += ex
    tot = sum(agg.values())
    for k, v in agg.most_common():
        print(f"{v / per_unit:9.0f} {100 * v / tot:5.1f}%  {k}")
    print(f"{tot / per_unit:9.0f} total warp-instructions per unit")


if __name__ == "__main__":
    main(sys.argv[1], float(sys.argv[2]) if len(sys.argv) > 2 else 1.0)
