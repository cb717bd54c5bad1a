"""Warp instructions per replica-epoch, per code region of replay.cu (regions = '// ----' phase
markers and the device functions above the kernel), from an ncu source page."""
import collections
import os
import re
import sys

sys.path.insert(0, os.path.dirname(__file__))
from ncu_lines import lines  # noqa: E402

SRC = os.path.join(os.path.dirname(__file__), "..", "paper_conf_middleware_bhasisjgpkd24_b200", "csrc", "replay.cu")


def regions():
    src = open(SRC).read().split("\n")
    marks = []
    for i, l in enumerate(src):
        if "// ----------------------------------------------------------------" in l:
            marks.append((i + 1, l.split("----")[-1].strip()[:30]))
        else:
            m = re.match(r"(?:template <[^>]*>\s*)?(?:static )?__(?:device|global)__.*?(\w+)\(", l)
            if m and not l.strip().startswith("//"):
                marks.append((i + 1, m.group(1)))
    return marks


def main(rep, per_unit):
    marks = regions()
    agg = collections.Counter()
    for s, ex, f, ln, _ in lines(rep):
        k = f
        if f == "replay.cu":
            k = "?"
            for i, name in marks:
                if int(ln) >= i:
                    k = name
        agg[k] += ex
    tot = sum(agg.values())
    for k, v in agg.most_common():
        print(f"{v / per_unit:9.0f} {100 * v / tot:5.1f}%  {k}")
    print(f"{tot / per_unit:9.0f} total warp-instructions per unit")


if __name__ == "__main__":
    main(sys.argv[1], float(sys.argv[2]) if len(sys.argv) > 2 else 1.0)
