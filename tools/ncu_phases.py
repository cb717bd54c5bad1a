"""Instruction / stall share per kernel phase (replay.cu '// ----' markers) of an ncu report."""
import collections
import os
import sys

sys.path.insert(0, os.path.dirname(__file__))
from ncu_lines import lines  # noqa: E402

SRC = os.path.join(os.path.dirname(__file__), "..", "paper_conf_middleware_bhasisjgpkd24_b200", "csrc", "replay.cu")


def main(rep):
    src = open(SRC).read().split("\n")
    marks = [(i + 1, l.split("----")[-1].strip()[:40]) for i, l in enumerate(src)
             if "// ----------------------------------------------------------------" in l]
    rows = lines(rep)
    agg, aggs = collections.Counter(), collections.Counter()
    for s, ex, f, ln, _ in rows:
        k = f
        if f == "replay.cu":
            k = "pre/helpers"
            for i, name in marks:
                if int(ln) >= i:
                    k = name
        agg[k] += ex
        aggs[k] += s
    tex, ts = sum(agg.values()) or 1, sum(aggs.values()) or 1
    for k, v in agg.most_common():
        print(f"{100 * v / tex:5.1f}% inst {100 * aggs[k] / ts:5.1f}% stall  {k}")


if __name__ == "__main__":
    main(sys.argv[1])
