"""Summarise one tools/gpu_measure.sh run (gpurun_out/) into profiles/<tag>_*: the bench line, the
ncu launch list (per-kernel durations and the replay kernel's share of the step), the ncu --set full
capture (headline metrics, stall breakdown, top lines, warp instructions per code region) and
profiles/ncu_summary.json (DRAM bytes per request, read by bench.py as roofline.traffic).
usage: python tools/make_profiles.py <tag>"""
import contextlib
import csv
import io
import json
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
sys.path.insert(0, HERE)
import ncu_regions  # noqa: E402
import ncu_stalls  # noqa: E402
import ncu_summary  # noqa: E402

OUT = os.path.join(ROOT, "gpurun_out")
PROF = os.path.join(ROOT, "profiles")


def main(tag):
    line = open(os.path.join(OUT, "bench_full.log")).read().strip().splitlines()[-1]
    json.dump(json.loads(line), open(os.path.join(PROF, f"{tag}_bench_line.json"), "w"), indent=1)
    rows, hdr = [], None
    for r in csv.reader(open(os.path.join(OUT, "launches.csv"))):
        if r and r[0] == "ID":
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            rows.append((d["Kernel Name"], float(d["Metric Value"]) / 1e6))
    with open(os.path.join(PROF, f"{tag}_launches.csv"), "w") as f:
        f.write("kernel,ms\n")
        for k, ms in rows:
            f.write(f"\"{k[:80]}\",{ms:.4f}\n")
    rep = [ms for k, ms in rows if "replay_kernel" in k]
    pre = [ms for k, ms in rows if "prepass_kernel" in k]
    parts = {n: [ms for k, ms in rows if n in k] for n in ("part_count", "part_scan", "part_scatter")}
    step = [a + b + sum(parts[n][i] for n in parts) for i, (a, b) in enumerate(zip(pre, rep))]
    json.dump({"command": "ncu --metrics gpu__time_duration.sum --clock-control none python bench.py "
                          "--steps 2 --warmup 1 --cpu-sample 0 --e2e-replicas 0",
               "replay_kernel_ms": rep, "prepass_ms": pre, **{f"{n}_ms": v for n, v in parts.items()},
               "replay_share_of_step": sum(rep) / sum(step) if step else None,
               "note": "cold-cache, serialised per-launch times; compare shares, not absolutes"},
              open(os.path.join(PROF, f"{tag}_launch_summary.json"), "w"), indent=1)
    ncu = os.path.join(OUT, "replay_full.ncu-rep")
    info = json.load(open(os.path.join(OUT, "profile_run_info.json")))
    buf = io.StringIO()
    with contextlib.redirect_stdout(buf):
        print(f"# ncu --set full, replay_kernel, tools/profile_run.py --replicas {info['replicas']} "
              f"--seconds {info['seconds']} (config-5 shape)")
        ncu_summary.main(ncu, 30)
        print("\n# stall reasons per code region")
        ncu_stalls.main(ncu)
        print(f"\n# warp instructions per replica-epoch, per code region")
        ncu_regions.main(ncu, info["replicas"] * (info["seconds"] + 1))
    open(os.path.join(PROF, f"{tag}_replay_kernel_ncu_full.txt"), "w").write(buf.getvalue())
    raw = subprocess.run(["ncu", "-i", ncu, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rr = list(csv.reader(raw.splitlines()))
    h, v = rr[0], rr[2]
    get = lambda n: float(v[h.index(n)].replace(",", ""))
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
    unit_r = rr[1][h.index("dram__bytes_read.sum")]
    unit_w = rr[1][h.index("dram__bytes_write.sum")]
    rd = get("dram__bytes_read.sum") * scale.get(unit_r, 1)
    wr = get("dram__bytes_write.sum") * scale.get(unit_w, 1)
    dur = get("gpu__time_duration.sum")
    s = {"report": f"{tag} replay_kernel ncu --set full", "workload": f"tools/profile_run.py --replicas "
         f"{info['replicas']} --seconds {info['seconds']} (config-5 shape)", "requests": info["requests"],
         "dram_bytes_read": rd, "dram_bytes_write": wr,
         "dram_bytes_per_request": (rd + wr) / info["requests"], "algorithmic_bytes_per_request": 4.0,
         "duration_ms_under_ncu": dur / 1e6 if dur > 1e4 else dur,
         "issue_active_pct": get("smsp__issue_active.avg.pct_of_peak_sustained_active"),
         "warp_instructions": get("smsp__inst_executed.sum")}
    json.dump(s, open(os.path.join(PROF, "ncu_summary.json"), "w"), indent=1)
    print(json.dumps(s, indent=1))


if __name__ == "__main__":
    main(sys.argv[1])
