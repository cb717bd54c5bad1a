"""Per-kernel ncu metrics of one protean_replay_traces call (and one sweep call) on a reduced
config-5 shape, summarised per request / per assignment into profiles/ncu_summary.json, which
bench.py reads for roofline.traffic, roofline.issue and the design's DRAM bytes per pass.

  (GPU box)  python tools/ncu_capture.py run   --replicas 444 --seconds 60
  (anywhere) python tools/ncu_capture.py parse --round r02 > profiles/ncu_summary.json

`run` writes gpurun_out/ncu_metrics.csv (+ profile_run_info.json) and gpurun_out/ncu_sweep.csv
(+ sweep_info.json); `parse` turns them into the summary.  Metric passes replay every kernel, so
the times in these files are cold-cache and serialised: only the per-request ratios are used."""
import argparse
import csv
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "gpurun_out")
METRICS = ["dram__bytes_read.sum", "dram__bytes_write.sum", "smsp__inst_executed.sum",
           "smsp__issue_active.avg.pct_of_peak_sustained_active", "smsp__warps_eligible.avg.per_cycle_active",
           "sm__warps_active.avg.pct_of_peak_sustained_active", "gpu__time_duration.sum",
           "sm__cycles_elapsed.avg.per_second", "smsp__thread_inst_executed_per_inst_executed.ratio"]
SHORT = {"replay_kernel": "replay_kernel", "prepass_kernel": "prepass", "part_count": "part_count",
         "part_scan": "part_scan", "part_scatter": "part_scatter", "sweep_kernel": "sweep_kernel",
         "walk_kernel": "walk_kernel", "cand_kernel": "cand_kernel", "chain_kernel": "chain_kernel",
         "acct_kernel": "acct_kernel"}


def run(a):
    os.makedirs(OUT, exist_ok=True)
    m = ",".join(METRICS)
    subprocess.check_call(["ncu", "--metrics", m, "--clock-control", "none", "--csv", "--log-file",
                           os.path.join(OUT, "ncu_metrics.csv"), sys.executable,
                           os.path.join(ROOT, "tools", "profile_run.py"), "--replicas", str(a.replicas),
                           "--seconds", str(a.seconds), "--repeat", "1"], cwd=ROOT)
    env = dict(os.environ, SWEEP_INFO=os.path.join(OUT, "sweep_info.json"))
    subprocess.check_call(["ncu", "--metrics", m, "--clock-control", "none", "-k", "regex:sweep_kernel", "--csv",
                           "--log-file", os.path.join(OUT, "ncu_sweep.csv"), sys.executable,
                           os.path.join(ROOT, "tools", "sweep_run.py"), str(a.sweep_replicas)], cwd=ROOT, env=env)


def _read(path):
    rows = list(csv.reader(l for l in open(path) if not l.startswith("==")))
    hdr = rows[0]
    per = {}
    for r in rows[1:]:
        d = dict(zip(hdr, r))
        name = d.get("Kernel Name", "")
        key = next((v for k, v in SHORT.items() if k in name), None)
        if key is None:
            continue
        try:
            val = float(d["Metric Value"].replace(",", ""))
        except (KeyError, ValueError):
            continue
        k = (key, d.get("ID"))
        per.setdefault(k, {})[d["Metric Name"]] = (val, d.get("Metric Unit", ""))
    agg = {}
    for (key, _), mv in per.items():  # sum extensive metrics over launches, average the rest
        a = agg.setdefault(key, {"launches": 0})
        a["launches"] += 1
        for name, (v, u) in mv.items():
            if name.endswith(".sum"):
                v = v * (1e-6 if u == "nsecond" and "time" in name else 1.0)
                a[name] = a.get(name, 0.0) + v
            else:
                a.setdefault("_avg", {}).setdefault(name, []).append(v)
    for a in agg.values():
        for name, vs in a.pop("_avg", {}).items():
            a[name] = sum(vs) / len(vs)
    return agg


def parse(a):
    info = json.load(open(os.path.join(OUT, "profile_run_info.json")))
    nreq = info["requests"]
    kern = {}
    for key, m in _read(os.path.join(OUT, "ncu_metrics.csv")).items():
        db = m.get("dram__bytes_read.sum", 0) + m.get("dram__bytes_write.sum", 0)
        kern[key] = {"launches": m["launches"], "dram_bytes_per_request": db / nreq,
                     "dram_bytes": db, "warp_instructions": m.get("smsp__inst_executed.sum"),
                     "warp_instructions_per_request": m.get("smsp__inst_executed.sum", 0) / nreq,
                     "issue_active_pct": m.get("smsp__issue_active.avg.pct_of_peak_sustained_active"),
                     "eligible_warps_per_scheduler": m.get("smsp__warps_eligible.avg.per_cycle_active"),
                     "warps_active_pct": m.get("sm__warps_active.avg.pct_of_peak_sustained_active"),
                     "active_threads_per_warp": m.get("smsp__thread_inst_executed_per_inst_executed.ratio"),
                     "sm_clock_hz": m.get("sm__cycles_elapsed.avg.per_second")}
        if key in ("replay_kernel", "cand_kernel") and info.get("slot_evals"):
            kern[key]["warp_instructions_per_slot_eval"] = m.get("smsp__inst_executed.sum", 0) / info["slot_evals"]
    out = {"report": f"{a.round}: ncu --metrics (per-kernel) of tools/profile_run.py --replicas "
                     f"{info['replicas']} --seconds {info['seconds']} (config-5 shape)",
           "workload": info, "requests": nreq, "kernels": kern}
    sp = os.path.join(OUT, "ncu_sweep.csv")
    si = os.path.join(OUT, "sweep_info.json")
    if os.path.exists(sp) and os.path.exists(si):
        s_info = json.load(open(si))
        m = _read(sp).get("sweep_kernel")
        if m:
            out["kernels"]["sweep_kernel"] = {
                "assignments": s_info["assignments"],
                "warp_instructions_per_assignment": m.get("smsp__inst_executed.sum", 0) / m["launches"]
                / s_info["assignments"],
                "issue_active_pct": m.get("smsp__issue_active.avg.pct_of_peak_sustained_active"),
                "eligible_warps_per_scheduler": m.get("smsp__warps_eligible.avg.per_cycle_active"),
                "active_threads_per_warp": m.get("smsp__thread_inst_executed_per_inst_executed.ratio"),
                "dram_bytes_per_request": None}
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("cmd", choices=["run", "parse"])
    ap.add_argument("--replicas", type=int, default=444)
    ap.add_argument("--seconds", type=int, default=60)
    ap.add_argument("--sweep-replicas", type=int, default=512)
    ap.add_argument("--round", default="r02")
    a = ap.parse_args()
    run(a) if a.cmd == "run" else parse(a)
