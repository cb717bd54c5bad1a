"""One replay of a reduced config-5 workload for ncu captures (not a bench number)."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_middleware_bhasisjgpkd24_b200 as pkg  # noqa: E402
from protean_inputs import mix_a_params, synth_profiles  # noqa: E402
from tools import tracegen  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--replicas", type=int, default=444)
ap.add_argument("--seconds", type=int, default=30)
ap.add_argument("--repeat", type=int, default=2)
a = ap.parse_args()
gp = mix_a_params(a.replicas, seed=1, seconds=a.seconds)
arr, meta, roff = tracegen.generate_on_device(gp, 0)
h = pkg.load_profiles(synth_profiles())
for _ in range(a.repeat):
    out = h.replay_traces(arr, meta, roff, trace_len_us=gp.trace_len_us, n_gpus=8)
torch.cuda.synchronize()
import json
c = out["counters"].sum(0).cpu().tolist()
info = {"replicas": a.replicas, "seconds": a.seconds, "requests": int(arr.shape[0]),
        "slot_evals": int(c[8]), "geom_candidates": int(c[9]), "timings": h.last_timings()[:2], "search_ms": h.last_search_ms(),
        "launch": h.last_timings()[2]}
print(json.dumps(info))
os.makedirs("gpurun_out", exist_ok=True)
json.dump(info, open("gpurun_out/profile_run_info.json", "w"))
