"""Kernel time of one replay per (replicas, seconds, policy) on a C5-shaped workload (experiments)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_middleware_bhasisjgpkd24_b200 as pkg  # noqa: E402
from protean_inputs import mix_a_params, synth_profiles  # noqa: E402
from tools import tracegen  # noqa: E402

h = pkg.load_profiles(synth_profiles())
for spec in sys.argv[1:]:
    R, S, pol = (int(x) for x in spec.split(":"))
    gp = mix_a_params(R, seed=1, seconds=S)
    arr, meta, roff = tracegen.generate_on_device(gp, 0)
    ts = []
    for _ in range(3):
        out = h.replay_traces(arr, meta, roff, trace_len_us=gp.trace_len_us, n_gpus=8, policy=pol)
        torch.cuda.synchronize()
        ts.append(h.last_timings()[1])
    c = out["counters"].sum(0).cpu().tolist()
    print(json.dumps({"R": R, "S": S, "policy": pol, "kernel_ms": [round(t, 2) for t in ts[1:]],
                      "reconfigs": c[7], "drops": c[3] + c[6], "req": c[0] + c[4]}), flush=True)
    del arr, meta, roff, out
