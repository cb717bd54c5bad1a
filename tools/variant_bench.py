"""Kernel time of a libprotean build variant on a reduced C5 shape (experiments; not a bench line).
usage: python tools/variant_bench.py LIB.so [replicas] [seconds]   (env knobs pass through)"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_middleware_bhasisjgpkd24_b200._abi as A  # noqa: E402

A._lib = None
A.load(os.path.abspath(sys.argv[1]))
import torch  # noqa: E402

import paper_conf_middleware_bhasisjgpkd24_b200 as pkg  # noqa: E402
from protean_inputs import mix_a_params, synth_profiles  # noqa: E402
from tools import tracegen  # noqa: E402

R = int(sys.argv[2]) if len(sys.argv) > 2 else 4096
S = int(sys.argv[3]) if len(sys.argv) > 3 else 60
POL = int(os.environ.get("PROTEAN_VB_POLICY", "0"))
gp = mix_a_params(R, seed=1, seconds=S)
arr, meta, roff = tracegen.generate_on_device(gp, 0)
h = pkg.load_profiles(synth_profiles())
ts = []
for _ in range(4):
    out = h.replay_traces(arr, meta, roff, trace_len_us=gp.trace_len_us, n_gpus=8, ewma_alpha_pm=0 if POL != 2 else 500, policy=POL)  # 0: also the reserved word of pre-N1 builds
    torch.cuda.synchronize()
    ts.append(h.last_timings()[1])
c = out["counters"].sum(0).cpu().tolist()
print(json.dumps({"lib": os.path.basename(sys.argv[1]), "env": {k: v for k, v in os.environ.items() if k.startswith("PROTEAN")},
                  "kernel_ms": [round(t, 3) for t in ts[1:]], "search_walk_acct_ms": [round(t, 3) for t in h.last_search_ms()], "launch": h.last_timings()[2], "slot_evals": c[8]}))
