"""One single-replica Mix-B replay (config-2 shape) for ncu captures (not a bench number)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_middleware_bhasisjgpkd24_b200._abi as A  # noqa: E402

if os.environ.get("PROTEAN_LIB"):  # a library variant (experiments)
    A._lib = None
    A.load(os.path.abspath(os.environ["PROTEAN_LIB"]))
import paper_conf_middleware_bhasisjgpkd24_b200 as pkg  # noqa: E402
from protean_inputs import mix_b_params, synth_profiles, tick_trace  # noqa: E402

S = int(sys.argv[1]) if len(sys.argv) > 1 else 120
tr = tick_trace(mix_b_params(1, seed=2, seconds=S))
dev = torch.device("cuda", 0)
arr = torch.from_numpy(np.ascontiguousarray(tr.arrival_us).view(np.int32)).to(dev)
meta = torch.from_numpy(np.ascontiguousarray(tr.meta)).to(dev)
off = torch.from_numpy(np.ascontiguousarray(tr.replica_off, np.int64)).to(dev)
h = pkg.load_profiles(synth_profiles())
POL = int(sys.argv[2]) if len(sys.argv) > 2 else 0
out = h.replay_traces(arr, meta, off, trace_len_us=tr.trace_len_us, n_gpus=8, policy=POL)
torch.cuda.synchronize()
print("replay ms", h.last_timings()[1], "launch", h.last_timings()[2])
