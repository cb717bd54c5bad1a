"""One sweep call on config-5-shaped GPU-epochs for ncu captures (not a bench number)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_middleware_bhasisjgpkd24_b200._abi as A  # noqa: E402

if len(sys.argv) > 2:  # a library variant (experiments)
    A._lib = None
    A.load(os.path.abspath(sys.argv[2]))
import paper_conf_middleware_bhasisjgpkd24_b200 as pkg  # noqa: E402
from protean_inputs import epoch_batches, pack_batch_rows, synth_profiles  # noqa: E402

R = int(sys.argv[1]) if len(sys.argv) > 1 else 512
batches, off, arr, cur = epoch_batches(1000, R, 8, max_batches=8)
dev = torch.device("cuda", 0)
h = pkg.load_profiles(synth_profiles())
args = dict(n_replicas=R, n_gpus=8, batches=torch.from_numpy(pack_batch_rows(batches).copy()).to(dev),
            batch_off=torch.from_numpy(off.copy()).to(dev),
            arrival_us=torch.from_numpy(arr.view(np.int32).copy()).to(dev),
            cur_geom=torch.from_numpy(cur.copy()).to(dev))
out = h.sweep_assignments(**args)
torch.cuda.synchronize()
reps = int(os.environ.get("SWEEP_REPS", "1"))
ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
ev[0].record()
for _ in range(reps):
    h.sweep_assignments(**args)
ev[1].record()
torch.cuda.synchronize()
print(os.path.basename(sys.argv[2]) if len(sys.argv) > 2 else "libprotean.so", "assignments",
      int(out["n_assign"].item()), "ms", round(ev[0].elapsed_time(ev[1]) / reps, 2))
if os.environ.get("SWEEP_INFO"):
    import json
    json.dump({"replicas": R, "assignments": int(out["n_assign"].item())}, open(os.environ["SWEEP_INFO"], "w"))
