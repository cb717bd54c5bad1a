"""Probe: n in-process mode-G ranks on cuda:0 (threads + streams), timing each rank's call."""
import os
import sys
import threading
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_middleware_bhasisjgpkd24_b200 as pkg  # noqa: E402
from protean_inputs import mix_a_params, synth_profiles, tick_trace  # noqa: E402

nranks = int(sys.argv[1]) if len(sys.argv) > 1 else 2
R = int(sys.argv[2]) if len(sys.argv) > 2 else 1
secs = int(sys.argv[3]) if len(sys.argv) > 3 else 3
prof = synth_profiles()
tr = tick_trace(mix_a_params(R, seed=21, seconds=secs))
dev = torch.device("cuda", 0)
arr = torch.from_numpy(np.ascontiguousarray(tr.arrival_us).view(np.int32)).to(dev)
meta = torch.from_numpy(np.ascontiguousarray(tr.meta)).to(dev)
off = torch.from_numpy(np.asarray(tr.replica_off, np.int64)).to(dev)
hs = [pkg.load_profiles(prof) for _ in range(nranks)]
# mode-R warm-up on every handle (loads modules, sizes scratch)
for h in hs:
    h.replay_traces(arr, meta, off, trace_len_us=tr.trace_len_us, n_gpus=8)
torch.cuda.synchronize()
pkg.Handle.xchg_attach(hs, R, 8)
streams = [torch.cuda.Stream(device=dev) for _ in range(nranks)]
E = hs[0].num_epochs(tr.trace_len_us)
outs = [h.alloc_replay_out(R, E, 8) for h in hs]
torch.cuda.synchronize()
res = [None] * nranks


def run(k):
    t0 = time.time()
    try:
        hs[k].replay_traces(arr, meta, off, trace_len_us=tr.trace_len_us, out=outs[k], stream=streams[k],
                            shard_mode=1, rank=k, nranks=nranks, max_ctas=min(R, 8), n_gpus=8)
        res[k] = ("ok", time.time() - t0)
    except Exception as e:  # noqa: BLE001
        res[k] = (repr(e), time.time() - t0)


th = [threading.Thread(target=run, args=(k,)) for k in range(nranks)]
for t in th:
    t.start()
for t in th:
    t.join()
print("XCHG_OFF" if os.environ.get("PROTEAN_XCHG_OFF") else "XCHG_ON", res, flush=True)
if all(r[0] == "ok" for r in res):
    d = [o["decisions"].cpu().numpy() for o in outs]
    print("decisions equal across ranks:", all(np.array_equal(d[0], x) for x in d))
