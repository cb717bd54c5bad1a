"""Single-replica configs (C2: 8 sim-GPUs x 3600 s, Mix B, G = 12; C4: 64 sim-GPUs x 600 s, Mix B
at 8x rates, G = 37) on one B200: one CTA (mode R, 1 rank) vs mode G with n in-process ranks
sharing the GPU (n CTAs exchanging min-loc keys per epoch over device memory); the CPU oracle on
one thread beside it.  Experiments for DESIGN §7 (not the bench line)."""
import json
import os
import sys
import threading
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")  # in-process mode-G ranks, before CUDA init
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_middleware_bhasisjgpkd24_b200 as pkg  # noqa: E402
from protean_inputs import mix_b_params, synth_profiles, tick_trace  # noqa: E402


def run(prof, tr, N, nranks, reps=3):
    dev = torch.device("cuda", 0)
    hs = [pkg.load_profiles(prof, device=0) for _ in range(nranks)]
    if nranks > 1:
        pkg.Handle.xchg_attach(hs, 1, N)
    arr = torch.from_numpy(np.ascontiguousarray(tr.arrival_us).view(np.int32)).to(dev)
    meta = torch.from_numpy(np.ascontiguousarray(tr.meta)).to(dev)
    off = torch.from_numpy(np.ascontiguousarray(tr.replica_off, np.int64)).to(dev)
    E = hs[0].num_epochs(tr.trace_len_us)
    outs = [h.alloc_replay_out(1, E, N) for h in hs]
    streams = [torch.cuda.Stream(device=dev) for _ in range(nranks)]
    best = None
    for _ in range(reps):
        torch.cuda.synchronize()

        errs = [None] * nranks

        def go(k):
            kw = dict(shard_mode=1, rank=k, nranks=nranks, max_ctas=1) if nranks > 1 else {}
            try:
                hs[k].replay_traces(arr, meta, off, trace_len_us=tr.trace_len_us, out=outs[k], stream=streams[k],
                                    n_gpus=N, **kw)
            except Exception as e:  # noqa: BLE001
                errs[k] = e
        t0 = time.perf_counter()
        th = [threading.Thread(target=go, args=(k,)) for k in range(nranks)]
        for t in th:
            t.start()
        for t in th:
            t.join()
        torch.cuda.synchronize()
        dt = time.perf_counter() - t0
        for e in errs:
            if e is not None:
                raise e
        kern = max(h.last_timings()[1] for h in hs)
        best = (dt, kern) if best is None or dt < best[0] else best
    dec = outs[0]["decisions"].cpu().numpy()
    return best, dec


def main():
    prof = synth_profiles()
    res = {}
    for name, gp, N, gs in (("C2", mix_b_params(1, seed=2, seconds=3600), 8, 0),
                            ("C4", mix_b_params(1, seed=4, seconds=600, scale=8.0), 64, 1)):
        tr = tick_trace(gp)
        P = prof.with_geometry_set(gs)
        row = {"requests": int(tr.arrival_us.shape[0])}
        ref = None
        for n in (1, 2, 4, 8):
            (dt, kern), dec = run(P, tr, N, n)
            if ref is None:
                ref = dec
            assert np.array_equal(dec, ref), "mode G decisions differ from 1 rank"
            row[f"ranks_{n}"] = {"wall_ms": round(dt * 1e3, 1), "replay_kernel_ms": round(kern, 1)}
        if "--oracle" in sys.argv:
            from oracle import oracle as O
            t0 = time.perf_counter()
            O.replay(P, tr, N=N, nthreads=1)
            row["oracle_1thread_s"] = round(time.perf_counter() - t0, 2)
        res[name] = row
        print(name, json.dumps(row), flush=True)
    os.makedirs("gpurun_out", exist_ok=True)
    json.dump(res, open("gpurun_out/single_replica.json", "w"), indent=1)


if __name__ == "__main__":
    main()
