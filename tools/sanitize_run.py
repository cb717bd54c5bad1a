"""Small invocations of every device entry point for compute-sanitizer (racecheck / synccheck /
memcheck): config 1 (1 sim-GPU, 3 models, 200 requests; virtual ranks: 12 CTAs share the replica),
a 60 s slice of config 2 (8 sim-GPUs, 22 models, Mix B) as one replica and as 8 replicas (the
many-replica kernel instance), score_epoch on config 1's batches, and the sweep.  Each result is
checked against the oracle so a sanitizer run also proves the instrumented build computed the same.

  compute-sanitizer --tool racecheck python tools/sanitize_run.py c1
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np  # noqa: E402

from gpu_common import compare, gpu_replay, oracle_replay  # noqa: E402
from oracle import oracle as O  # noqa: E402  (test infrastructure: the parity check)
from protean_inputs import (c1_profiles, c1_trace, epoch_batches, mix_b_params, pack_batch_rows,  # noqa: E402
                            synth_profiles, tick_trace)


def main(which: str):
    O.build()
    if which == "c1":
        prof, tr = c1_profiles(), c1_trace()
        compare(gpu_replay(prof, tr, n_gpus=1), oracle_replay(O, prof, tr, n_gpus=1), 1)
        print("c1 replay ok")
    elif which == "lean":  # the lean path (cand.cu + chain.cu), forced on small Mix A replicas
        os.environ["PROTEAN_LEAN"] = "2"
        from protean_inputs import mix_a_params
        prof = synth_profiles()
        tr = tick_trace(mix_a_params(3, seed=11, seconds=12))
        compare(gpu_replay(prof, tr, n_gpus=8), oracle_replay(O, prof, tr, n_gpus=8), 3)
        print("lean replay ok")
    elif which in ("c2", "c2many"):
        prof = synth_profiles()
        R = 1 if which == "c2" else 8
        tr = tick_trace(mix_b_params(R, seed=2, seconds=60))
        compare(gpu_replay(prof, tr, n_gpus=8), oracle_replay(O, prof, tr, n_gpus=8), R)
        print(which, "replay ok")
    elif which == "sweep":
        import torch
        import paper_conf_middleware_bhasisjgpkd24_b200 as pkg
        P = synth_profiles()
        batches, off, arr, cur = epoch_batches(5, 2, 4, max_batches=5)
        dev = torch.device("cuda", 0)
        h = pkg.load_profiles(P, device=0)
        g = h.sweep_assignments(n_replicas=2, n_gpus=4, batches=torch.from_numpy(pack_batch_rows(batches).copy()).to(dev),
                                batch_off=torch.from_numpy(off.copy()).to(dev),
                                arrival_us=torch.from_numpy(arr.view(np.int32).copy()).to(dev),
                                cur_geom=torch.from_numpy(cur.copy()).to(dev), max_batches=5)
        o = O.sweep(P, R=2, N=4, batches=batches, batch_off=off, arrival=arr, cur_geom=cur, max_batches=5)
        assert g["sweep_key"].cpu().tolist() == o["sweep_key"].tolist()
        print("sweep ok")
    elif which == "score":
        import torch
        import paper_conf_middleware_bhasisjgpkd24_b200 as pkg
        from paper_conf_middleware_bhasisjgpkd24_b200 import _abi as A
        prof, tr = c1_profiles(), c1_trace()
        dev = torch.device("cuda", 0)
        h = pkg.load_profiles(prof, device=0)
        arr = torch.from_numpy(np.ascontiguousarray(tr.arrival_us).view(np.int32)).to(dev)
        meta = torch.from_numpy(np.ascontiguousarray(tr.meta)).to(dev)
        off = torch.from_numpy(np.ascontiguousarray(tr.replica_off, np.int64)).to(dev)
        fb = h.form_batches(arr, meta, off, trace_len_us=tr.trace_len_us, n_gpus=1, e_lo=0, e_hi=1)
        st = A.GpuState()
        st.geom, st.target, st.has_vm, st.vm_type = 2, 255, 1, 1
        state = torch.from_numpy(np.frombuffer(bytes(st), np.uint8).copy()).to(dev)
        out = h.score_epoch(n_replicas=1, n_gpus=1, epoch=0, batches=fb["rows"].reshape(-1),
                            batch_off=fb["batch_off"][:2].contiguous(), arrival_us=fb["members"], state=state)
        print("score_epoch ok", out["best_key"].cpu().tolist())
    else:
        raise SystemExit(f"unknown {which}")


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "c1")
