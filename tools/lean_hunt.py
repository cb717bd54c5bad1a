"""Debug: the wide lean fuzz over many seeds (tests/test_gpu_lean.py::wide_case) on the GPU,
printing each seed before it runs (a hang names its seed) and every mismatch."""
import os, sys, numpy as np
sys.path.insert(0, os.getcwd()); sys.path.insert(0, os.path.join(os.getcwd(), "tests"))
os.environ["PROTEAN_LEAN"] = os.environ.get("LEANV", "2")  # 0: the fused engine, "": auto
if not os.environ["PROTEAN_LEAN"]: del os.environ["PROTEAN_LEAN"]
from oracle import oracle as O; O.build()
from gpu_common import compare, oracle_replay, GPU_LOG_DTYPE
from test_gpu_lean import wide_case
import paper_conf_middleware_bhasisjgpkd24_b200 as pkg
bad = 0; lean_n = 0
for seed in range(int(sys.argv[1]), int(sys.argv[2])):
    print("seed", seed, flush=True)
    prof, tr, cfg = wide_case(seed)
    h = pkg.load_profiles(prof, device=0)
    log_cap = max(1, int(np.max(np.diff(tr.replica_off))))
    try:
        oracle_replay(O, prof, tr, want_keys=False, want_log=False, **cfg)
    except O.OracleError:  # ERANGE (a pool above 128 containers): the GPU must say so too
        try:
            h.replay_traces_host(tr, **cfg); bad += 1; print("MISMATCH (no ERANGE)", seed, flush=True)
        except pkg.ProteanError:
            pass
        h.close(); continue
    try:
        g = h.replay_traces_host(tr, want_cand_keys=True, log_cap=log_cap, **cfg)
        s, w, a = h.last_search_ms(); lean_n += a > 0
        g["log"] = g["log"].reshape(tr.n_replicas, log_cap, 32).view(GPU_LOG_DTYPE).reshape(tr.n_replicas, log_cap)
        g["hist"] = g["hist"].view(np.uint32)
        compare(g, oracle_replay(O, prof, tr, **cfg), tr.n_replicas)
    except Exception as e:
        bad += 1; print("MISMATCH", seed, cfg, repr(e)[:300], flush=True)
    h.close()
print("done bad", bad, "lean", lean_n, flush=True)
