"""Debug: mode G (geometry ranges, in-process ranks on cuda:0, the in-kernel key exchange) on the
wide random cases of tests/test_gpu_lean.py::wide_case (policy 0 only: mode G shards the search),
every rank and the merged result compared with the oracle; prints each seed first."""
import os, sys, numpy as np
sys.path.insert(0, os.getcwd()); sys.path.insert(0, os.path.join(os.getcwd(), "tests"))
os.environ.setdefault("PROTEAN_XCHG_TIMEOUT_S", "10")
from oracle import oracle as O; O.build()
from gpu_common import oracle_replay
from test_gpu_lean import wide_case
from test_gpu_modeg import modeg_replay, _check_ranks
bad = n = 0
for seed in range(int(sys.argv[1]), int(sys.argv[2])):
    prof, tr, cfg = wide_case(seed)
    cfg["policy"] = 0
    for k in ("ewma_alpha_pm", "t_low_milli", "t_high_milli"):
        cfg.pop(k, None)
    nr = 2 + seed % 3
    print("seed", seed, "ranks", nr, flush=True)
    try:
        o = oracle_replay(O, prof, tr, **cfg)
    except O.OracleError:
        continue
    try:
        res, bounds = modeg_replay(prof, tr, nr, **cfg)
        host, merged = res[0]
        _check_ranks(host, merged, o, tr.n_replicas, bounds)
        n += 1
    except Exception as e:
        bad += 1; print("MISMATCH", seed, nr, cfg, repr(e)[:300], flush=True)
print("done bad", bad, "ok", n, flush=True)
