"""Helpers for the -m gpu parity tests: run the CUDA path and the CPU oracle on the same seeded
inputs and compare element by element (bit-exact; cost/util within 1e-6 relative)."""
import ctypes as C

import numpy as np

NB = 3328
GPU_LOG_DTYPE = np.dtype([("ready", "<u4"), ("epoch", "<u4"), ("n", "<u2"), ("model", "u1"),
                          ("strict", "u1"), ("gpu", "u1"), ("slice", "u1"), ("dropped", "u1"),
                          ("pad", "u1"), ("start", "<i8"), ("end", "<i8")])


def gpu_replay(prof, trace, *, want_keys=True, want_log=True, **cfg):
    import paper_conf_middleware_bhasisjgpkd24_b200 as pkg
    h = pkg.load_profiles(prof, device=0)
    log_cap = 0
    if want_log:
        log_cap = max(1, int(np.max(np.diff(trace.replica_off))) if trace.n_replicas else 1)
    out = h.replay_traces_host(trace, want_cand_keys=want_keys, log_cap=log_cap, **cfg)
    h.close()
    if want_log:
        out["log"] = out["log"].reshape(trace.n_replicas, log_cap, 32).view(GPU_LOG_DTYPE).reshape(
            trace.n_replicas, log_cap)
    out["hist"] = out["hist"].view(np.uint32)
    return out


ORACLE_CFG_KEYS = {"n_gpus": "N", "epoch_len_us": "W", "reconfig_cap_pct": "cap_pct",
                   "price_od_node_hr": "price_od", "price_spot_node_hr": "price_spot",
                   "rev_interval_us": "rev_interval", "notice_us": "notice", "t_low_milli": "t_low",
                   "t_high_milli": "t_high", "cold_start_us": "cold_us"}


def oracle_replay(O, prof, trace, *, want_keys=True, want_log=True, nthreads=8, **cfg):
    oc = {ORACLE_CFG_KEYS.get(k, k): v for k, v in cfg.items()}
    return O.replay(prof, trace, want_keys=want_keys, want_log=want_log, nthreads=nthreads, **oc)


def compare(g, o, R, *, keys=True, log=True):
    for k in ("counters", "accum", "p50_p99", "decisions"):
        a, b = np.asarray(g[k]), np.asarray(o[k])
        assert a.shape == b.shape, (k, a.shape, b.shape)
        if not np.array_equal(a, b):
            bad = np.argwhere(a != b)[:5]
            raise AssertionError(f"{k} mismatch at {bad.tolist()}: gpu {a[tuple(bad[0])]} oracle {b[tuple(bad[0])]}")
    assert np.array_equal(g["hist"], o["hist"]), "hist mismatch"
    assert np.array_equal(g["n_batches"], o["n_batches"]), "n_batches mismatch"
    assert np.array_equal(g["cold_starts"], o["cold_starts"]), "cold_starts mismatch"
    np.testing.assert_allclose(g["cost"], o["cost"], rtol=1e-6, atol=0)
    np.testing.assert_allclose(g["util"], o["util"], rtol=1e-6, atol=0)
    assert np.array_equal(g["cost"], o["cost"]) and np.array_equal(g["util"], o["util"])
    if keys:
        a, b = g["cand_keys"], o["cand_keys"]
        if not np.array_equal(a, b):
            bad = np.argwhere(a != b)[:5]
            raise AssertionError(f"cand_keys mismatch at {bad.tolist()}: gpu {a[tuple(bad[0])]} oracle {b[tuple(bad[0])]}")
    if log:
        for r in range(R):
            n = int(o["n_batches"][r])
            gl, ol = g["log"][r][:n], o["log"][r][:n]
            for f in ("ready", "epoch", "n", "model", "strict", "gpu", "slice", "dropped", "start", "end"):
                ga = gl[f].astype(np.int64)
                oa = ol[f].astype(np.int64)
                if f in ("gpu", "slice"):
                    oa = np.where(oa < 0, 255, oa)
                if not np.array_equal(ga, oa):
                    i = int(np.argwhere(ga != oa)[0][0])
                    raise AssertionError(f"log field {f} replica {r} row {i}: gpu {gl[i]} oracle {ol[i]}")
