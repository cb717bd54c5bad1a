"""N3 (the Autoscaler's container pools: cold starts, delayed termination):
CUDA replay vs the CPU oracle, bit-exact on every output including the cold-start counts.  -m gpu."""
import json
import os

import numpy as np
import pytest

from gpu_common import compare, gpu_replay, oracle_replay
from helpers import GOLDEN, tables, trace_from
from protean_inputs import concat, mix_a_params, mix_b_params, pack_meta, random_profiles, synth_profiles, \
    tick_trace, uniform_trace

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("case,kw", [("keepalive_2", dict(keepalive_epochs=2)),
                                     ("keepalive_600", dict(keepalive_epochs=600)),
                                     ("prewarm_2", dict(keepalive_epochs=600, prewarm=2))])
def test_t14_golden_gpu(oracle, case, kw):
    g = json.load(open(os.path.join(GOLDEN, "t14_cold_start.json")))
    m = g["model"]
    P = tables([m["solo_us"]], [m["fbr_ppm"]], [m["mem_mib"]], bsz=[m["batch_size"]], slo=[m["slo_us"]],
               tmo=[m["timeout_us"]])
    a = np.array(g["trace"]["arrival_us"], np.uint32)
    tr = concat([(a, pack_meta(np.zeros(a.size, int), np.full(a.size, m["strict"])))], g["trace"]["trace_len_us"])
    cfg = dict(n_gpus=1, cold_start_us=g["cold_us"], **kw)
    out = gpu_replay(P, tr, **cfg)
    assert out["cold_starts"][0] == g[case]["cold_starts"]
    assert out["counters"][0, 1] == g[case]["strict_met"]
    compare(out, oracle_replay(oracle, P, tr, **cfg), 1)


@pytest.mark.parametrize("seed", range(6))
def test_fuzz_cold_starts(oracle, seed):
    rng = np.random.default_rng(2100 + seed)
    M = int(rng.integers(1, 6))
    prof = random_profiles(rng, M).with_geometry_set(int(rng.integers(0, 2)))
    N = int(rng.choice([1, 2, 3, 8]))
    R = int(rng.integers(1, 5))
    tr = uniform_trace(rng, R, M, int(rng.integers(3, 14)) * 1_000_000, int(rng.integers(20, 800)))
    cfg = dict(n_gpus=N, policy=int(rng.choice([0, 1, 2])), cold_start_us=int(rng.integers(1, 400_000)),
               keepalive_epochs=int(rng.integers(1, 4)), prewarm=int(rng.integers(0, 3)),
               max_live=int(rng.choice([2, 8, 64])), vm_policy=int(seed % 3),
               p_rev=float(rng.choice([0.354, 0.708, 1.0])), rev_interval_us=2_000_000, notice_us=300_000,
               seed=seed)
    compare(gpu_replay(prof, tr, **cfg), oracle_replay(oracle, prof, tr, **cfg), R)


def test_mix_a_cold_starts(oracle):
    """Config-5 shape (Mix A, 22 models, 8 sim-GPUs) with 2 s cold starts and a 30-epoch keep-alive,
    4 replicas x 90 s; the GPU's count of cold starts matches the oracle's and is non-trivial."""
    tr = tick_trace(mix_a_params(4, seed=9, seconds=90))
    P = synth_profiles()
    cfg = dict(n_gpus=8, cold_start_us=2_000_000, keepalive_epochs=30)
    g = gpu_replay(P, tr, want_keys=False, **cfg)
    o = oracle_replay(oracle, P, tr, want_keys=False, **cfg)
    compare(g, o, tr.n_replicas, keys=False)
    assert o["cold_starts"].min() > 8


def test_mix_b_spot_only_pool_resets(oracle):
    """Spot-Only node losses reset the pools (R27): Mix B with revocations, 2 replicas x 60 s."""
    tr = tick_trace(mix_b_params(2, seed=6, seconds=60))
    P = synth_profiles()
    cfg = dict(n_gpus=8, cold_start_us=500_000, keepalive_epochs=5, vm_policy=2, p_rev=0.708,
               rev_interval_us=5_000_000, notice_us=1_000_000, seed=3)
    compare(gpu_replay(P, tr, want_keys=False, **cfg), oracle_replay(oracle, P, tr, want_keys=False, **cfg),
            tr.n_replicas, keys=False)


def test_n3_error_codes(oracle):
    import paper_conf_middleware_bhasisjgpkd24_b200 as pkg
    P = tables([[1000] * 5], [[0] * 5], [100])
    tr = trace_from([(5, 0, 1), (7, 0, 0)], 1_000_000)
    for kw in (dict(cold_start_us=-1), dict(keepalive_epochs=0), dict(prewarm=-1), dict(prewarm=129),
               dict(cold_start_us=10, prewarm=128)):
        try:
            pkg.load_profiles(P).replay_traces_host(tr, n_gpus=1, **kw)
            gc = 0
        except pkg.ProteanError as e:
            gc = e.code
        try:
            oracle_replay(oracle, P, tr, want_keys=False, want_log=False, n_gpus=1, **kw)
            oc = 0
        except oracle.OracleError as e:
            oc = e.code
        assert gc == oc, (kw, gc, oc)
