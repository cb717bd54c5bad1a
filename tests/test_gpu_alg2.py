"""Policy 2 (N1, Alg 2's own heuristic): CUDA path vs the CPU oracle through the C ABI,
bit-exact on every output (decisions, counters, histograms, accumulators, per-batch log).  -m gpu."""
import json
import os

import numpy as np
import pytest

from gpu_common import compare, gpu_replay, oracle_replay
from helpers import GOLDEN, tables
from protean_inputs import concat, mix_a_params, mix_b_params, pack_meta, random_profiles, synth_profiles, \
    tick_trace, uniform_trace

pytestmark = pytest.mark.gpu


def _t12_trace():
    arr = []
    for e in range(12):
        for off in ((100_000, 300_000) if e < 4 else (100_000, 300_000, 500_000)):
            arr.append(e * 1_000_000 + off)
    n = len(arr)
    return concat([(np.array(arr, np.uint32), pack_meta(np.zeros(n, int), np.zeros(n, int)))], 12_000_000)


@pytest.mark.parametrize("alpha", [1000, 500])
def test_t12_golden_gpu(oracle, alpha):
    t12 = json.load(open(os.path.join(GOLDEN, "t12_alg2_epochs.json")))
    P = tables([[1000] * 5], [[0] * 5], [t12["model"]["mem_mib"]], bsz=[1], tmo=[0])
    tr = _t12_trace()
    cfg = dict(n_gpus=1, policy=2, ewma_alpha_pm=alpha, t_low_milli=500, t_high_milli=4000)
    g = gpu_replay(P, tr, **cfg)
    exp = t12[f"alpha_{alpha}"]
    assert g["decisions"].reshape(-1).tolist() == exp["decisions"]
    assert g["counters"][0, 7] == exp["reconfigs"] and g["counters"][0, 6] == exp["be_drop"]
    compare(g, oracle_replay(oracle, P, tr, **cfg), 1)


@pytest.mark.parametrize("seed", range(6))
def test_fuzz_alg2(oracle, seed):
    rng = np.random.default_rng(700 + seed)
    M = int(rng.integers(1, 7))
    prof = random_profiles(rng, M).with_geometry_set(int(rng.integers(0, 2)))
    N = int(rng.choice([1, 2, 3, 8]))
    R = int(rng.integers(1, 6))
    tr = uniform_trace(rng, R, M, int(rng.integers(2, 14)) * 1_000_000, int(rng.integers(5, 600)))
    lo = int(rng.integers(0, 3000))
    cfg = dict(n_gpus=N, policy=2, ewma_alpha_pm=int(rng.choice([1, 250, 500, 1000])), t_low_milli=lo,
               t_high_milli=lo + int(rng.integers(0, 6000)), max_live=int(rng.choice([2, 8, 64])),
               wait_limit=int(rng.integers(0, 4)), reconfig_us=int(rng.integers(0, 3_000_000)),
               vm_policy=int(seed % 3), p_rev=float(rng.choice([0.0, 0.354, 0.708, 1.0])),
               rev_interval_us=2_000_000, notice_us=300_000, seed=seed)
    compare(gpu_replay(prof, tr, **cfg), oracle_replay(oracle, prof, tr, **cfg), R)


def test_mix_a_alg2(oracle):
    """Config-5 shape (Mix A, 22-model table, 8 sim-GPUs), 6 replicas x 120 s, default knobs."""
    gp = mix_a_params(6, seed=3, seconds=120)
    tr = tick_trace(gp)
    P = synth_profiles()
    cfg = dict(n_gpus=8, policy=2)
    g = gpu_replay(P, tr, want_keys=False, **cfg)
    o = oracle_replay(oracle, P, tr, want_keys=False, **cfg)
    compare(g, o, tr.n_replicas, keys=False)
    dec = o["decisions"]
    assert (dec[dec != 255] == 2).any() and (dec[dec != 255] == 1).any()  # both outcomes occur
    assert o["counters"][:, 7].sum() > 0 and o["counters"][:, 8].sum() == 0


def test_mix_b_vm_alg2(oracle):
    """Config-3 shape: Mix B with spot/on-demand revocations, 2 replicas x 90 s."""
    gp = mix_b_params(2, seed=5, seconds=90)
    tr = tick_trace(gp)
    P = synth_profiles()
    for vm_policy, p_rev in [(1, 0.708), (2, 0.354)]:
        cfg = dict(n_gpus=8, policy=2, vm_policy=vm_policy, p_rev=p_rev, rev_interval_us=5_000_000,
                   notice_us=1_000_000, seed=11)
        compare(gpu_replay(P, tr, want_keys=False, **cfg), oracle_replay(oracle, P, tr, want_keys=False, **cfg),
                tr.n_replicas, keys=False)
