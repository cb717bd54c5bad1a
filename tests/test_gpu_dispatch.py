"""Dispatch (O4 round robin over the GPUs available at a batch's ready time) when not every GPU is
available all epoch: the warp path with 64-bit availability masks (N <= 64: runs of equal masks in
closed form, per-GPU lists by a warp-stable counting sort) and the serial path (N > 64), against the
oracle bit for bit.  Spot VMs with revocations and reconfiguration windows make GPUs unavailable
inside epochs.  -m gpu."""
import numpy as np
import pytest

from gpu_common import compare, gpu_replay, oracle_replay
from protean_inputs import random_profiles, uniform_trace

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("N,seed", [(31, 0), (32, 1), (33, 2), (47, 3), (63, 4), (64, 5), (65, 6), (90, 7)])
def test_dispatch_wide(oracle, N, seed):
    rng = np.random.default_rng(700 + seed)
    M = int(rng.integers(2, 6))
    prof = random_profiles(rng, M).with_geometry_set(int(rng.integers(0, 2)))
    R = int(rng.integers(1, 4))
    # many requests per epoch so most GPUs receive several batches, and runs of equal masks break
    tr = uniform_trace(rng, R, M, 6_000_000, int(rng.integers(2000, 6000)))
    cfg = dict(n_gpus=N, vm_policy=1 + seed % 2, p_rev=float(rng.choice([0.354, 0.708, 1.0])),
               rev_interval_us=1_000_000, notice_us=300_000, seed=seed,
               reconfig_us=int(rng.integers(100_000, 900_000)), wait_limit=0)
    g = gpu_replay(prof, tr, **cfg)
    o = oracle_replay(oracle, prof, tr, **cfg)
    compare(g, o, R)
    # the scenario exercises dispatch drops or partial availability
    assert (o["decisions"] != 255).any()
