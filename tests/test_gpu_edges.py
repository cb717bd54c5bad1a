"""Targeted edge cases of PEM on the GPU (-m gpu), each bit-exact against the oracle on every output
(counters, accumulators, histograms, percentiles, decisions, every candidate key, the batch log),
and each asserting that its edge actually occurs (test plan 292-295):

* arrivals and batch ready times exactly at epoch starts eW (half-open epochs, reading Q31);
* Eq 1's co-runner sum exactly 10^6 (max(F, 10^6) boundary, reading Q9/Q10);
* a batch ready exactly at recfg_end (dispatch allowed, install before Place, O5.3, Q24);
* revocation boundaries at an epoch start and inside an epoch (O11, reading R4);
* epochs shorter than the largest batch timeout (W = 20 ms < T_m: open batches span several
  epochs; the prepass's window search from the replica start, the maxT > W branch)."""
import numpy as np
import pytest

from gpu_common import compare, gpu_replay, oracle_replay
from helpers import tables, trace_from, w1
from protean_inputs import random_profiles, uniform_trace

pytestmark = pytest.mark.gpu


def _both(oracle, P, tr, **cfg):
    g = gpu_replay(P, tr, **cfg)
    o = oracle_replay(oracle, P, tr, **cfg)
    compare(g, o, tr.n_replicas)
    return o


def test_arrivals_and_ready_at_epoch_starts(oracle):
    W = 1_000_000
    # model 0: B = 2, timeout 0 -> batches ready at their last arrival; model 1: B = 4, timeout
    # 250,000 -> a lone request at 750,000 times out exactly at the epoch start 1,000,000
    P = tables([[300_000, 200_000, 150_000, 120_000, 100_000]] * 2, [[500_000] * 5] * 2, [4096, 6144],
               bsz=[2, 4], slo=[400_000, 400_000], tmo=[0, 250_000])
    rows = [(0, 0, 1), (W, 0, 1), (W, 0, 0), (2 * W, 0, 1), (750_000, 1, 1), (1_750_000, 1, 0),
            (2 * W - 1, 0, 0), (2 * W, 0, 0), (3 * W, 1, 1)]
    tr = trace_from(rows, 4 * W)
    o = _both(oracle, P, tr, n_gpus=2, epoch_len_us=W)
    log = o["log"][0][: o["n_batches"][0]]
    assert any(int(b["ready"]) == W and int(b["epoch"]) == 1 for b in log)
    assert any(int(b["ready"]) == 2 * W and int(b["epoch"]) == 2 for b in log)


def test_fbr_sum_exactly_one(oracle):
    """Two co-runners whose FBRs sum to exactly 10^6 run at Solo; one ppm more slows the second by
    solo x 10^-6 (solo 10^7 us, so the extra ppm is visible after the floor)."""
    for extra, want in ((0, 10_000_000), (1, 10_000_010)):
        P = tables([[10_000_000] * 5, [10_000_000] * 5], [[400_000] * 5, [600_000 + extra] * 5],
                   [4096, 4096], bsz=[1, 1], slo=[50_000_000, 50_000_000], tmo=[0, 0], geoms=[[4], [2, 3]])
        tr = trace_from([(0, 0, 1), (10_000, 1, 1)], 1_000_000)
        o = _both(oracle, P, tr, n_gpus=1, init_geom=0, epoch_len_us=1_000_000)
        log = o["log"][0][: o["n_batches"][0]]
        assert int(log[1]["end"]) - int(log[1]["start"]) == want


def test_ready_exactly_at_reconfiguration_end(oracle):
    """W1 on (4g,2g,1g); wait_limit 0 opens [1e6, 1.1e6) at the end of epoch 0 (best = (7g));
    a batch ready exactly at recfg_end = 1.1e6 is dispatched and placed on the installed (7g)."""
    g, P, _ = w1()
    base = [tuple(r) for r in g["requests"]]
    rows = base + [(1_020_000, 0, 1), (1_030_000, 0, 1), (1_050_000, 1, 0), (1_100_000, 1, 0)]
    tr = trace_from(rows, 2_000_000)
    o = _both(oracle, P, tr, n_gpus=1, init_geom=2, wait_limit=0, reconfig_us=100_000)
    log = o["log"][0][: o["n_batches"][0]]
    at_end = [b for b in log if int(b["ready"]) == 1_100_000]
    assert at_end and all(int(b["dropped"]) == 0 and int(b["start"]) >= 1_100_000 for b in at_end)
    assert any(int(b["ready"]) < 1_100_000 and int(b["dropped"]) == 1 for b in log)  # inside the window
    assert o["counters"][0, 7] == 1


@pytest.mark.parametrize("rev_s", [5.0, 2.5])
@pytest.mark.parametrize("vm_policy", [1, 2])
def test_revocation_at_and_inside_epochs(oracle, rev_s, vm_policy):
    rng = np.random.default_rng(77)
    P = random_profiles(rng, 4, max_batch=6)
    tr = uniform_trace(rng, 2, 4, 30_000_000, 400)
    _both(oracle, P, tr, n_gpus=4, vm_policy=vm_policy, p_rev=0.6, rev_interval_us=int(rev_s * 1e6),
          notice_us=1_000_000, seed=11)


@pytest.mark.parametrize("seed", range(3))
def test_epochs_shorter_than_batch_timeouts(oracle, seed):
    """W = 20 ms with batch timeouts up to 100 ms: a batch stays open across several epochs and the
    prepass bounds every epoch's window from the replica start (maxT > W)."""
    rng = np.random.default_rng(300 + seed)
    M = 4
    P = random_profiles(rng, M, max_batch=6)
    P.timeout_us[:] = rng.integers(20_000, 100_000, M)
    P.slo_us[:] = np.maximum(P.slo_us, 3 * P.timeout_us)
    tr = uniform_trace(rng, 3, M, 2_000_000, 300)
    o = _both(oracle, P, tr, n_gpus=3, epoch_len_us=20_000)
    assert int(P.timeout_us.max()) > 20_000 and o["decisions"].shape[1] > 100
