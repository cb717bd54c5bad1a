"""Pins of the oracle's form_dispatch helper (O3 batch formation + O5.2 round-robin dispatch for
an epoch range, SURVEY §8(b) protean_form_batches): agreement with the replay's own batch log (a
separate statement of the dispatch loop), a hand-derived example with an availability window, and
the formation invariants (readings Q14, Q18, Q31)."""
import numpy as np
import pytest

from helpers import tables, trace_from
from protean_inputs import mix_b_params, random_profiles, synth_profiles, tick_trace, uniform_trace
from oracle import oracle


def _by_epoch_gpu(f, R, Ew, N):
    out = {}
    for r in range(R):
        for e in range(Ew):
            for g in range(N):
                k = (r * Ew + e) * N + g
                lo, hi = f["batch_off"][k], f["batch_off"][k + 1]
                out[(r, e, g)] = [(int(f["ready"][i]), int(f["n"][i]), int(f["model"][i]), int(f["strict"][i]))
                                  for i in range(lo, hi)]
    return out


def test_matches_replay_log(oracle):
    rng = np.random.default_rng(51)
    for trial in range(6):
        M = int(rng.integers(1, 5))
        P = random_profiles(rng, M)
        N = int(rng.integers(1, 5))
        tr = uniform_trace(rng, 3, M, 6_000_000, 300)
        E = oracle.num_epochs(P, tr.trace_len_us, 1_000_000)
        e_lo, e_hi = int(rng.integers(0, 3)), E
        f = oracle.form_dispatch(P, tr, N=N, e_lo=e_lo, e_hi=e_hi)
        o = oracle.replay(P, tr, N=N, policy=1, want_log=True)  # fixed geometry: every GPU always available
        got = _by_epoch_gpu(f, tr.n_replicas, e_hi - e_lo, N)
        for r in range(tr.n_replicas):
            log = o["log"][r][: int(o["n_batches"][r])]
            for e in range(e_lo, e_hi):
                for g in range(N):
                    sel = (log["epoch"] == e) & (log["gpu"] == g)
                    exp = [(int(a), int(b), int(c), int(d)) for a, b, c, d in
                           zip(log["ready"][sel], log["n"][sel], log["model"][sel], log["strict"][sel])]
                    assert got[(r, e - e_lo, g)] == exp


def test_members_and_closing_rule(oracle):
    P = synth_profiles()
    tr = tick_trace(mix_b_params(1, seed=3, seconds=6))
    E = oracle.num_epochs(P, tr.trace_len_us, 1_000_000)
    f = oracle.form_dispatch(P, tr, N=8, e_lo=0, e_hi=E)
    arr = np.asarray(tr.arrival_us)
    for i in range(len(f["ready"])):
        mem = f["members"][f["req_off"][i]: f["req_off"][i] + f["n"][i]]
        m = f["model"][i]
        assert (np.diff(mem.astype(np.int64)) >= 0).all() and mem[-1] <= f["ready"][i]
        if f["n"][i] == P.batch_size[m]:
            assert f["ready"][i] == mem[-1]                   # full batch closes on its last member
        else:
            assert f["ready"][i] == mem[0] + P.timeout_us[m]  # otherwise at first arrival + T_m (Q14)
    assert int(f["n"].sum()) == arr.shape[0]                  # every request in exactly one batch


def test_availability_window_example(oracle):
    # T15 (hand-derived): 2 GPUs, batch size 1, requests at 0.1, 0.2, 0.6, 0.7, 1.6 s (model 0,
    # strict).  (a) GPU 1 available only in [0, 0.5 s): round-robin from cursor 0 gives 0.1 -> GPU 0,
    # 0.2 -> GPU 1, 0.6 -> GPU 0, 0.7 -> GPU 0 (cursor at GPU 1, which is down), 1.6 -> GPU 0; rows
    # by (epoch, gpu): epoch 0 GPU 0 {0.1, 0.6, 0.7}, GPU 1 {0.2}; epoch 1 GPU 0 {1.6}.
    P = tables([[1000] * 5], [[0] * 5], [100], bsz=[1], tmo=[0])
    tr = trace_from([(100_000, 0, 1), (200_000, 0, 1), (600_000, 0, 1), (700_000, 0, 1), (1_600_000, 0, 1)],
                    2_000_000)
    avail = np.array([[[0, 1 << 60], [0, 500_000]]], np.int64)
    f = oracle.form_dispatch(P, tr, N=2, e_lo=0, e_hi=2, avail=avail)
    assert f["gpu"].tolist() == [0, 0, 0, 1, 0]
    assert f["ready"].tolist() == [100_000, 600_000, 700_000, 200_000, 1_600_000]
    assert f["batch_off"].tolist() == [0, 3, 4, 5, 5]
    # (b) GPU 1 available only from 1.5 s: everything before goes to GPU 0, 1.6 s to GPU 1
    avail2 = np.array([[[0, 1 << 60], [1_500_000, 1 << 60]]], np.int64)
    f2 = oracle.form_dispatch(P, tr, N=2, e_lo=0, e_hi=2, avail=avail2)
    # GPU 1 only from 1.5 s: everything before goes to GPU 0, 1.6 s to GPU 1 (cursor 1)
    assert f2["batch_off"].tolist() == [0, 4, 4, 4, 5] and f2["gpu"].tolist() == [0, 0, 0, 0, 1]
    f3 = oracle.form_dispatch(P, tr, N=2, e_lo=1, e_hi=2, avail=avail2)  # epoch 1 only
    assert f3["ready"].tolist() == [1_600_000] and f3["gpu"].tolist() == [1]


def test_form_dispatch_errors(oracle):
    P = tables([[1000] * 5], [[0] * 5], [100])
    tr = trace_from([(5, 0, 1)], 1_000_000)
    for kw in (dict(e_lo=1, e_hi=0), dict(e_lo=0, e_hi=99)):
        with pytest.raises(oracle.OracleError) as e:
            oracle.form_dispatch(P, tr, N=1, **kw)
        assert e.value.code == -1
