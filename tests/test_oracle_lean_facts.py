"""The formation fact the lean replay path (csrc/cand.cu walk_kernel / cand_kernel) is built on,
checked on the oracle's own replay log (the oracle forms batches epoch by epoch, O3; P:L229, P:L239;
reading Q14):

  every stream's batches are ONE greedy chain over the stream's arrivals from its first request --
  contiguous member runs, each closed at B_m requests (on its last member) or at its first arrival
  + T_m -- whose ready times never decrease, and each batch is formed in the epoch that holds its
  ready time (epoch = ready div W).

So the stream cursor at the start of epoch e (the first request not yet batched) is the start of
the first batch of the chain with ready >= eW, which walk_kernel computes for every epoch at once,
and an epoch's batches can be formed from that cursor without the earlier epochs."""
import numpy as np
import pytest

from protean_inputs import mix_a_params, mix_b_params, random_profiles, synth_profiles, tick_trace, uniform_trace


def _check(oracle, P, tr, W, N=2):
    o = oracle.replay(P, tr, N=N, W=W, policy=1, want_log=True)
    for r in range(tr.n_replicas):
        log = o["log"][r][: int(o["n_batches"][r])]
        lo, hi = int(tr.replica_off[r]), int(tr.replica_off[r + 1])
        arr = np.asarray(tr.arrival_us[lo:hi], np.int64)
        meta = np.asarray(tr.meta[lo:hi])
        model, strict = meta & 0x3F, ((meta >> 7) & 1) == 1
        assert (log["epoch"].astype(np.int64) == log["ready"].astype(np.int64) // W).all()
        for m in np.unique(log["model"]):
            for s in (0, 1):
                sel = (log["model"] == m) & (log["strict"] == s)
                bl = log[sel]
                order = np.lexsort((bl["ready"], bl["epoch"]))
                bl = bl[order]
                stream = np.sort(arr[(model == m) & (strict == bool(s))], kind="stable")
                assert (np.diff(bl["ready"].astype(np.int64)) >= 0).all()
                pos = 0
                B, T = int(P.batch_size[m]), int(P.timeout_us[m])
                for b in bl:  # contiguous runs from the stream's first request, in order
                    n = int(b["n"])
                    mem = stream[pos: pos + n]
                    assert len(mem) == n
                    if n == B and mem[-1] <= mem[0] + T:
                        assert int(b["ready"]) == mem[-1]
                    else:
                        assert int(b["ready"]) == mem[0] + T
                        if pos + n < len(stream):  # closed because the next one misses the timeout
                            assert stream[pos + n] > mem[0] + T
                    pos += n
    return o


def test_chain_fact_fuzz(oracle):
    rng = np.random.default_rng(808)
    for trial in range(8):
        M = int(rng.integers(1, 6))
        P = random_profiles(rng, M, small_time=bool(trial % 2))
        tr = uniform_trace(rng, 2, M, int(rng.integers(2, 6)) * 1_000_000, int(rng.integers(50, 400)))
        _check(oracle, P, tr, W=int(rng.choice([20_000, 250_000, 1_000_000])))


@pytest.mark.parametrize("mix", ["a", "b"])
def test_chain_fact_paper_mixes(oracle, mix):
    P = synth_profiles()
    gp = mix_a_params(1, seed=3, seconds=8) if mix == "a" else mix_b_params(1, seed=3, seconds=8)
    _check(oracle, P, tick_trace(gp), W=1_000_000, N=8)
