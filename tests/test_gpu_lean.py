"""The lean replay path (csrc/cand.cu + csrc/chain.cu) vs the CPU oracle.  -m gpu.

The lean path (a data-parallel candidate search ahead of a warp-per-replica chain, accounting in
its own pass) serves many-replica mode-R calls; PROTEAN_LEAN=2 makes small cases take it too.  Each
test asserts the path was taken (the accounting pass reports a time) and compares every output
element by element with the oracle: closed-form epochs scored by cand.cu, epochs with an
unavailable GPU scored in the chain, units cand.cu cannot hold (a class above 10 batches,
completions 2^25 us past the epoch start), and calls with an epoch above 64 batches, which go back
to the fused engine."""
import numpy as np
import pytest

from gpu_common import GPU_LOG_DTYPE, compare, oracle_replay
from protean_inputs import mix_a_params, mix_b_params, random_profiles, synth_profiles, tick_trace, uniform_trace

pytestmark = pytest.mark.gpu


def lean_replay(monkeypatch, prof, trace, *, expect_lean=True, **cfg):
    import paper_conf_middleware_bhasisjgpkd24_b200 as pkg
    monkeypatch.setenv("PROTEAN_LEAN", "2")
    h = pkg.load_profiles(prof, device=0)
    log_cap = max(1, int(np.max(np.diff(trace.replica_off))))
    out = h.replay_traces_host(trace, want_cand_keys=True, log_cap=log_cap, **cfg)
    search, walk, acct = h.last_search_ms()
    h.close()
    assert search > 0 or expect_lean is None, "the candidate search did not run"
    if expect_lean is not None:  # None: either (an epoch above 64 batches goes back to the fused engine)
        assert (acct > 0) == expect_lean, f"lean chain {'not ' if expect_lean else ''}taken (acct {acct} ms)"
    out["log"] = out["log"].reshape(trace.n_replicas, log_cap, 32).view(GPU_LOG_DTYPE).reshape(
        trace.n_replicas, log_cap)
    out["hist"] = out["hist"].view(np.uint32)
    return out


@pytest.mark.parametrize("seed", range(10))
def test_lean_fuzz(oracle, monkeypatch, seed):
    rng = np.random.default_rng(700 + seed)
    M = int(rng.integers(1, 7))
    gset = int(rng.integers(0, 2))
    prof = random_profiles(rng, M).with_geometry_set(gset)
    N = int(rng.choice([2, 4, 8])) if gset else int(rng.choice([1, 2, 3, 8]))  # N * G even
    R = int(rng.integers(1, 6))
    tr = uniform_trace(rng, R, M, int(rng.integers(2, 12)) * 1_000_000, int(rng.integers(5, 600)))
    cfg = dict(n_gpus=N, init_geom=int(rng.integers(0, 12)), max_live=int(rng.choice([2, 8, 64])),
               wait_limit=int(rng.integers(0, 4)), reconfig_us=int(rng.integers(0, 3_000_000)),
               vm_policy=int(seed % 3), p_rev=float(rng.choice([0.0, 0.354, 0.708, 1.0])),
               rev_interval_us=2_000_000, notice_us=300_000, seed=seed)
    tr.replica_base = int(rng.integers(0, 100))
    g = lean_replay(monkeypatch, prof, tr, **cfg)
    compare(g, oracle_replay(oracle, prof, tr, **cfg), R)


@pytest.mark.parametrize("n_gpus", [8, 5])
def test_lean_mix_a(oracle, monkeypatch, n_gpus):
    """Config-5-shaped replicas (Mix A, 12 geometries): nearly every epoch closed-form."""
    gp = mix_a_params(3, seed=11, seconds=40)
    tr = tick_trace(gp)
    P = synth_profiles()
    g = lean_replay(monkeypatch, P, tr, n_gpus=n_gpus)
    compare(g, oracle_replay(oracle, P, tr, n_gpus=n_gpus), 3)


def test_lean_reconfig_heavy(oracle, monkeypatch):
    """Short epochs and long reconfigurations: many epochs with an unavailable GPU (in-chain keys),
    batches dropped for want of an available GPU, spot revocations."""
    rng = np.random.default_rng(5)
    prof = random_profiles(rng, 4, small_time=True)
    tr = uniform_trace(rng, 4, 4, 3_000_000, 900)
    cfg = dict(n_gpus=4, epoch_len_us=50_000, wait_limit=0, reconfig_us=120_000, vm_policy=2,
               p_rev=0.5, rev_interval_us=200_000, notice_us=30_000, seed=3)
    g = lean_replay(monkeypatch, prof, tr, **cfg)
    compare(g, oracle_replay(oracle, prof, tr, **cfg), 4)


def test_lean_units_not_held(oracle, monkeypatch):
    """Units cand.cu does not hold: a residue class above 10 batches (one sim-GPU, dense tiny
    batches) and completions beyond 2^25 us past the epoch start (solo times x 400)."""
    rng = np.random.default_rng(9)
    prof = random_profiles(rng, 3, max_batch=2)
    tr = uniform_trace(rng, 2, 3, 4_000_000, 160)
    g = lean_replay(monkeypatch, prof, tr, n_gpus=1)
    compare(g, oracle_replay(oracle, prof, tr, n_gpus=1), 2)
    slow = random_profiles(np.random.default_rng(10), 3)
    slow.solo_us[:] = np.minimum(slow.solo_us.astype(np.int64) * 400, 2**31 - 1).astype(slow.solo_us.dtype)
    tr2 = uniform_trace(np.random.default_rng(11), 2, 3, 3_000_000, 60)
    g = lean_replay(monkeypatch, slow, tr2, n_gpus=2)
    compare(g, oracle_replay(oracle, slow, tr2, n_gpus=2), 2)


def test_lean_overflow_falls_back(oracle, monkeypatch):
    """An epoch above 64 batches (Mix B x 8 on 8 sim-GPUs): the call goes back to the fused
    engine, with identical results."""
    gp = mix_b_params(1, seed=4, seconds=6, scale=8.0)
    tr = tick_trace(gp)
    P = synth_profiles()
    g = lean_replay(monkeypatch, P, tr, expect_lean=False, n_gpus=8)
    compare(g, oracle_replay(oracle, P, tr, n_gpus=8), 1)


@pytest.mark.parametrize("W", [5_000, 40_000_000])
def test_lean_epoch_length_extremes(oracle, monkeypatch, W):
    """Epochs of 5 ms (most batches straddle epochs: the cursor walk's epoch fill) and of 40 s
    (ready times up to 2^25 us past the epoch start: every unit falls back from 32-bit time)."""
    rng = np.random.default_rng(31 + W % 7)
    prof = random_profiles(rng, 3, small_time=W < 100_000)
    tr = uniform_trace(rng, 3, 3, 80_000_000 if W > 1_000_000 else 400_000, 60 if W > 1_000_000 else 300)
    cfg = dict(n_gpus=4, epoch_len_us=W, reconfig_us=W // 2, wait_limit=1)
    g = lean_replay(monkeypatch, prof, tr, **cfg)
    compare(g, oracle_replay(oracle, prof, tr, **cfg), 3)


@pytest.mark.parametrize("case", ["arrivals_and_ready_at_epoch_starts", "fbr_sum_exactly_one",
                                  "ready_exactly_at_reconfiguration_end", "revocation_at_and_inside_epochs",
                                  "epochs_shorter_than_batch_timeouts"])
def test_lean_targeted_edges(oracle, monkeypatch, case):
    """tests/test_gpu_edges.py's targeted edges (each asserts its edge occurs) on the lean path."""
    import test_gpu_edges as edges
    monkeypatch.setenv("PROTEAN_LEAN", "2")
    fn = getattr(edges, "test_" + case)
    if case == "revocation_at_and_inside_epochs":
        fn(oracle, 2.5, 2)
    elif case == "epochs_shorter_than_batch_timeouts":
        fn(oracle, 0)
    else:
        fn(oracle)


@pytest.mark.parametrize("seed", range(4))
def test_lean_alg2_policy(oracle, monkeypatch, seed):
    """Alg 2's own heuristic (policy 2, N1) on the lean path: the search pass forms and ranks the
    epoch's batches without scoring candidates; the chain's decision step runs the heuristic."""
    rng = np.random.default_rng(950 + seed)
    if seed < 2:
        gp = mix_a_params(2, seed=20 + seed, seconds=30)
        tr, P, N = tick_trace(gp), synth_profiles(), 8
    else:
        M = int(rng.integers(2, 6))
        P = random_profiles(rng, M)
        tr = uniform_trace(rng, 3, M, 8_000_000, 200)  # <= 64 batches per epoch: the lean chain
        N = int(rng.choice([2, 4]))
    cfg = dict(n_gpus=N, policy=2, wait_limit=int(rng.integers(0, 3)), ewma_alpha_pm=int(rng.integers(100, 900)),
               t_low_milli=int(rng.integers(0, 2000)), t_high_milli=int(rng.integers(2000, 8000)))
    g = lean_replay(monkeypatch, P, tr, **cfg)
    compare(g, oracle_replay(oracle, P, tr, **cfg), tr.n_replicas)


def test_lean_unheld_epoch_sentinel_race(oracle, monkeypatch):
    """Regression: an epoch with every GPU available whose unit cand.cu did not hold (the
    kfc[r][e][0][0] sentinel) makes the chain score it and overwrite kst[0]; a lane behind the
    others used to read the key instead of the sentinel, take the other branch and deadlock the
    warp in the reconfiguration cap's collectives.  The sentinel is now read once and broadcast."""
    rng = np.random.default_rng(1301)
    M = int(rng.integers(2, 6))
    P = random_profiles(rng, M)
    tr = uniform_trace(rng, 3, M, 8_000_000, 200)
    N = int(rng.choice([2, 4]))
    g = lean_replay(monkeypatch, P, tr, n_gpus=N)
    compare(g, oracle_replay(oracle, P, tr, n_gpus=N), 3)


@pytest.mark.parametrize("seed", range(6))
def test_lean_container_pools(oracle, monkeypatch, seed):
    """N3 container pools (cold starts, keep-alive, pre-warm, readings R22-R27)
    on the lean chain, lane = sim-GPU, with spot revocations taking a VM's containers (R27)."""
    rng = np.random.default_rng(1300 + seed)
    M = int(rng.integers(2, 6))
    P = random_profiles(rng, M)
    tr = uniform_trace(rng, 3, M, 8_000_000, 200)
    N = int(rng.choice([2, 4]))
    cfg = dict(n_gpus=N, cold_start_us=int(rng.integers(100_000, 3_000_000)),
               keepalive_epochs=int(rng.integers(1, 5)), prewarm=int(rng.integers(0, 3)),
               vm_policy=int(seed % 3), p_rev=0.5, rev_interval_us=2_000_000, notice_us=200_000, seed=seed)
    g = lean_replay(monkeypatch, P, tr, **cfg)
    o = oracle_replay(oracle, P, tr, **cfg)
    assert int(np.sum(o["cold_starts"])) > 0
    compare(g, o, 3)


def wide_case(seed):
    """One random lean-path case mixing every option the lean path takes: geometry sets, N, epoch
    length, max_live, hysteresis, reconfiguration time, VM policies and revocations, container pools
    (N3), the search policy or Alg 2's heuristic (N1)."""
    rng = np.random.default_rng(4000 + seed)
    M = int(rng.integers(1, 7))
    gset = int(rng.integers(0, 2))
    prof = random_profiles(rng, M, small_time=bool(rng.integers(0, 2))).with_geometry_set(gset)
    N = int(rng.choice([2, 4, 6, 8, 16])) if gset else int(rng.choice([1, 2, 3, 5, 8, 12, 32]))
    R = int(rng.integers(1, 5))
    tr = uniform_trace(rng, R, M, int(rng.integers(1, 10)) * 1_000_000, int(rng.integers(5, 400)))
    tr.replica_base = int(rng.integers(0, 1000))
    W = int(rng.choice([100_000, 250_000, 1_000_000, 2_000_000]))
    policy = int(rng.choice([0, 0, 2]))
    cfg = dict(n_gpus=N, epoch_len_us=W, init_geom=int(rng.integers(0, 12)), max_live=int(rng.choice([1, 4, 16, 64])),
               wait_limit=int(rng.integers(0, 3)), reconfig_us=int(rng.integers(0, 2 * W)), policy=policy,
               vm_policy=int(rng.integers(0, 3)), p_rev=float(rng.choice([0.0, 0.354, 1.0])),
               rev_interval_us=int(rng.choice([W, 2_000_000])), notice_us=int(rng.integers(0, W)), seed=seed)
    if rng.integers(0, 2):
        cfg.update(cold_start_us=int(rng.integers(1, 2_000_000)), keepalive_epochs=int(rng.integers(1, 6)),
                   prewarm=int(rng.integers(0, 3)))
    if policy == 2:
        cfg.update(ewma_alpha_pm=int(rng.integers(100, 900)), t_low_milli=int(rng.integers(0, 2000)),
                   t_high_milli=int(rng.integers(2000, 8000)))
    return prof, tr, cfg


@pytest.mark.parametrize("seed", list(range(24)) + [596])
def test_lean_fuzz_wide(oracle, monkeypatch, seed):
    """24 wide cases, plus seed 596, whose container pool outgrows 128 containers: both sides
    report ERANGE (R22).  tools/lean_hunt.py ran seeds 0-5999 (14 ERANGE on both sides, the rest
    identical)."""
    import paper_conf_middleware_bhasisjgpkd24_b200 as pkg
    prof, tr, cfg = wide_case(seed)
    try:
        o = oracle_replay(oracle, prof, tr, **cfg)
    except oracle.OracleError as e:
        assert "range" in str(e).lower() or "-2" in str(e), e
        with pytest.raises(pkg.ProteanError, match="128 containers"):
            lean_replay(monkeypatch, prof, tr, expect_lean=None, **cfg)
        return
    g = lean_replay(monkeypatch, prof, tr, expect_lean=None, **cfg)
    compare(g, o, tr.n_replicas)
