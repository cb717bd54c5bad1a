"""Mode G on the GPU: n ranks, each scoring its slot-balanced geometry range and
exchanging (best, current) keys once per replica-epoch inside the replay kernel over peer memory,
must reproduce the 1-rank result of the CPU oracle exactly.  All ranks run in this process on
cuda:0 (one handle + one host thread + one stream per rank, grids capped so the kernels are
co-resident); across GPUs the same kernel stores over NVLink through CUDA IPC mappings."""
import threading

import numpy as np
import pytest

from gpu_common import GPU_LOG_DTYPE, compare, oracle_replay
from protean_inputs import mix_a_params, mix_b_params, random_profiles, synth_profiles, tick_trace, uniform_trace

pytestmark = pytest.mark.gpu


@pytest.fixture(autouse=True)
def _short_exchange_timeout(monkeypatch):
    monkeypatch.setenv("PROTEAN_XCHG_TIMEOUT_S", "10")  # a broken exchange fails, never hangs


def modeg_replay(prof, trace, nranks, *, calls=1, max_ctas=None, **cfg):
    import torch

    import paper_conf_middleware_bhasisjgpkd24_b200 as pkg
    from paper_conf_middleware_bhasisjgpkd24_b200.parallel import merge_geometry_shards
    N = cfg.get("n_gpus", 8)
    R = trace.n_replicas
    hs = [pkg.load_profiles(prof, device=0) for _ in range(nranks)]
    pkg.Handle.xchg_attach(hs, R, N)
    bounds = pkg.geometry_split(prof, nranks)
    dev = torch.device("cuda", 0)
    arr = torch.from_numpy(np.ascontiguousarray(trace.arrival_us).view(np.int32)).to(dev)
    meta = torch.from_numpy(np.ascontiguousarray(trace.meta)).to(dev)
    off = torch.from_numpy(np.ascontiguousarray(trace.replica_off, np.int64)).to(dev)
    E = hs[0].num_epochs(trace.trace_len_us, cfg.get("epoch_len_us", 1_000_000))
    log_cap = max(1, int(np.max(np.diff(trace.replica_off))))
    outs = [hs[k].alloc_replay_out(R, E, N, cand_keys=True, log_cap=log_cap) for k in range(nranks)]
    streams = [torch.cuda.Stream(device=dev) for _ in range(nranks)]
    torch.cuda.synchronize()
    cap = max_ctas if max_ctas is not None else max(1, min(R, 96 // nranks))
    results = []
    for _ in range(calls):
        errs = [None] * nranks

        def run(k):
            try:
                hs[k].replay_traces(arr, meta, off, trace_len_us=trace.trace_len_us, out=outs[k],
                                    stream=streams[k], shard_mode=1, rank=k, nranks=nranks,
                                    max_ctas=cap, replica_base=trace.replica_base, **cfg)
            except Exception as e:  # noqa: BLE001
                errs[k] = e
        th = [threading.Thread(target=run, args=(k,)) for k in range(nranks)]
        for t in th:
            t.start()
        for t in th:
            t.join(timeout=120)
        assert not any(t.is_alive() for t in th), "mode G ranks did not finish"
        for e in errs:
            if e is not None:
                raise e
        torch.cuda.synchronize()
        host = []
        for o in outs:
            d = {k: (v.cpu().numpy() if hasattr(v, "cpu") else v) for k, v in o.items()}
            d["hist"] = d["hist"].view(np.uint32)
            d["log"] = d["log"].reshape(R, log_cap, 32).view(GPU_LOG_DTYPE).reshape(R, log_cap)
            host.append(d)
        results.append((host, merge_geometry_shards(host, bounds)))
    for h in hs:
        h.close()
    return results, bounds


def _check_ranks(host, merged, o, R, bounds):
    compare(merged, o, R)
    for k, h in enumerate(host):  # every rank holds the full (redundant) result
        assert np.array_equal(h["decisions"], o["decisions"])
        assert np.array_equal(h["counters"][:, :8], o["counters"][:, :8])
        assert np.array_equal(h["hist"], o["hist"])
        lo, hi = bounds[k], bounds[k + 1]
        assert np.array_equal(h["cand_keys"][..., lo:hi], o["cand_keys"][..., lo:hi])


@pytest.mark.parametrize("nranks", [2, 3, 5, 8])
def test_mode_g_mix_a(oracle, nranks):
    prof = synth_profiles()
    tr = tick_trace(mix_a_params(3, seed=21, seconds=20))
    res, bounds = modeg_replay(prof, tr, nranks, n_gpus=8)
    o = oracle_replay(oracle, prof, tr, n_gpus=8)
    host, merged = res[0]
    _check_ranks(host, merged, o, 3, bounds)
    assert (o["decisions"] != 255).any()


def test_mode_g_all_37_vm_and_repeat(oracle):
    """G = 37, spot/on-demand VMs with revocations, and two consecutive calls (the exchange's
    sequence numbers continue across calls)."""
    prof = synth_profiles().with_geometry_set(1)
    tr = tick_trace(mix_b_params(2, seed=4, seconds=10))
    cfg = dict(n_gpus=8, vm_policy=1, p_rev=0.708, rev_interval_us=3_000_000, notice_us=1_000_000, seed=9)
    res, bounds = modeg_replay(prof, tr, 4, calls=2, **cfg)
    o = oracle_replay(oracle, prof, tr, **cfg)
    for host, merged in res:
        _check_ranks(host, merged, o, 2, bounds)


def test_mode_g_fuzz_small(oracle):
    rng = np.random.default_rng(77)
    prof = random_profiles(rng, 4)
    tr = uniform_trace(rng, 4, 4, 5_000_000, 250)
    cfg = dict(n_gpus=3, wait_limit=0, reconfig_us=300_000, init_geom=5)
    res, bounds = modeg_replay(prof, tr, 2, max_ctas=1, **cfg)  # one CTA walks all replicas
    o = oracle_replay(oracle, prof, tr, **cfg)
    host, merged = res[0]
    _check_ranks(host, merged, o, 4, bounds)


def test_mode_g_errors():
    import torch

    import paper_conf_middleware_bhasisjgpkd24_b200 as pkg
    from paper_conf_middleware_bhasisjgpkd24_b200 import _abi
    prof = synth_profiles()
    tr = tick_trace(mix_a_params(1, seed=2, seconds=3))
    dev = torch.device("cuda", 0)
    arr = torch.from_numpy(np.ascontiguousarray(tr.arrival_us).view(np.int32)).to(dev)
    meta = torch.from_numpy(tr.meta).to(dev)
    off = torch.from_numpy(np.asarray(tr.replica_off, np.int64)).to(dev)
    h = pkg.load_profiles(prof)
    with pytest.raises(_abi.ProteanError) as e:  # no exchange set up
        h.replay_traces(arr, meta, off, trace_len_us=tr.trace_len_us, shard_mode=1, rank=0, nranks=2)
    assert e.value.code == _abi.ESTATE
    h2 = pkg.load_profiles(prof)
    pkg.Handle.xchg_attach([h, h2], 1, 8)
    with pytest.raises(_abi.ProteanError) as e:  # rank mismatch
        h.replay_traces(arr, meta, off, trace_len_us=tr.trace_len_us, shard_mode=1, rank=1, nranks=2)
    assert e.value.code == _abi.EINVAL
    with pytest.raises(_abi.ProteanError) as e:  # more sim-GPUs than the exchange holds
        h.replay_traces(arr, meta, off, trace_len_us=tr.trace_len_us, shard_mode=1, rank=0, nranks=2,
                        n_gpus=9)
    assert e.value.code == _abi.ERANGE
    h.close()
    h2.close()
