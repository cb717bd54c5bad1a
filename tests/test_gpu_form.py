"""protean_form_batches (the SURVEY §8(b) helper: O3 batch formation + O5.2 round-robin dispatch
for an epoch range) vs the oracle's form_dispatch: every row's (ready, size, model, class, GPU),
the CSR offsets and every row's member arrivals, bit-exact.  -m gpu."""
import numpy as np
import pytest

from helpers import tables, trace_from
from protean_inputs import mix_a_params, mix_b_params, random_profiles, synth_profiles, tick_trace, uniform_trace

pytestmark = pytest.mark.gpu

ROW = np.dtype([("ready", "<u4"), ("req_off", "<u4"), ("n", "<u2"), ("model", "u1"), ("strict", "u1"),
                ("gpu", "<u4")])


def _gpu_form(prof, tr, N, e_lo, e_hi, avail=None):
    import torch
    import paper_conf_middleware_bhasisjgpkd24_b200 as pkg
    dev = torch.device("cuda", 0)
    arr = torch.from_numpy(np.ascontiguousarray(tr.arrival_us).view(np.int32).copy()).to(dev)
    meta = torch.from_numpy(np.ascontiguousarray(tr.meta).copy()).to(dev)
    off = torch.from_numpy(np.ascontiguousarray(tr.replica_off, np.int64).copy()).to(dev)
    av = torch.from_numpy(np.ascontiguousarray(avail, np.int64)).to(dev) if avail is not None else None
    h = pkg.load_profiles(prof)
    f = h.form_batches(arr, meta, off, trace_len_us=tr.trace_len_us, n_gpus=N, e_lo=e_lo, e_hi=e_hi, avail=av)
    rows = f["rows"].cpu().numpy().reshape(-1).view(ROW)
    return rows, f["batch_off"].cpu().numpy(), f["members"].cpu().numpy().view(np.uint32)


def _compare(prof, tr, N, e_lo, e_hi, oracle, avail=None):
    rows, boff, mem = _gpu_form(prof, tr, N, e_lo, e_hi, avail)
    o = oracle.form_dispatch(prof, tr, N=N, e_lo=e_lo, e_hi=e_hi, avail=avail)
    assert np.array_equal(boff, o["batch_off"])
    assert rows.shape[0] == o["ready"].shape[0]
    for f in ("ready", "n", "model", "strict", "gpu"):
        assert np.array_equal(rows[f].astype(np.int64), o[f].astype(np.int64)), f
    for i in range(rows.shape[0]):
        g = mem[rows["req_off"][i]: rows["req_off"][i] + rows["n"][i]]
        w = o["members"][o["req_off"][i]: o["req_off"][i] + o["n"][i]]
        assert np.array_equal(g, w), i
    return rows


def test_hand_example_with_windows(oracle):
    P = tables([[1000] * 5], [[0] * 5], [100], bsz=[1], tmo=[0])
    tr = trace_from([(100_000, 0, 1), (200_000, 0, 1), (600_000, 0, 1), (700_000, 0, 1), (1_600_000, 0, 1)],
                    2_000_000)
    rows = _compare(P, tr, 2, 0, 2, oracle, avail=np.array([[[0, 1 << 60], [0, 500_000]]], np.int64))
    assert rows["gpu"].tolist() == [0, 0, 0, 1, 0]


@pytest.mark.parametrize("seed", range(5))
def test_fuzz_form(oracle, seed):
    rng = np.random.default_rng(3100 + seed)
    M = int(rng.integers(1, 6))
    P = random_profiles(rng, M)
    N = int(rng.integers(1, 6))
    R = int(rng.integers(1, 5))
    tr = uniform_trace(rng, R, M, int(rng.integers(2, 9)) * 1_000_000, int(rng.integers(5, 700)))
    E = oracle.num_epochs(P, tr.trace_len_us, 1_000_000)
    e_lo = int(rng.integers(0, E))
    e_hi = int(rng.integers(e_lo, E + 1))
    avail = None
    if seed % 2:
        lo = rng.integers(0, tr.trace_len_us, size=(R, N))
        avail = np.stack([lo, lo + rng.integers(0, tr.trace_len_us, size=(R, N))], -1).astype(np.int64)
    _compare(P, tr, N, e_lo, e_hi, oracle, avail)


def test_mix_shapes(oracle):
    P = synth_profiles()
    _compare(P, tick_trace(mix_a_params(3, seed=2, seconds=8)), 8, 0, 9, oracle)
    _compare(P, tick_trace(mix_b_params(2, seed=4, seconds=6)), 8, 2, 5, oracle)


def test_form_errors(oracle):
    import paper_conf_middleware_bhasisjgpkd24_b200 as pkg
    P = tables([[1000] * 5], [[0] * 5], [100])
    tr = trace_from([(5, 0, 1)], 1_000_000)
    for e_lo, e_hi in ((1, 0), (0, 99)):
        with pytest.raises(pkg.ProteanError) as e:
            _gpu_form(P, tr, 1, e_lo, e_hi)
        assert e.value.code == -1
