"""N4a exhaustive assignment sweep: CUDA (protean_sweep_assignments) vs the CPU oracle (orc_sweep)
through the C ABI -- every sweep key, every minimising assignment, the best keys and the
assignment count bit-exact.  -m gpu."""
import json
import os

import numpy as np
import pytest

from helpers import GOLDEN, tables
from protean_inputs import epoch_batches, pack_batch_rows, random_profiles, synth_profiles

pytestmark = pytest.mark.gpu


def _gpu_sweep(prof, R, N, batches, batch_off, arrival, cur_geom, **kw):
    import torch
    import paper_conf_middleware_bhasisjgpkd24_b200 as pkg
    dev = torch.device("cuda", 0)
    rows = pack_batch_rows(batches)
    t_rows = torch.from_numpy(rows.copy()).to(dev) if rows.size else torch.zeros(0, dtype=torch.uint8, device=dev)
    t_off = torch.from_numpy(np.asarray(batch_off, np.int32).copy()).to(dev)
    arr = np.asarray(arrival, np.uint32)
    t_arr = torch.from_numpy(arr.view(np.int32).copy()).to(dev) if arr.size else torch.zeros(1, dtype=torch.int32, device=dev)
    t_cur = torch.from_numpy(np.asarray(cur_geom, np.uint8).copy()).to(dev)
    h = pkg.load_profiles(prof)
    out = h.sweep_assignments(n_replicas=R, n_gpus=N, batches=t_rows, batch_off=t_off, arrival_us=t_arr,
                              cur_geom=t_cur, **kw)
    torch.cuda.synchronize()
    res = {k: v.cpu().numpy() for k, v in out.items()}
    h.close()
    res["assign"] = res["assign"].view(np.uint32)
    res["n_assign"] = int(res["n_assign"][0])
    return res


def _compare(g, o, nc):
    assert g["best_key"].tolist() == o["best_key"].tolist()
    assert g["sweep_key"][: o["sweep_key"].shape[0]].tolist() == o["sweep_key"].tolist()
    assert g["assign"][: o["assign"].shape[0]].tolist() == o["assign"].tolist()
    assert g["n_assign"] == o["n_assign"]


def test_t13_golden_gpu(oracle):
    t13 = json.load(open(os.path.join(GOLDEN, "t13_sweep.json")))
    m = t13["models"]
    P = tables(m["solo_us"], m["fbr_ppm"], m["mem_mib"], bsz=[1, 1], slo=m["slo_us"], tmo=[0, 0])
    b = t13["batches"]
    batches = {k: np.asarray(v) for k, v in dict(ready=b["ready"], req_off=[0, 1], n=[1, 1], model=b["model"],
                                                 strict=b["strict"]).items()}
    g = _gpu_sweep(P, 1, 1, batches, [0, 2], b["arrival"], [0])
    j = t13["geometry_index"]
    assert g["sweep_key"][j] == t13["sweep"]["key"] and g["assign"][j] == t13["sweep"]["assign"]
    o = oracle.sweep(P, R=1, N=1, batches=batches, batch_off=[0, 2], arrival=b["arrival"], cur_geom=[0])
    _compare(g, o, 12)


@pytest.mark.parametrize("seed", range(6))
def test_fuzz_sweep(oracle, seed):
    rng = np.random.default_rng(1300 + seed)
    M = int(rng.integers(1, 6))
    prof = random_profiles(rng, M).with_geometry_set(int(rng.integers(0, 2)))
    G = 12 if prof.geometry_set == 0 else 37
    R, N = int(rng.integers(1, 4)), int(rng.integers(1, 5))
    maxb = int(rng.integers(1, 6))
    batches, off, arr, cur = epoch_batches(2000 + seed, R, N, models=range(M), mean_batches=2.5,
                                           max_batches=maxb, batch_size=int(rng.integers(1, 9)), ragged=True,
                                           spread_us=int(rng.integers(0, 400_000)), G=G)
    cur[rng.random(cur.shape[0]) < 0.2] = 255
    lo = int(rng.integers(0, G // 2))
    hi = int(rng.integers(lo + 1, G + 1))
    kw = dict(max_live=int(rng.choice([1, 2, 64])), max_batches=maxb, geom_lo=lo, geom_hi=hi)
    g = _gpu_sweep(prof, R, N, batches, off, arr, cur, **kw)
    o = oracle.sweep(prof, R=R, N=N, batches=batches, batch_off=off, arrival=arr, cur_geom=cur, **kw)
    _compare(g, o, hi - lo)


def test_config5_shape_sampled(oracle):
    """The bench shape (config-5 GPU-epochs: ~4.9 batches of 128 vision requests, 22-model table,
    12 geometries) on 64 units; the oracle re-derives every unit."""
    P = synth_profiles()
    R, N = 8, 8
    batches, off, arr, cur = epoch_batches(7, R, N, max_batches=6)
    g = _gpu_sweep(P, R, N, batches, off, arr, cur, max_batches=6)
    o = oracle.sweep(P, R=R, N=N, batches=batches, batch_off=off, arrival=arr, cur_geom=cur, max_batches=6)
    _compare(g, o, 12)


def test_sweep_error_codes_match_oracle(oracle):
    import paper_conf_middleware_bhasisjgpkd24_b200 as pkg
    P = tables([[1000] * 5], [[0] * 5], [100])
    base = {k: np.asarray(v) for k, v in dict(ready=[5] * 9, req_off=list(range(9)), n=[1] * 9, model=[0] * 9,
                                              strict=[1] * 9).items()}
    arr = [5] * 9

    def codes(batches, off, cur=(0,), **kw):
        try:
            _gpu_sweep(P, 1, 1, batches, off, arr, cur, **kw)
            gc = 0
        except pkg.ProteanError as e:
            gc = e.code
        try:
            oracle.sweep(P, R=1, N=1, batches=batches, batch_off=off, arrival=arr, cur_geom=cur, **kw)
            oc = 0
        except oracle.OracleError as e:
            oc = e.code
        return gc, oc
    cases = [
        (base, [0, 9], {}), (base, [0, 9], dict(max_batches=9)), (base, [0, 3], {}),
        (dict(base, model=np.ones(9, int)), [0, 3], {}),
        (dict(base, ready=np.array([5, 4, 6, 7, 8, 9, 10, 11, 12])), [0, 3], {}),
        (dict(base, n=np.zeros(9, int)), [0, 3], {}),
        (base, [0, 3], dict(max_live=0)), (base, [0, 3], dict(geom_lo=3, geom_hi=3)),
    ]
    for batches, off, kw in cases:
        gc, oc = codes(batches, off, **kw)
        assert gc == oc, (kw, gc, oc)
    gc, oc = codes(base, [0, 3], cur=(12,))
    assert gc == oc == -1


@pytest.mark.parametrize("seed", range(3))
def test_wide_times_64bit_path(oracle, seed):
    """Solo times of minutes: a GPU-epoch's completion bound exceeds 2^31 us, so the sweep runs its
    64-bit instance (the 32-bit one needs relative times below 2^31); heavy footprints exercise the
    memory-wait branch.  Both instances meet in one call (units with and without wide models)."""
    rng = np.random.default_rng(1700 + seed)
    M = 3
    solo7 = np.array([150_000_000, 300_000_000, 2_000])  # two very long models (x6 on 1g < 2^31), one short
    prof = tables(np.stack([solo7 * f for f in (6, 4, 3, 2, 1)], 1), rng.integers(200_000, 1_000_000, (M, 5)),
                  rng.integers(2_000, 18_000, M), bsz=[2, 3, 1], slo=3 * solo7, tmo=[0, 0, 0])
    R, N = 2, 4
    batches, off, arr, cur = epoch_batches(3000 + seed, R, N, models=range(M), mean_batches=3.0, max_batches=5,
                                           batch_size=3, ragged=True)
    g = _gpu_sweep(prof, R, N, batches, off, arr, cur, max_batches=5)
    o = oracle.sweep(prof, R=R, N=N, batches=batches, batch_off=off, arrival=arr, cur_geom=cur, max_batches=5)
    _compare(g, o, 12)
    assert (o["sweep_key"] & 0xFFFFFFFFFF00 != 0).any()  # some BE tails are long


def test_bench_launch_sampled_units(oracle):
    """The exact bench.py --path sweep launch (4096 replicas x 8 sim-GPUs, seed 1000, <= 8 batches):
    sampled GPU-epochs (<= 6 batches, so the oracle's brute force stays in seconds) re-derived."""
    P = synth_profiles()
    R, N = 4096, 8
    batches, off, arr, cur = epoch_batches(1000, R, N, max_batches=8)
    g = _gpu_sweep(P, R, N, batches, off, arr, cur)
    b = np.diff(off)
    rng = np.random.default_rng(5)
    picks = [u for u in rng.permutation(R * N)[:400] if b[u] <= 6][:12] + [0, R * N - 1]
    for u in picks:
        if b[u] > 6:
            continue
        lo, hi = int(off[u]), int(off[u + 1])
        sb = {k: v[lo:hi] for k, v in batches.items()}
        o = oracle.sweep(P, R=1, N=1, batches=sb, batch_off=[0, hi - lo], arrival=arr, cur_geom=cur[u:u + 1])
        assert g["sweep_key"][u * 12:(u + 1) * 12].tolist() == o["sweep_key"].tolist()
        assert g["assign"][u * 12:(u + 1) * 12].tolist() == o["assign"].tolist()
        assert g["best_key"][u] == o["best_key"][0]
