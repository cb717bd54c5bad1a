"""N4b on the GPU (-m gpu): protean_sweep_depths bit-exact against the oracle's sweep_depths — the
hand-derived fixture tests/golden/n4b_reserve_depth.json, random tables and batch lists (ragged,
empty GPUs, the 37-geometry set, max_live limits), config-5-shaped GPU-epochs, a geometry range,
and the error code of an invalid batch list."""
import json
import os

import numpy as np
import pytest

from helpers import GOLDEN, tables
from protean_inputs import epoch_batches, pack_batch_rows, random_profiles, synth_profiles

pytestmark = pytest.mark.gpu


def _run(prof, R, N, batches, off, arr, cur, **kw):
    import torch
    import paper_conf_middleware_bhasisjgpkd24_b200 as pkg
    dev = torch.device("cuda", 0)
    h = pkg.load_profiles(prof, device=0)
    rows = pack_batch_rows({k: np.asarray(v) for k, v in batches.items()})
    g = h.sweep_depths(n_replicas=R, n_gpus=N, batches=torch.from_numpy(rows.reshape(-1).copy()).to(dev),
                       batch_off=torch.from_numpy(np.asarray(off, np.int32).copy()).to(dev),
                       arrival_us=torch.from_numpy(np.asarray(arr, np.uint32).view(np.int32).copy()).to(dev),
                       cur_geom=torch.from_numpy(np.asarray(cur, np.uint8).copy()).to(dev), **kw)
    return {k: v.cpu().numpy() for k, v in g.items()}


def _cmp(g, o):
    assert g["depth_key"].tolist() == o["depth_key"].tolist()
    assert g["depth_code"].tolist() == o["depth_code"].tolist()
    assert g["best_key"].tolist() == o["best_key"].tolist()
    assert int(g["n_eval"][0]) == o["n_eval"]


def test_golden(oracle):
    gd = json.load(open(os.path.join(GOLDEN, "n4b_reserve_depth.json")))
    m = gd["models"]
    P = tables(m["solo_us"], m["fbr_ppm"], m["mem_mib"], m["batch_size"], m["slo_us"], m["timeout_us"],
               geoms=gd["geoms"])
    b = gd["batches"]
    nb = len(b["ready"])
    batches = dict(ready=b["ready"], req_off=list(range(nb)), n=[1] * nb, model=b["model"], strict=b["strict"])
    arr = np.array(b["ready"], np.uint32)
    g = _run(P, 1, 1, batches, [0, nb], arr, [gd["current_geometry"]])
    assert g["depth_key"][0].tolist() == gd["expected"]["depth_key"]
    assert g["depth_code"][0].tolist() == gd["expected"]["depth_code"]
    o = oracle.sweep_depths(P, R=1, N=1, batches=batches, batch_off=[0, nb], arrival=arr,
                            cur_geom=[gd["current_geometry"]])
    _cmp(g, o)


@pytest.mark.parametrize("seed", range(5))
def test_random(oracle, seed):
    rng = np.random.default_rng(9100 + seed)
    M = 4
    P = random_profiles(rng, M, max_batch=4)
    if seed % 2:
        P = P.with_geometry_set(1)
    R, N = 2, 3
    b = dict(ready=[], req_off=[], n=[], model=[], strict=[])
    off, arr = [0], []
    for _ in range(R * N):
        for t in np.sort(rng.integers(0, 1_000_000, int(rng.integers(0, 12)))):
            n = int(rng.integers(1, 6))
            a = np.sort(rng.integers(max(0, t - 200_000), t + 1, n))
            b["ready"].append(int(t)); b["req_off"].append(len(arr)); b["n"].append(n)
            b["model"].append(int(rng.integers(0, M))); b["strict"].append(int(rng.integers(0, 2)))
            arr.extend(a.tolist())
        off.append(len(b["ready"]))
    G = 37 if seed % 2 else 12
    cur = rng.integers(0, G, R * N).astype(np.uint8)
    cur[0] = 255
    ml = [64, 3, 1, 64, 8][seed]
    lo, hi = (0, G) if seed < 3 else (2, G - 1)
    g = _run(P, R, N, b, off, np.array(arr, np.uint32), cur, max_live=ml, geom_lo=lo, geom_hi=hi)
    o = oracle.sweep_depths(P, R=R, N=N, batches=b, batch_off=off, arrival=np.array(arr, np.uint32), cur_geom=cur,
                            max_live=ml, geom_lo=lo, geom_hi=hi)
    _cmp(g, o)


def test_config5_shape(oracle):
    P = synth_profiles()
    batches, off, arr, cur = epoch_batches(77, 16, 8, max_batches=8)
    g = _run(P, 16, 8, batches, off, arr, cur)
    o = oracle.sweep_depths(P, R=16, N=8, batches=batches, batch_off=off, arrival=arr, cur_geom=cur)
    _cmp(g, o)
    assert (g["depth_code"] != 0).any()  # a depth beats the tags somewhere


def test_invalid(oracle):
    import paper_conf_middleware_bhasisjgpkd24_b200 as pkg
    P = synth_profiles()
    batches, off, arr, cur = epoch_batches(5, 1, 2, max_batches=4)
    batches = dict(batches)
    batches["model"] = np.array(batches["model"]).copy()
    batches["model"][0] = 99
    with pytest.raises(pkg.ProteanError) as e:
        _run(P, 1, 2, batches, off, arr, cur)
    assert e.value.code == -1
