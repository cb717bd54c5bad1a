"""N4b: the BE-reserve depth as an enumerated dimension (reading R28), pinned
(-m "not gpu") by the hand-derived fixture tests/golden/n4b_reserve_depth.json (Alg 1's tag walk
reserves the 3g for BE that actually sits on the 4g; depth 0 frees it and saves the strict batch),
by the identities auto == Alg 1's greedy candidate key (score_epoch) and depth d >= S equivalent to
d = 0 (every slice ineligible -> the fallback), and by brute force: each depth's key equals the key
of the exhaustive assignment sweep restricted to the assignment Alg 1 makes under that depth."""
import json
import os

import numpy as np
import pytest

from helpers import GOLDEN, tables
from protean_inputs import random_profiles


def _fixture():
    g = json.load(open(os.path.join(GOLDEN, "n4b_reserve_depth.json")))
    m = g["models"]
    P = tables(m["solo_us"], m["fbr_ppm"], m["mem_mib"], m["batch_size"], m["slo_us"], m["timeout_us"],
               geoms=g["geoms"])
    b = g["batches"]
    nb = len(b["ready"])
    batches = dict(ready=b["ready"], req_off=list(range(nb)), n=[1] * nb, model=b["model"], strict=b["strict"])
    return g, P, batches, np.array(b["ready"], np.uint32)


def test_golden_reserve_depth(oracle):
    g, P, batches, arr = _fixture()
    ex = g["expected"]
    o = oracle.sweep_depths(P, R=1, N=1, batches=batches, batch_off=[0, len(arr)], arrival=arr,
                            cur_geom=[g["current_geometry"]])
    assert o["depth_key"][0].tolist() == ex["depth_key"]
    assert o["depth_code"][0].tolist() == ex["depth_code"]
    assert o["best_key"][0] == ex["best_key"]
    assert o["n_eval"] == ex["n_eval"]
    st = (oracle.State * 1)()
    st[0].geom, st[0].target, st[0].has_vm = g["current_geometry"], -1, 1
    s = oracle.score_epoch(P, R=1, N=1, epoch=0, batches=batches, batch_off=[0, len(arr)], arrival=arr, states=st)
    assert s["cand_key"].tolist() == ex["greedy_cand_keys"]


def _random_epoch(rng, M, N, nb_max=6):
    b = dict(ready=[], req_off=[], n=[], model=[], strict=[])
    off, arr = [0], []
    for _ in range(N):
        for t in np.sort(rng.integers(0, 1_000_000, int(rng.integers(0, nb_max + 1)))):
            n = int(rng.integers(1, 5))
            a = np.sort(rng.integers(max(0, t - 200_000), t + 1, n))
            b["ready"].append(int(t)); b["req_off"].append(len(arr)); b["n"].append(n)
            b["model"].append(int(rng.integers(0, M))); b["strict"].append(int(rng.integers(0, 2)))
            arr.extend(a.tolist())
        off.append(len(b["ready"]))
    return b, off, np.array(arr, np.uint32)


@pytest.mark.parametrize("seed", range(6))
def test_auto_is_greedy_and_depths_bounded(oracle, seed):
    rng = np.random.default_rng(8100 + seed)
    M, N = 4, 3
    P = random_profiles(rng, M, max_batch=4)
    b, off, arr = _random_epoch(rng, M, N)
    cur = rng.integers(0, 12, N).astype(np.uint8)
    o = oracle.sweep_depths(P, R=1, N=N, batches=b, batch_off=off, arrival=arr, cur_geom=cur)
    st = (oracle.State * N)()
    for x in range(N):
        st[x].geom, st[x].target, st[x].has_vm = int(cur[x]), -1, 1
    s = oracle.score_epoch(P, R=1, N=N, epoch=0, batches=b, batch_off=off, arrival=arr, states=st)
    G = 12
    dk = o["depth_key"]
    # code 0 (Alg 1's tags) is exactly the greedy candidate of O8
    assert dk[:, :, 0].reshape(-1).tolist() == s["cand_key"].tolist()
    geoms = oracle.table_geometries(P)
    for x in range(N):
        for j in range(G):
            S = int((geoms[j] != 255).sum())
            assert all(v == -1 for v in dk[x, j, S + 1:])
            assert all(v >= 0 for v in dk[x, j, : S + 1])
            code = int(o["depth_code"][x, j])
            assert dk[x, j, code] == dk[x, j, : S + 1].min()
            assert code == int(np.argmin(dk[x, j, : S + 1]))  # lowest code among equal keys
        assert o["best_key"][x] == dk[x][dk[x] >= 0].min()
    assert o["n_eval"] == sum(int((geoms[j] != 255).sum()) + 1 for j in range(G)) * N


@pytest.mark.parametrize("seed", range(4))
def test_depth_keys_are_assignments_of_the_sweep(oracle, seed):
    """Brute force: every depth's greedy replay is one assignment of the exhaustive sweep (N4a), so
    the sweep's minimum never exceeds the best depth, and depth 0 on a single-slice geometry is the
    sweep itself."""
    rng = np.random.default_rng(8200 + seed)
    M, N = 3, 2
    P = random_profiles(rng, M, max_batch=3)
    b, off, arr = _random_epoch(rng, M, N, nb_max=4)
    cur = np.zeros(N, np.uint8)
    d = oracle.sweep_depths(P, R=1, N=N, batches=b, batch_off=off, arrival=arr, cur_geom=cur)
    sw = oracle.sweep(P, R=1, N=N, batches=b, batch_off=off, arrival=arr, cur_geom=cur, max_batches=8)
    sk = sw["sweep_key"].reshape(N, -1)
    for x in range(N):
        for j in range(sk.shape[1]):
            dk = d["depth_key"][x, j]
            assert sk[x, j] <= dk[dk >= 0].min()
        assert sk[x, 0] == d["depth_key"][x, 0, 1]  # (7g): one slice, every assignment is Alg 1's
