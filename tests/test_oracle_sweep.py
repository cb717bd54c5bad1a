"""Pins of the oracle's exhaustive assignment sweep (N4a, the paper's "Oracle" scheme's offline
scheduling sweeps; readings R18-R21 of DESIGN.md) against things other than itself:
- the hand-derived T13 example (tests/golden/t13_sweep.json) where Alg 1's greedy misses an SLO
  that a different assignment meets;
- a brute force over every assignment whose start/end times come from the 1-us tick simulator
  (oracle/tick.cpp, a second formulation of O6(a)/(b)) and whose key is written out here;
- the invariant that Alg 1's greedy assignment is one of the candidates: sweep key <= the greedy
  candidate key of score_epoch for every geometry, equal for a single strict batch;
- the assignment count sum_j S_j^b."""
import itertools
import json
import os

import numpy as np
import pytest

from helpers import CAP, GOLDEN, tables
from protean_inputs import random_profiles
from oracle import oracle


def _key(misses, tail, tag):
    return (min(misses, (1 << 23) - 1) << 40) | (min(tail, 0xFFFFFFFF) << 8) | tag


@pytest.fixture(scope="module")
def t13():
    return json.load(open(os.path.join(GOLDEN, "t13_sweep.json")))


def _t13_inputs(g):
    m = g["models"]
    P = tables(m["solo_us"], m["fbr_ppm"], m["mem_mib"], bsz=[1, 1], slo=m["slo_us"], tmo=[0, 0])
    b = g["batches"]
    batches = dict(ready=b["ready"], req_off=list(range(len(b["ready"]))), n=[1] * len(b["ready"]),
                   model=b["model"], strict=b["strict"])
    return P, batches, b["arrival"]


def test_t13_golden(oracle, t13):
    P, batches, arrival = _t13_inputs(t13)
    j = t13["geometry_index"]
    out = oracle.sweep(P, R=1, N=1, batches=batches, batch_off=[0, 2], arrival=arrival, cur_geom=[0])
    assert out["sweep_key"][j] == t13["sweep"]["key"]
    assert out["assign"][j] == t13["sweep"]["assign"]
    assert out["n_assign"] == t13["n_assign"]
    # Alg 1's greedy candidate on the same geometry misses B's SLO
    st = (oracle.State * 1)()
    st[0].geom, st[0].target, st[0].has_vm = 0, -1, 1
    g = oracle.score_epoch(P, R=1, N=1, epoch=0, batches=batches, batch_off=[0, 2], arrival=arrival,
                           states=st)
    assert g["cand_key"][j] == t13["greedy"]["key"]


def _bruteforce(P, j, bs, arrival, tag):
    """Every assignment: drops by the footprint rule, times by the tick simulator, key by O8."""
    geom = [int(x) for x in oracle.table_geometries(P)[j] if x != 255]
    S = len(geom)
    best = None
    for idx, combo in enumerate(itertools.product(range(S), repeat=len(bs))):
        sl = combo[::-1]  # itertools varies the last position fastest; batch 0 = least significant
        keep = [x for x in range(len(bs)) if P.mem_mib[bs[x][1]] <= CAP[geom[sl[x]]]]
        end = {}
        if keep:
            st, en = oracle.tick_simulate(P, j, [bs[x][0] for x in keep], [bs[x][1] for x in keep],
                                          [sl[x] for x in keep])
            end = {x: int(e) for x, e in zip(keep, en)}
        misses = tail = 0
        for x, (t, m, strict, members) in enumerate(bs):
            if strict:
                misses += len(members) if x not in end else sum(end[x] - a > P.slo_us[m] for a in members)
            else:
                tail = max(tail, 0xFFFFFFFF if x not in end else end[x] - members[0])
        k = _key(misses, tail, tag)
        code = sum(s << (3 * x) for x, s in enumerate(sl))
        if best is None or k < best[0]:
            best = (k, code)
    return best


def _random_epoch(rng, M, nb):
    t = np.sort(rng.integers(0, 600, size=nb))
    bs, arrival, req_off = [], [], []
    for x in range(nb):
        n = int(rng.integers(1, 4))
        members = sorted(int(a) for a in rng.integers(max(0, t[x] - 50), t[x] + 1, size=n))
        req_off.append(len(arrival))
        arrival += members
        bs.append((int(t[x]), int(rng.integers(0, M)), int(rng.integers(0, 2)), members))
    batches = dict(ready=[b[0] for b in bs], req_off=req_off, n=[len(b[3]) for b in bs],
                   model=[b[1] for b in bs], strict=[b[2] for b in bs])
    return bs, batches, arrival


def test_bruteforce_tick_simulator(oracle):
    rng = np.random.default_rng(31)
    for _ in range(40):
        M = 3
        P = random_profiles(rng, M, small_time=True)
        nb = int(rng.integers(1, 4))
        bs, batches, arrival = _random_epoch(rng, M, nb)
        j = int(rng.integers(0, 12))
        cur = int(rng.integers(0, 12))
        out = oracle.sweep(P, R=1, N=1, batches=batches, batch_off=[0, nb], arrival=arrival, cur_geom=[cur],
                           geom_lo=j, geom_hi=j + 1)
        k, code = _bruteforce(P, j, bs, arrival, 0 if cur == j else j + 1)
        assert out["sweep_key"][0] == k and out["assign"][0] == code


def test_never_above_greedy(oracle):
    rng = np.random.default_rng(32)
    strictly_better = 0
    for trial in range(60):
        M = int(rng.integers(1, 5))
        P = random_profiles(rng, M)
        N = int(rng.integers(1, 4))
        parts, off, arrival = [], [0], []
        batches = dict(ready=[], req_off=[], n=[], model=[], strict=[])
        for g in range(N):
            nb = int(rng.integers(0, 5))
            bs, b, arr = _random_epoch(rng, M, nb)
            for k in batches:
                batches[k] += [v + len(arrival) for v in b[k]] if k == "req_off" else b[k]
            arrival += arr
            off.append(off[-1] + nb)
        cur = rng.integers(0, 12, size=N)
        st = (oracle.State * N)()
        for g in range(N):
            st[g].geom, st[g].target, st[g].has_vm = int(cur[g]), -1, 1
        ml = int(rng.choice([2, 64]))
        greedy = oracle.score_epoch(P, R=1, N=N, epoch=0, batches=batches, batch_off=off, arrival=arrival,
                                    states=st, max_live=ml)
        sw = oracle.sweep(P, R=1, N=N, batches=batches, batch_off=off, arrival=arrival, cur_geom=cur,
                          max_live=ml)
        assert (sw["sweep_key"] <= greedy["cand_key"]).all()
        assert (sw["best_key"] <= greedy["best_key"]).all()
        strictly_better += int((sw["sweep_key"] < greedy["cand_key"]).sum())
        sizes = [int((oracle.table_geometries(P)[j] != 255).sum()) for j in range(12)]
        assert sw["n_assign"] == sum(s ** (off[g + 1] - off[g]) for g in range(N) for s in sizes)
    assert strictly_better > 0  # the sweep does find better assignments than the greedy rule


def test_single_strict_batch_equals_greedy(oracle):
    rng = np.random.default_rng(33)
    for _ in range(30):
        P = random_profiles(rng, 3)
        bs, batches, arrival = _random_epoch(rng, 3, 1)
        batches["strict"] = [1]
        st = (oracle.State * 1)()
        st[0].geom, st[0].target, st[0].has_vm = 0, -1, 1
        g = oracle.score_epoch(P, R=1, N=1, epoch=0, batches=batches, batch_off=[0, 1], arrival=arrival, states=st)
        s = oracle.sweep(P, R=1, N=1, batches=batches, batch_off=[0, 1], arrival=arrival, cur_geom=[0])
        assert np.array_equal(g["cand_key"] >> 40, s["sweep_key"] >> 40)


def test_sweep_errors(oracle):
    P = tables([[1000] * 5], [[0] * 5], [100])
    b = dict(ready=[5] * 9, req_off=list(range(9)), n=[1] * 9, model=[0] * 9, strict=[1] * 9)
    arr = [5] * 9

    def code(**kw):
        try:
            oracle.sweep(P, R=1, N=1, arrival=arr, cur_geom=[0], **kw)
        except oracle.OracleError as e:
            return e.code
        return 0
    assert code(batches=b, batch_off=[0, 9]) == -2                       # > 8 batches on a GPU
    assert code(batches=b, batch_off=[0, 9], max_batches=9) == -1        # cap above 8
    assert code(batches=b, batch_off=[0, 3]) == 0
    bad = dict(b, model=[1] * 9)
    assert code(batches=bad, batch_off=[0, 3]) == -1                     # model id >= M
    bad = dict(b, ready=[5, 4, 6, 7, 8, 9, 10, 11, 12])
    assert code(batches=bad, batch_off=[0, 3]) == -1                     # ready not sorted
