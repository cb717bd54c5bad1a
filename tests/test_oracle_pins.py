"""Pins of the CPU oracle against what the paper and mathematics fix (not GPU).

Each test names the passage / closed form / brute force it pins (DESIGN.md §5 lists them).
"""
import itertools

import numpy as np
import pytest

from helpers import CAP, COMPUTE, NAMES, tables, trace_from, w1
from protean_inputs import concat, pack_meta, random_profiles, uniform_trace


# ---------------------------------------------------------------- O2: geometry set (T2)
def test_geometry_counts_and_canonical_order(oracle):
    g12, st = oracle.enumerate_geometries(0)
    assert st == dict(feasible=37, maximal_placements=19, placement_maximal_multisets=14,
                      multiset_maximal=12)
    names = [tuple(NAMES[x] for x in r if x != 255) for r in g12]
    assert names == [("7g",), ("3g", "4g"), ("1g", "2g", "4g"), ("1g", "1g", "1g", "4g"),
                     ("3g", "3g"), ("2g", "2g", "3g"), ("1g", "1g", "2g", "3g"),
                     ("1g", "1g", "1g", "1g", "3g"), ("1g", "2g", "2g", "2g"),
                     ("1g", "1g", "1g", "2g", "2g"), ("1g",) * 5 + ("2g",), ("1g",) * 7]
    assert sum(len([x for x in r if x != 255]) for r in g12) == 46
    g37, _ = oracle.enumerate_geometries(1)
    assert len(g37) == 37
    # (7g), (4g,3g), (4g,2g,1g) are indices 0, 1, 2 in both sets
    for g in (g12, g37):
        assert [tuple(x for x in r if x != 255) for r in g[:3]] == [(4,), (2, 3), (0, 1, 3)]


def test_geometry_placement_rule_equals_t2_sum_rule(oracle):
    """The oracle enumerates by MIG placement intervals; T2's sum constraints (counts, 7/7
    compute, 40 GB) must give the same multisets — brute force over all count vectors."""
    feasible = set()
    mem_units = [1, 2, 4, 4, 8]
    for c in itertools.product(*[range(m + 1) for m in (7, 3, 2, 1, 1)]):
        if sum(c) == 0:
            continue
        if sum(ci * k for ci, k in zip(c, COMPUTE)) <= 7 and sum(ci * u for ci, u in zip(c, mem_units)) <= 8:
            feasible.add(c)
    g37, _ = oracle.enumerate_geometries(1)
    got = {tuple(int(np.sum(r == p)) for p in range(5)) for r in g37}
    assert got == feasible
    maximal = {a for a in feasible
               if not any(b != a and all(bi >= ai for bi, ai in zip(b, a)) for b in feasible)}
    g12, _ = oracle.enumerate_geometries(0)
    assert {tuple(int(np.sum(r == p)) for p in range(5)) for r in g12} == maximal
    for c in feasible:  # T2 limits
        assert all(ci <= m for ci, m in zip(c, (7, 3, 2, 1, 1)))


# ---------------------------------------------------------------- Eq 1 / Eq 2 closed forms
def test_exec_closed_forms(oracle):
    assert oracle.exec_us(100_000, 1_300_000) == 130_000      # F = 0.7 + 0.6
    assert oracle.exec_us(100_000, 400_000) == 100_000        # alone / sum <= 1 -> Solo
    assert oracle.exec_us(100_000, 1_000_000) == 100_000
    assert oracle.exec_us(100_000, 2_000_000) == 200_000      # sum = 2 -> 2 x Solo
    assert oracle.exec_us(33_333, 1_500_001) == 49_999        # floor(49,999,533,333 / 10^6)
    assert oracle.exec_us(100_000, 1_200_000) == 120_000      # "FBR 0.2 -> 20%"


def _state(oracle, geom, residents=()):
    return oracle.new_state(geom, [(s, e, mem, sl, m, st) for (s, e, mem, sl, m, st) in residents])


def test_place_eq1_and_rdf(oracle):
    # model 0: RDF 1.3 on 4g ("+30%"), FBR 0.6; model 1 co-runner FBR 0.7 on 4g
    P = tables([[400_000, 220_000, 150_000, 130_000, 100_000],
                [400_000, 220_000, 150_000, 130_000, 100_000]],
               [[600_000] * 5, [700_000] * 5], [4096, 4096], geoms=[[3], [4]])
    S = _state(oracle, 0)
    r = oracle.place(P, S, 0, 0, 1)          # alone on 4g: exactly Solo_4g = 1.3 x Solo_7g
    assert (r["slice"], r["start"], r["end"]) == (0, 0, 130_000)
    S = _state(oracle, 0, [(0, 500_000, 4096, 0, 1, 0)])
    r = oracle.place(P, S, 10, 0, 1)         # F = 0.6 + 0.7 = 1.3 -> 130,000 * 1.3
    assert r["end"] - r["start"] == 169_000
    S = _state(oracle, 1, [(0, 500_000, 4096, 0, 1, 0)])
    r = oracle.place(P, S, 10, 0, 1)         # 7g: eta = RDF(1.0) x 1.3
    assert r["end"] - r["start"] == 130_000


# ---------------------------------------------------------------- Alg 1 tag walk (T1)
def test_tag_walk_T1(oracle):
    """(4g,2g,1g) ascends to 1g/2g/4g = 5120/10240/20480 MiB (Alg 1 lines 1-8)."""
    P = tables([[100_000] * 5, [100_000] * 5], [[100_000] * 5] * 2, [4096, 4096])  # default set
    for be_mem, expect in [(12288, [False, True, True]), (0, [True, True, True]),
                           (5120, [False, True, True]), (5119, [True, True, True]),
                           (15360, [False, False, True]), (35840, [False, False, False])]:
        # BE residents of total be_mem, spread on the 4g slice (position 2) in 1..4096 chunks
        res, left = [], be_mem
        while left > 0:
            q = min(4096, left)
            res.append((0, 900_000, q, 2, 1, 0))
            left -= q
        S = _state(oracle, 2, res)
        r = oracle.place(P, S, 10, 0, 1)
        assert list(r["eligible"][:3]) == expect, be_mem
    # none eligible -> fall back to every fitting slice (reading Q6): still placed
    S = _state(oracle, 2, [(0, 900_000, 4096, 2, 1, 0)] * 8 + [(0, 900_000, 3072, 2, 1, 0)])
    r = oracle.place(P, S, 10, 0, 1)
    assert not r["eligible"][:3].any() and r["dropped"] == 0


# ---------------------------------------------------------------- choose_strict_slice (T3)
def test_strict_choice_T3(oracle):
    # (4g,3g): positions 0 = 3g, 1 = 4g.  m0 solo 3g 150k, 4g 120k, 7g 100k, FBR 0.5.
    def run(corunner_fbr_4g):
        P = tables([[400_000, 220_000, 150_000, 120_000, 100_000], [100_000] * 5],
                   [[500_000] * 5, [0, 0, 0, corunner_fbr_4g, 0]], [4096, 4096])
        S = _state(oracle, 1, [(0, 10**6, 4096, 1, 1, 1)])     # strict co-runner on the 4g
        return oracle.place(P, S, 0, 0, 1)
    r = run(800_000)              # c(3g) = 150,000 < c(4g) = 156,000  (eta 1.5 vs 1.56)
    assert (r["slice"], r["s_end"][0], r["s_end"][1]) == (0, 150_000, 156_000)
    r = run(700_000)              # c(4g) = 144,000 -> 4g
    assert (r["slice"], r["s_end"][1]) == (1, 144_000)
    r = run(750_000)              # tie at 150,000 -> larger profile (4g)
    assert r["s_end"][0] == r["s_end"][1] == 150_000 and r["slice"] == 1


# ---------------------------------------------------------------- first fit + spill (T4, F7 P:L368)
def test_be_first_fit_and_spill_T4(oracle):
    P = tables([[100_000] * 5, [100_000] * 5], [[300_000] * 5] * 2, [4096, 4096])
    S = _state(oracle, 2)                       # (4g,2g,1g) -> 1g, 2g, 4g
    got = [oracle.place(P, S, 10 * i, 1, 0)["slice"] for i in range(4)]
    assert got == [0, 1, 1, 2]                  # 1g, 2g, 2g, then spill to the 4g
    r = oracle.place(P, S, 50, 0, 1)            # BE_mem 16384: only the 4g is eligible, shared
    assert list(r["eligible"][:3]) == [False, False, True] and r["slice"] == 2
    S = _state(oracle, 1)                       # (4g,3g): all four BE fit the 3g
    got = [oracle.place(P, S, 10 * i, 1, 0)["slice"] for i in range(4)]
    assert got == [0, 0, 0, 0]
    r = oracle.place(P, S, 50, 0, 1)
    assert r["slice"] == 1 and r["end"] - r["start"] == 100_000   # a BE-free 4g


# ---------------------------------------------------------------- FIFO memory wait (T5, Lindley)
def test_memory_wait_lindley_T5(oracle):
    P = tables([[100_000] * 5], [[200_000] * 5], [30720], geoms=[[4]])
    S = _state(oracle, 0)
    rs = [oracle.place(P, S, t, 0, 1) for t in (0, 50_000, 60_000)]
    assert [(r["start"], r["end"]) for r in rs] == [(0, 100_000), (100_000, 200_000), (200_000, 300_000)]
    # start_k = max(ready_k, end_{k-1})
    ready, prev = [0, 50_000, 60_000], 0
    for r, t in zip(rs, ready):
        assert r["start"] == max(t, prev)
        prev = r["end"]


# ---------------------------------------------------------------- no contention closed form
def test_no_contention_closed_form(oracle):
    rng = np.random.default_rng(5)
    M = 5
    solo = rng.integers(1000, 50_000, size=(M, 5))
    solo[0] = [5000, 4000, 3000, 3000, 2000]     # tie 3g/4g -> 4g
    P = tables(solo, np.zeros((M, 5)), np.ones(M), bsz=[3] * M, tmo=[20_000] * M)
    tr = uniform_trace(rng, 1, M, 2_000_000, 300, tie_frac=0.2)
    for strict_only in (True, False):
        meta = tr.meta.copy()
        meta = (meta & 63) | (np.uint8(128) if strict_only else np.uint8(0))
        t2 = concat([(tr.arrival_us, meta)], tr.trace_len_us)
        out = oracle.replay(P, t2, N=1, policy=1, init_geom=6, want_log=True)  # (3g,2g,1g,1g)
        geom = [0, 0, 1, 2]
        log = out["log"][0][: out["n_batches"][0]]
        for b in log:
            assert b["dropped"] == 0 and b["start"] == b["ready"]
            if strict_only:
                best = min(range(4), key=lambda s: (solo[b["model"], geom[s]], -geom[s], s))
            else:
                best = 0                               # first fit: the smallest slice
            assert b["slice"] == best
            assert b["end"] - b["start"] == solo[b["model"], geom[b["slice"]]]


# ---------------------------------------------------------------- tick simulator (2nd formulation)
def _random_case(rng, oracle, nb, geom_idx=None):
    M = 4
    P = random_profiles(rng, M, small_time=True)
    g12, _ = oracle.enumerate_geometries(0)
    j = int(rng.integers(0, 12)) if geom_idx is None else geom_idx
    t = np.sort(rng.integers(0, 600, size=nb))
    model = rng.integers(0, M, size=nb)
    strict = rng.integers(0, 2, size=nb)
    return P, j, t, model, strict


def test_tick_simulator_matches_event_driven(oracle):
    rng = np.random.default_rng(11)
    checked = 0
    for _ in range(60):
        P, j, t, model, strict = _random_case(rng, oracle, int(rng.integers(1, 12)))
        S = oracle.new_state(j)
        placed = []
        for i in range(len(t)):
            r = oracle.place(P, S, t[i], model[i], strict[i])
            if r["dropped"] == 0:
                placed.append((t[i], model[i], r["slice"], r["start"], r["end"]))
        if not placed:
            continue
        tt, mm, ss, st, en = map(np.array, zip(*placed))
        s2, e2 = oracle.tick_simulate(P, j, tt, mm, ss)
        assert np.array_equal(s2, st) and np.array_equal(e2, en)
        checked += len(placed)
    assert checked > 100


def test_greedy_is_per_step_argmin_bruteforce(oracle):
    """Brute force over every slice for each step (<= 4 batches): the event-driven choice is the
    argmin of Alg 1's rule, with start/end re-derived by the tick simulator and eligibility by
    the tag walk written out here."""
    rng = np.random.default_rng(12)
    for _ in range(80):
        P, j, t, model, strict = _random_case(rng, oracle, int(rng.integers(1, 5)))
        geom = [int(x) for x in oracle.table_geometries(P)[j] if x != 255]
        S = oracle.new_state(j)
        fixed = []   # (t, m, slice, strict)
        for i in range(len(t)):
            r = oracle.place(P, S, t[i], model[i], strict[i])
            q = P.mem_mib[model[i]]
            alts = {}
            for s in range(len(geom)):
                if q > CAP[geom[s]]:
                    continue
                rows = fixed + [(t[i], model[i], s, strict[i])]
                st, en = oracle.tick_simulate(P, j, [x[0] for x in rows], [x[1] for x in rows],
                                              [x[2] for x in rows])
                alts[s] = (st[-1], en[-1], st[:-1], en[:-1])
            if not alts:
                assert r["dropped"] == 2
                continue
            assert r["dropped"] == 0
            if strict[i]:
                some = next(iter(alts.values()))
                be_mem = sum(P.mem_mib[f[1]] for f, e in zip(fixed, some[3]) if not f[3] and e > t[i])
                R, elig = be_mem, []
                for s in range(len(geom)):
                    if R >= CAP[geom[s]]:
                        elig.append(False)
                        R -= CAP[geom[s]]
                    else:
                        elig.append(True)
                        R = 0
                cand = [s for s in alts if elig[s]] or list(alts)
                best = min(cand, key=lambda s: (alts[s][1], -geom[s], s))
            else:
                now = [s for s in sorted(alts) if alts[s][0] == t[i]]
                best = now[0] if now else min(alts, key=lambda s: (alts[s][0], s))
            assert r["slice"] == best
            assert (r["start"], r["end"]) == (alts[best][0], alts[best][1])
            fixed.append((t[i], model[i], best, strict[i]))


# ---------------------------------------------------------------- batch formation (T9)
def test_batch_formation_T9(oracle):
    P = tables([[1000] * 5], [[0] * 5], [100], bsz=[4], tmo=[100])
    arr = np.array([0, 10, 20, 30, 40, 150, 300], np.uint32)
    b = oracle.form_batches(P, arr, pack_meta(np.zeros(7), np.ones(7)))
    assert b["ready"].tolist() == [30, 140, 250, 400] and b["n"].tolist() == [4, 1, 1, 1]
    arr = np.array([0, 100, 101], np.uint32)           # exactly first + T joins
    b = oracle.form_batches(P, arr, pack_meta(np.zeros(3), np.ones(3)))
    assert b["n"].tolist() == [2, 1] and b["ready"].tolist() == [100, 201]
    # with no timeout pressure: #batches = sum ceil(n_r / B) (reactive scale-up)
    rng = np.random.default_rng(3)
    P = tables([[1000] * 5] * 3, [[0] * 5] * 3, [100] * 3, bsz=[4, 7, 1], tmo=[2**31 - 1] * 3)
    arr = np.sort(rng.integers(0, 10**6, size=500)).astype(np.uint32)
    model, strict = rng.integers(0, 3, 500), rng.integers(0, 2, 500)
    b = oracle.form_batches(P, arr, pack_meta(model, strict))
    expect = sum(-(-int(np.sum((model == m) & (strict == s))) // [4, 7, 1][m])
                 for m in range(3) for s in range(2))
    assert len(b["n"]) == expect and int(b["n"].sum()) == 500
    # id order: (ready, strict first, model, first index)
    keys = list(zip(b["ready"], 1 - b["strict"], b["model"], b["first_raw"]))
    assert keys == sorted(keys)


# ---------------------------------------------------------------- key (T10) and histogram (T11)
def test_key_T10(oracle):
    assert oracle.key(3, 250_000, 0) == 3_298_598_883_328
    assert oracle.key(0, 220_000, 1) == 56_320_001
    assert oracle.key(2**30, 2**40, 5) == ((2**23 - 1) << 40) | ((2**32 - 1) << 8) | 5  # saturation
    ks = [oracle.key(m, t, g) for m, t, g in [(0, 5, 3), (0, 5, 0), (1, 0, 0), (0, 6, 1)]]
    assert min(ks) == oracle.key(0, 5, 0)       # misses, then tail, then prefer current (tag 0)


def test_histogram_T11(oracle):
    assert [oracle.bucket(x) for x in (0, 100, 127, 128, 255, 256, 10**6, 2**32 - 1, 2**40)] == \
        [0, 100, 127, 128, 255, 256, 1780, 3327, 3327]
    assert oracle.bucket_lower(1780) == 999_424
    for b in range(0, 3328, 7):   # lower edge round trip and <= 1/128 width
        lo = oracle.bucket_lower(b)
        assert oracle.bucket(lo) == b
        if b >= 128:
            assert oracle.bucket(lo - 1) == b - 1
    h = np.zeros(3328, np.uint32)
    h[:100] = 1
    assert oracle.percentile(h, 99) == 98          # rank 99 of 100
    h[100] = 1
    assert oracle.percentile(h, 99) == 99          # rank ceil(99.99) = 100 of 101
    h[:] = 0
    h[500] = 1
    assert oracle.percentile(h, 99) == oracle.bucket_lower(500) and oracle.percentile(h, 50) == oracle.bucket_lower(500)
    assert oracle.percentile(np.zeros(3328, np.uint32), 50) == 0


def test_splitmix64_reference_vectors(oracle):
    # splitmix64 of state 0 + golden gamma: the published first output of SplitMix64(seed=0)
    from protean_inputs.traces import splitmix64
    assert int(splitmix64(np.array([0], np.uint64))[0]) == 0xE220A8397B1DCDAF
    d = oracle.vm_draw(7, 3, 2, 5, 1)
    inner = int(splitmix64(np.array([(3 << 32) ^ (2 << 20) ^ (5 << 2) ^ 1], np.uint64))[0])
    assert d == int(splitmix64(np.array([7 ^ inner], np.uint64))[0]) >> 11


# ---------------------------------------------------------------- W1 worked epoch (golden)
def test_w1_worked_epoch(oracle):
    g, P, tr = w1()
    ex = g["expected"]
    out = oracle.replay(P, tr, N=1, init_geom=2, want_keys=True, want_log=True)
    assert out["cand_keys"][0, 0, 0].tolist() == ex["cand_keys_epoch0"]
    assert out["decisions"][0, 0, 0] == ex["best_epoch0"]
    log = out["log"][0][: out["n_batches"][0]]
    assert [[b["ready"], b["n"], b["model"], b["strict"]] for b in log] == ex["batches_id_order"]
    assert [[b["slice"], b["start"], b["end"]] for b in log] == ex["actual_placement_j2"]
    assert out["p50_p99"][0].tolist() == ex["p50_p99_us"]
    for c, bk in enumerate(ex["p_buckets"]):
        assert [oracle.bucket(out["p50_p99"][0, c, q]) for q in range(2)] == bk
    hist = out["hist"][0]
    assert sorted(np.repeat(np.arange(3328), hist[0]).tolist()) == sorted(oracle.bucket(x) for x in ex["strict_latencies"])
    assert sorted(np.repeat(np.arange(3328), hist[1]).tolist()) == sorted(oracle.bucket(x) for x in ex["be_latencies"])
    c = out["counters"][0]
    assert c[0] == 4 and c[1] == 4 and c[4] == 4 and c[5] == 4
    # epoch 1 is idle: every key ties -> current geometry (T10) -> counters: 24 slot-evals total
    assert c[8] == ex["slot_evals_epoch0"] and c[9] == 2 * ex["geom_candidates_epoch0"]
    assert out["cand_keys"][0, 1, 0].tolist() == [1, 2, 0] and out["decisions"][0, 1, 0] == 2
    # O6e / O12 busy union, memory-time and utilisation (hand-derived in the golden)
    assert out["accum"][0, 0] == ex["accum_busy_weighted"]
    assert out["accum"][0, 1] == ex["accum_mem_time"]
    assert out["util"][0].tolist() == pytest.approx(ex["util"], rel=1e-12)


def test_w1_variants(oracle):
    g, P, tr = w1()
    ex = g["expected"]
    out = oracle.replay(P, tr, N=1, init_geom=0, want_keys=True)
    assert out["cand_keys"][0, 0, 0].tolist() == ex["variant_current_j0_keys"]
    assert out["decisions"][0, 0, 0] == 0
    P.slo_us[0] = 250_000
    out = oracle.replay(P, tr, N=1, init_geom=2, want_keys=True)
    v = ex["variant_slo_A_250000"]
    assert out["decisions"][0, 0, 0] == v["best"]
    assert int(out["cand_keys"][0, 0, 0].min()) == v["best_key"]
    assert out["cand_keys"][0, 0, 0, 0] >> 40 == v["j0_misses"]


def test_score_epoch_matches_w1(oracle):
    g, P, tr = w1()
    ex = g["expected"]
    arr = np.array([0, 5000, 0, 10000, 20000, 30000, 40000, 45000], np.uint32)
    batches = dict(ready=[5000, 10000, 30000, 45000], req_off=[0, 2, 4, 6], n=[2, 2, 2, 2],
                   model=[1, 0, 1, 0], strict=[0, 1, 0, 1])
    states = (oracle.State * 1)()
    states[0].geom, states[0].target, states[0].has_vm = 2, -1, 1
    out = oracle.score_epoch(P, R=1, N=1, epoch=0, batches=batches, batch_off=[0, 4], arrival=arr,
                             states=states)
    assert out["cand_key"].tolist() == ex["cand_keys_epoch0"]
    assert out["best_key"][0] == min(ex["cand_keys_epoch0"])
    assert [[s, a, b] for s, a, b in zip(out["slice"], out["start"], out["end"])] == ex["actual_placement_j2"]
    assert out["counters"][0, 8] == ex["slot_evals_epoch0"] and out["counters"][0, 9] == 3
    assert states[0].n_res == 4  # all four batches stay resident (every end > the epoch start)
    # per-slice busy union (O6e): 1g [5000,305000), 2g [30000,230000), 4g [10000,165000) (W1)
    assert list(states[0].busy_us) == [300_000, 200_000, 155_000, 0, 0, 0, 0]
    assert out["accum"][0, 0] == g["expected"]["accum_busy_weighted"]


def test_score_epoch_node_cost_closed_form(oracle):
    """Node-epoch VM cost = price(vm_type) x W (T3; cost projection P:L333; Q27 per-node
    price = T3 / 8): 8 nodes x 3600 one-second epochs on-demand sum to T3's AWS $32.7726 per hour,
    all spot to $9.8318 (the "70% lower cost" ratio 0.300001); no VM -> 0."""
    g, P, tr = w1()
    per = {}
    for vm, has in ((1, 1), (2, 1), (1, 0), (0, 1)):
        states = (oracle.State * 1)()
        states[0].geom, states[0].target, states[0].has_vm, states[0].vm_type = 2, -1, has, vm
        out = oracle.score_epoch(P, R=1, N=1, epoch=0, batches=dict(ready=[], req_off=[], n=[], model=[], strict=[]),
                                 batch_off=[0, 0], arrival=np.zeros(0, np.uint32), states=states,
                                 price_od=32.7726 / 8, price_spot=9.8318 / 8)
        per[(vm, has)] = float(out["cost"][0])
    assert per[(1, 0)] == 0.0 and per[(0, 1)] == 0.0
    assert 8 * 3600 * per[(1, 1)] == pytest.approx(32.7726, rel=1e-12)
    assert 8 * 3600 * per[(2, 1)] == pytest.approx(9.8318, rel=1e-12)
    assert per[(2, 1)] / per[(1, 1)] == pytest.approx(0.300001, abs=5e-7)


# ---------------------------------------------------------------- hysteresis (T6) + cap (T7)
def _w1_repeated(P, epochs, copies=1):
    """W1's request pattern repeated in every epoch on `copies` identical model pairs."""
    base = [(0, 0, 1), (0, 1, 0), (5000, 1, 0), (10000, 0, 1), (20000, 1, 0), (30000, 1, 0),
            (40000, 0, 1), (45000, 0, 1)]
    rows = []
    for e in range(epochs):
        for c in range(copies):
            rows += [(a + e * 1_000_000, m + 2 * c, s) for a, m, s in base]
    M = 2 * copies
    P2 = tables(np.tile(P.solo_us, (copies, 1)), np.tile(P.fbr_ppm, (copies, 1)),
                np.tile(P.mem_mib, copies), np.tile(P.batch_size, copies), np.tile(P.slo_us, copies),
                np.tile(P.timeout_us, copies), geoms=[[4], [2, 3], [0, 1, 3]])
    assert P2.n_models == M
    return P2, trace_from(rows, epochs * 1_000_000)


def test_hysteresis_T6(oracle):
    _, P, _ = w1()
    P, tr = _w1_repeated(P, 8)
    out = oracle.replay(P, tr, N=1, init_geom=2, want_keys=True, want_log=True)
    d = out["decisions"][0, :, 0].tolist()
    # epochs 0-3 mismatch (best 7g): ctr 1,2,3, then the 4th mismatch opens a window at T = 4 s
    assert d[:4] == [0, 0, 0, 0]
    assert out["counters"][0, 7] == 1
    # window [4 s, 6 s): undecidable in epoch 4; installed at 6 s <= T of epoch 5: current = 7g
    assert d[4] == 255 and d[5] == 0 and d[6] == 0
    log = out["log"][0][: out["n_batches"][0]]
    drops = [b for b in log if b["dropped"] == 1]
    assert drops and all(4_000_000 <= b["ready"] < 6_000_000 for b in drops)   # no dispatch in window
    assert all(b["dropped"] == 0 for b in log if b["ready"] >= 6_000_000)


def test_hysteresis_reset_on_match(oracle):
    _, P, _ = w1()
    P, tr = _w1_repeated(P, 3)
    # three mismatching epochs then idle epochs (best == current) -> ctr resets, never reconfigures
    out = oracle.replay(P, concat([tr.replica(0)], 12_000_000), N=1, init_geom=2)
    assert out["counters"][0, 7] == 0


def test_reconfig_cap_T7(oracle):
    _, P, _ = w1()
    P, tr = _w1_repeated(P, 5, copies=8)
    out = oracle.replay(P, tr, N=8, init_geom=2, want_keys=True)
    d = out["decisions"][0]
    # all 8 GPUs want (4th mismatch at T = 4 s); cap = max(1, floor(0.3 * 8)) = 2 (F7: "2 GPUs"),
    # chosen by (delta misses desc, gpu asc): GPUs 0 and 1 open windows [4 s, 6 s)
    assert (d[:4] == 0).all()
    assert list(d[4][:2]) == [255, 255] and (d[4][2:] != 255).all()
    assert out["counters"][0, 7] == 2   # epoch 4: 2 windows open -> no free slot; epoch 5 idle
    for alive, cap in [(8, 2), (1, 1), (3, 1), (64, 19)]:
        assert max(1, 30 * alive // 100) == cap


# ---------------------------------------------------------------- VM / cost (T8)
@pytest.mark.parametrize("od,spot,ratio", [(32.7726, 9.8318, 0.300001), (32.7700, 18.0235, 0.550000),
                                           (30.0846, 8.8147, 0.292997)])
def test_cost_T8(oracle, od, spot, ratio):
    P = tables([[1000] * 5], [[0] * 5], [100])
    tr = trace_from([(10, 0, 1)], 3_600_000_000)
    kw = dict(N=8, price_od=od / 8, price_spot=spot / 8, W=10_000_000)
    a = oracle.replay(P, tr, vm_policy=0, **kw)
    b = oracle.replay(P, tr, vm_policy=1, p_rev=0.0, **kw)
    H = a["E"] * 10_000_000
    assert a["accum"][0, 2] == 8 * H and b["accum"][0, 3] == 8 * H
    assert a["cost"][0] == pytest.approx(od * H / 3.6e9, rel=1e-12)
    assert round(b["cost"][0] / a["cost"][0], 6) == ratio


def test_vm_spot_only_p1_and_protean_p1(oracle):
    P = tables([[1000] * 5], [[0] * 5], [100], bsz=[1])
    rows = [(t, 0, 1) for t in range(0, 900_000_000, 7_000_000)]
    tr = trace_from(rows, 900_000_000)
    kw = dict(N=2, W=1_000_000, rev_interval=300_000_000, notice=30_000_000)
    out = oracle.replay(P, tr, vm_policy=2, p_rev=1.0, **kw)
    # every node revoked at 300 s with no spot replacement: billed 330 s each, then nothing
    assert out["accum"][0, 3] == 2 * 330_000_000 and out["accum"][0, 2] == 0
    assert out["counters"][0, 3] == sum(1 for t, _, _ in rows if t >= 300_000_000)
    assert (out["decisions"][0, 300:] == 255).all()
    out = oracle.replay(P, tr, vm_policy=1, p_rev=1.0, **kw)
    H = out["E"] * 1_000_000
    assert out["accum"][0, 3] == 2 * 330_000_000 and out["accum"][0, 2] == 2 * (H - 330_000_000)
    assert out["counters"][0, 3] == 0


def test_vm_mechanism_paths(oracle):
    """Every draw outcome of a small config-3 run, re-derived from the O11 mechanism with the
    specified counter-based draws."""
    P = tables([[1000] * 5], [[0] * 5], [100])
    tr = trace_from([(5, 0, 1)], 1_500_000_000)
    Trev, notice, W = 300_000_000, 30_000_000, 1_000_000
    seen = set()
    for seed in range(40):
        for pol in (1, 2):
            p_rev = 0.354 if seed % 2 else 0.708
            out = oracle.replay(P, tr, N=2, W=W, vm_policy=pol, p_rev=p_rev, seed=seed,
                                rev_interval=Trev, notice=notice)
            H = out["E"] * W
            thr = int(p_rev * 2**53)
            od = spot = 0
            for n in range(2):
                vm, since, bill = "spot", 0, "spot"
                acc = {"od": 0, "spot": 0, None: 0}
                path = []
                for k in range(1, 6):
                    tau = k * Trev
                    if tau >= H:
                        break
                    rev = oracle.vm_draw(seed, 0, n, k, 0) < thr
                    ok = oracle.vm_draw(seed, 0, n, k, 1) >= thr
                    path.append((vm, rev, ok))
                    if pol == 1 and vm == "spot" and rev and not ok:
                        acc[bill] += min(tau + notice, H) - since; vm, bill, since = "od", "od", tau + notice
                    elif pol == 1 and vm == "od" and ok:
                        acc[bill] += tau - min(since, H); vm, bill, since = "spot", "spot", tau
                    elif pol == 2 and vm == "spot" and rev and not ok:
                        acc[bill] += min(tau + notice, H) - since; vm, bill, since = None, None, tau + notice
                    elif pol == 2 and vm is None and ok:
                        vm, bill, since = "spot", "spot", tau
                if bill is not None:
                    acc[bill] += max(0, H - min(since, H))
                od += acc["od"]
                spot += acc["spot"]
                seen.add((pol, tuple(path)))
            assert out["accum"][0, 2] == od and out["accum"][0, 3] == spot, (seed, pol)
    assert len(seen) > 20


# ---------------------------------------------------------------- invariants on random replays
@pytest.mark.parametrize("seed", [1, 2, 3])
def test_replay_invariants(oracle, seed):
    rng = np.random.default_rng(seed)
    M = 5
    P = random_profiles(rng, M)
    tr = uniform_trace(rng, 3, M, 20_000_000, 800)
    for policy in (0, 1):
        out = oracle.replay(P, tr, N=3, policy=policy, want_log=True, nthreads=2, vm_policy=2 if seed == 3 else 0,
                            p_rev=0.5, rev_interval=5_000_000, notice=1_000_000)
        c = out["counters"]
        assert (c[:, 0] == c[:, 1] + c[:, 2] + c[:, 3]).all()           # strict conservation
        assert (c[:, 4] == c[:, 5] + c[:, 6]).all()                      # BE conservation
        for r in range(3):
            a, m = tr.replica(r)
            assert c[r, 0] == int(np.sum(m >> 7)) and c[r, 4] == int(np.sum((m >> 7) == 0))
            assert out["hist"][r, 0].sum() == c[r, 1] + c[r, 2] and out["hist"][r, 1].sum() == c[r, 5]
            log = out["log"][r][: out["n_batches"][r]]
            ok = log[log["dropped"] == 0]
            assert (ok["start"] >= ok["ready"]).all()
            assert (ok["end"] - ok["start"] >= P.solo_us[ok["model"]].min(axis=1)).all()
            if policy == 1 and seed != 3:   # fixed geometry (4g,2g,1g), no VM resets:
                # concurrent memory <= slice capacity at every start (T2, F7 spillage)
                caps = [5120, 10240, 20480]
                for g in range(3):
                    for s in range(3):
                        bs = ok[(ok["gpu"] == g) & (ok["slice"] == s)]
                        for b in bs:
                            live = bs[(bs["start"] <= b["start"]) & (bs["end"] > b["start"])]
                            assert P.mem_mib[live["model"]].sum() <= caps[s]
        # 1 thread vs 2 threads identical
        out1 = oracle.replay(P, tr, N=3, policy=policy, nthreads=1, vm_policy=2 if seed == 3 else 0,
                             p_rev=0.5, rev_interval=5_000_000, notice=1_000_000)
        for k in ("counters", "accum", "hist", "decisions"):
            assert np.array_equal(out1[k], out[k])


def test_error_codes(oracle):
    P = tables([[1000] * 5], [[0] * 5], [100])
    tr = trace_from([(5, 0, 1), (7, 0, 0)], 1_000_000)

    def code(f):
        try:
            f()
        except oracle.OracleError as e:
            return e.code
        return 0
    assert code(lambda: oracle.replay(P, concat([(np.array([7, 5], np.uint32), pack_meta([0, 0], [1, 1]))],
                                                 10**6))) == -1
    assert code(lambda: oracle.replay(P, concat([(np.array([5], np.uint32), pack_meta([3], [1]))], 10**6))) == -1
    bad = tables([[1000] * 5], [[1_000_001] * 5], [100])
    assert code(lambda: oracle.replay(bad, tr)) == -1
    bad = tables([[0] * 5], [[0] * 5], [100])
    assert code(lambda: oracle.replay(bad, tr)) == -1
    assert code(lambda: oracle.replay(P, tr, N=256)) == -2
    assert code(lambda: oracle.replay(tables([[1000] * 5], [[0] * 5], [100], geoms=[[4]] * 255), tr)) == -2
    assert code(lambda: oracle.replay(tables([[1000] * 5], [[0] * 5], [100], geoms=[[3, 4]]), tr)) == -1
    assert code(lambda: oracle.replay(P, concat([(np.array([5], np.uint32), pack_meta([0], [1]))], 2**32 + 5))) == -2
    assert code(lambda: oracle.replay(P, tr, policy=3)) == -1
    assert code(lambda: oracle.replay(P, tr)) == 0


# ---------------------------------------------------------------- O6e / O12 utilisation fixtures
def _util_golden():
    import json
    import os
    from helpers import GOLDEN
    return json.load(open(os.path.join(GOLDEN, "utilisation.json")))


def test_utilisation_clipped_at_horizon(oracle):
    """Busy = union of intervals per slice, clipped to [0, H); memory-time clipped likewise
    (readings Q29, R8).  Hand-derived in tests/golden/utilisation.json."""
    u = _util_golden()["clip_past_H"]
    t = u["tables"]
    P = tables(t["solo_us"], t["fbr_ppm"], t["mem_mib"], t["batch_size"], t["slo_us"], t["timeout_us"],
               geoms=u["geoms"])
    out = oracle.replay(P, trace_from([tuple(r) for r in u["requests"]], u["trace_len_us"]), N=1,
                        init_geom=u["init_geom"], want_log=True)
    log = out["log"][0][: out["n_batches"][0]]
    assert [[b["start"], b["end"]] for b in log] == u["placements"]
    assert out["accum"][0, 0] == u["busy_weighted"]
    assert out["accum"][0, 1] == u["mem_time"]
    assert out["util"][0].tolist() == pytest.approx(u["util"], rel=1e-12)
    c = out["counters"][0]
    assert c[0] == 3 and c[1] == 3  # the batch ending after H still counts for latency (R8)


def test_utilisation_across_reconfiguration(oracle):
    """Busy summed over every slice instance ever installed (O12): W1 on (4g,2g,1g), a window,
    then W1 shifted onto the installed (7g).  Hand-derived in tests/golden/utilisation.json."""
    u = _util_golden()["across_reconfiguration"]
    g, P, _ = w1()
    base = [tuple(r) for r in g["requests"]]
    rows = base + [(a + u["shift_us"], m, s) for a, m, s in base]
    out = oracle.replay(P, trace_from(rows, u["trace_len_us"]), N=1, init_geom=2,
                        wait_limit=u["wait_limit"], reconfig_us=u["reconfig_us"], want_log=True)
    log = out["log"][0][: out["n_batches"][0]]
    assert [[b["start"], b["end"]] for b in log[4:]] == u["epoch1_placements_7g"]
    assert all(b["slice"] == 0 for b in log[4:])
    assert out["counters"][0, 7] == u["reconfigs"]
    assert out["decisions"][0, :, 0].tolist() == u["decisions_epoch0_2"]
    assert out["accum"][0, 0] == u["busy_weighted"]
    assert out["accum"][0, 1] == u["mem_time"]
    assert out["util"][0].tolist() == pytest.approx(u["util"], rel=1e-12)


def test_w1_workload_self_check_stats(oracle):
    """The h5 self-check counters on W1, hand-counted: 2 decidable GPU-epochs, 1 with
    best != current (epoch 0: (7g) vs (4g,2g,1g)); 24 (batch, feasible slice) candidate evaluations,
    9 with Eq 1's F > 10^6: (7g) a1 1.3, b2 2.1, a2 2.6; (4g,3g) a1@3g 1.3, b2@3g 1.6, b2@4g 1.3,
    a2@3g 2.1 (a2@4g is exactly 1.0); (4g,2g,1g) b2@4g 1.3, a2@2g 1.3 (the 1g starts wait until b1
    ends at 305,000 and run alone)."""
    _, P, tr = w1()
    out = oracle.replay(P, tr, N=1, init_geom=2)
    assert out["stats"][0].tolist() == [2, 1, 9, 24]
