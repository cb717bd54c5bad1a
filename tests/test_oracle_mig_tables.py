"""N4c: other MIG profile tables ("Generalizability"; the H100 / H200 / B200 tables are NVIDIA's
MIG user guide, not the paper).  Those GPUs keep T2's structure — compute sevenths 1,2,3,4,7, memory
eighths 1,2,4,4,8, max counts 7,3,2,1,1 — over a larger memory (80 / 141 / 180 GB), so the model is
the A100-40GB one with `gpu_mem_mib` scaling every slice capacity (the double-memory 1g profiles,
e.g. 1g.20gb / 1g.45gb, are not modelled).  Pins (-m "not gpu"):
* scale invariance: every memory quantity scaled by k (slice capacities AND footprints) leaves every
  decision, key, placement and histogram unchanged; memory-time scales by k, utilisation does not;
* a hand-derived decision that flips with the table: a 24,000 MiB strict batch cannot fit
  (4g,3g) on the A100-40GB (4g = 3g = 20,480 MiB) but fits both slices of the H100-80GB (40,960);
* validation: a footprint above the GPU's memory is EINVAL; the geometry set does not change."""
import dataclasses

import numpy as np
import pytest

from helpers import tables, trace_from
from protean_inputs import random_profiles, uniform_trace

H100_80 = 81920
B200_180 = 184320


def _scaled(P, k):
    return dataclasses.replace(P, mem_mib=(np.asarray(P.mem_mib, np.int64) * k).astype(np.int32),
                               gpu_mem_mib=40960 * k)


@pytest.mark.parametrize("seed", range(4))
def test_memory_scale_invariance(oracle, seed):
    rng = np.random.default_rng(4000 + seed)
    P = random_profiles(rng, 4, max_batch=6)
    tr = uniform_trace(rng, 2, 4, 8_000_000, 500)
    base = oracle.replay(P, tr, N=3, want_keys=True, want_log=True)
    for k in (2, 4):
        o = oracle.replay(_scaled(P, k), tr, N=3, want_keys=True, want_log=True)
        for key in ("counters", "decisions", "cand_keys", "hist", "p50_p99", "n_batches"):
            assert np.array_equal(o[key], base[key]), key
        assert np.array_equal(o["log"], base["log"])
        assert o["accum"][:, 0].tolist() == base["accum"][:, 0].tolist()
        assert o["accum"][:, 1].tolist() == (k * base["accum"][:, 1]).tolist()
        np.testing.assert_allclose(o["util"], base["util"], rtol=1e-12, atol=0)


def _flip_case(gpu_mem):
    P = tables([[400_000, 220_000, 150_000, 120_000, 100_000]], [[500_000] * 5], [24_000], bsz=[1], slo=[300_000],
               tmo=[0], geoms=[[4], [2, 3]])
    return dataclasses.replace(P, gpu_mem_mib=gpu_mem), trace_from([(10_000, 0, 1)], 1_000_000)


def test_decision_flips_with_the_mig_table(oracle):
    """A100-40GB: (4g,3g) has no slice for 24,000 MiB -> placement drop -> key(j=1, current) =
    1<<40 (one strict miss, tag 0); (7g) runs it in 100,000 us (met) -> key 0<<40 | 0<<8 | 1 = 1 ->
    best = (7g).  H100-80GB / B200-180GB: 4g holds it, c = 10,000 + 120,000 (3g: 160,000) -> met ->
    key(j=1) = 0 (tag 0) < key(j=0) = 1 -> best = current (4g,3g)."""
    P, tr = _flip_case(0)
    o = oracle.replay(P, tr, N=1, init_geom=1, want_keys=True, want_log=True)
    assert o["cand_keys"][0, 0, 0].tolist() == [1, 1 << 40]
    assert o["decisions"][0, 0, 0] == 0
    assert o["log"][0][0]["dropped"] == 2
    for mem in (H100_80, B200_180):
        P, tr = _flip_case(mem)
        o = oracle.replay(P, tr, N=1, init_geom=1, want_keys=True, want_log=True)
        assert o["cand_keys"][0, 0, 0].tolist() == [1, 0]
        assert o["decisions"][0, 0, 0] == 1
        b = o["log"][0][0]
        assert (b["dropped"], b["slice"], b["start"], b["end"]) == (0, 1, 10_000, 130_000)
        # memory utilisation over H = 1 s: 24,000 MiB x 120,000 us / (gpu_mem x 1 x 1e6)
        assert o["util"][0, 1] == pytest.approx(24_000 * 120_000 / (mem * 1e6), rel=1e-12)


def test_footprint_bound_and_geometry_set(oracle):
    P = tables([[1000] * 5], [[0] * 5], [50_000])
    with pytest.raises(oracle.OracleError) as e:
        oracle.replay(P, trace_from([(5, 0, 1)], 1_000_000))
    assert e.value.code == -1
    o = oracle.replay(dataclasses.replace(P, gpu_mem_mib=H100_80), trace_from([(5, 0, 1)], 1_000_000), init_geom=0)
    assert o["counters"][0, 1] == 1
    for bad in (H100_80 + 4, -8, (1 << 24) + 8):
        with pytest.raises(oracle.OracleError):
            oracle.replay(dataclasses.replace(P, gpu_mem_mib=bad), trace_from([(5, 0, 1)], 1_000_000))
    g40 = oracle.table_geometries(tables([[1000] * 5], [[0] * 5], [100]))
    g80 = oracle.table_geometries(dataclasses.replace(tables([[1000] * 5], [[0] * 5], [100]), gpu_mem_mib=H100_80))
    assert np.array_equal(g40, g80) and g40.shape[0] == 12
