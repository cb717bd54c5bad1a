"""Pins of the oracle's policy 2 (N1, Alg 2's own heuristic) against hand-derived values.

The golden fixture T12 (tests/golden/t12_alg2_epochs.json) carries every decision, counter and the
arithmetic behind them, derived by hand from Alg 2 and the readings R10-R17 of DESIGN.md; the
boundary cases below are closed forms of lines 11 and 19 (inclusive capacity, strict threshold
comparisons) and of the (4g,3g) fallback (line 20)."""
import json
import os

import numpy as np
import pytest

from helpers import GOLDEN, tables
from protean_inputs import concat, pack_meta
from oracle import oracle

G43, G421 = 1, 2  # canonical indices in the 12-set (pinned in test_oracle_pins)


def _one_model(mem, n_models=1):
    return tables([[1000] * 5] * n_models, [[0] * 5] * n_models, [mem] * n_models,
                  bsz=[1] * n_models, tmo=[0] * n_models)


def _trace(per_epoch, offsets=(100_000, 300_000, 500_000, 600_000, 700_000, 800_000), strict=None,
           models=None):
    """per_epoch[e] BE (or strict) batch-size-1 requests in epoch e at e*W + offsets[i]."""
    arr, mdl, st = [], [], []
    for e, k in enumerate(per_epoch):
        for i in range(k):
            arr.append(e * 1_000_000 + offsets[i])
            mdl.append(models[e][i] if models is not None else 0)
            st.append(strict[e] if strict is not None else 0)
    return concat([(np.array(arr, np.uint32), pack_meta(np.array(mdl), np.array(st)))],
                  len(per_epoch) * 1_000_000)


@pytest.fixture(scope="module")
def t12():
    return json.load(open(os.path.join(GOLDEN, "t12_alg2_epochs.json")))


@pytest.mark.parametrize("alpha", [1000, 500])
def test_t12_golden(t12, alpha):
    P = _one_model(t12["model"]["mem_mib"])
    tr = _trace([2] * 4 + [3] * 8)
    exp = t12[f"alpha_{alpha}"]
    out = oracle.replay(P, tr, N=1, policy=2, ewma_alpha_pm=alpha, t_low=500, t_high=4000, want_keys=True)
    assert out["decisions"][0, :, 0].tolist() == exp["decisions"]
    c = out["counters"][0]
    assert c[7] == exp["reconfigs"] and c[4] == exp["be_arr"] and c[5] == exp["be_served"]
    assert c[6] == exp["be_drop"]
    assert c[8] == 0 and c[9] == 0  # no candidate is scored under policy 2 (R17)
    assert (out["cand_keys"] == -1).all()


def test_capacity_boundary_inclusive():
    # line 11: sum_max_mem(slice_set) >= pred_BE_mem; 3 x 5120 MiB = 15360 = 5 GB + 10 GB exactly
    out = oracle.replay(_one_model(5120), _trace([3] * 3), N=1, policy=2, ewma_alpha_pm=1000)
    assert out["decisions"][0, :, 0].tolist() == [G421] * 3
    out = oracle.replay(_one_model(5121), _trace([3] * 3), N=1, policy=2, ewma_alpha_pm=1000)
    assert out["decisions"][0, :, 0].tolist() == [G43] * 3  # [3g] chosen -> (4g,3g)


def test_thresholds_and_fallback():
    one = dict(N=1, policy=2, ewma_alpha_pm=1000)
    # pot = T_high exactly stays inside (line 19 compares with >); one more batch leaves it
    out = oracle.replay(_one_model(1024), _trace([4, 5]), t_low=500, t_high=4000, **one)
    assert out["decisions"][0, :, 0].tolist() == [G421, G43]
    # pot = T_low exactly stays inside (<); below it -> (4g,3g)
    out = oracle.replay(_one_model(1024), _trace([1, 1]), t_low=1000, t_high=4000, **one)
    assert out["decisions"][0, :, 0].tolist() == [G421, G421]
    out = oracle.replay(_one_model(1024), _trace([1, 1]), t_low=1001, t_high=4000, **one)
    assert out["decisions"][0, :, 0].tolist() == [G43, G43]
    # no small-slice set holds 4 x 6144 = 24576 MiB > 20480: found = False -> (4g,3g)
    out = oracle.replay(_one_model(6144), _trace([4, 4]), **one)
    assert out["decisions"][0, :, 0].tolist() == [G43, G43]
    # strict-only load: pred_BE_num = 0 < T_low -> (4g,3g); the 4th mismatch reconfigures
    out = oracle.replay(_one_model(1024), _trace([1] * 6, strict=[1] * 6), **one)
    assert out["decisions"][0, :, 0].tolist() == [G43] * 4 + [255, G43]
    assert out["counters"][0, 7] == 1


def test_mixed_footprints_sum():
    # pred_BE_mem sums the footprints of the observed BE batches (R10): 2048 + 4096 + 8192 = 14336
    # fits [1g,2g]; + 2048 more (16384) needs [3g]
    P = tables([[1000] * 5] * 3, [[0] * 5] * 3, [2048, 4096, 8192], bsz=[1] * 3, tmo=[0] * 3)
    tr = _trace([3, 4], models=[[0, 1, 2], [0, 1, 2, 0]])
    out = oracle.replay(P, tr, N=1, policy=2, ewma_alpha_pm=1000)
    assert out["decisions"][0, :, 0].tolist() == [G421, G43]


def test_cap_orders_by_gpu():
    # 4 GPUs, strict-only: every GPU wants (4g,3g) at its 4th mismatch; cap = max(1, 30*4/100) = 1,
    # granted by GPU index (R16): GPU 0 first, the next only after GPU 0's window closes
    P = _one_model(1024)
    per = [4] * 10
    tr = _trace(per, strict=[1] * 10)
    out = oracle.replay(P, tr, N=4, policy=2, ewma_alpha_pm=1000)
    dec = out["decisions"][0]
    assert dec[4, 0] == 255 and (dec[4, 1:] == G43).all()  # GPU 0 in its window at e4
    assert out["counters"][0, 7] >= 2


def test_policy2_requires_its_geometries():
    # an explicit set without (4g,3g) cannot run Alg 2 (R15)
    P = tables([[1000] * 5], [[0] * 5], [1024], geoms=[[4], [0, 1, 3]])
    with pytest.raises(oracle.OracleError) as e:
        oracle.replay(P, _trace([1]), N=1, policy=2)
    assert e.value.code == -1
    with pytest.raises(oracle.OracleError) as e:
        oracle.replay(_one_model(1024), _trace([1]), N=1, policy=2, ewma_alpha_pm=0)
    assert e.value.code == -1
    with pytest.raises(oracle.OracleError) as e:
        oracle.replay(_one_model(1024), _trace([1]), N=1, policy=2, t_low=10, t_high=5)
    assert e.value.code == -1
