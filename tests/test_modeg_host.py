"""Mode G host logic on CPU: the slot-balanced geometry split, the IPC-handle
wiring over torch.distributed (gloo, world_size 2), the per-rank output merge, and the min-loc
property the fused exchange relies on -- per-rank range minima of the packed O8 keys, reduced by
MIN across ranks, decode to the decisions a single full-range run takes (oracle keys)."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

from paper_conf_middleware_bhasisjgpkd24_b200 import _abi
from paper_conf_middleware_bhasisjgpkd24_b200.api import geometry_split
from paper_conf_middleware_bhasisjgpkd24_b200.parallel import merge_geometry_shards
from protean_inputs import c1_profiles

# slice counts of the 12 multiset-maximal geometries in canonical order (SURVEY §8(c) O2 list)
SLICES12 = [1, 2, 3, 4, 2, 3, 4, 5, 4, 5, 6, 7]


def test_split_two_ranks_by_hand():
    # 46 slots; the running count nearest 23 is 24, after geometry 7 (1+2+3+4+2+3+4+5)
    assert geometry_split(c1_profiles(), 2) == [0, 8, 12]
    assert geometry_split(c1_profiles(), 1) == [0, 12]
    assert geometry_split(c1_profiles(), 12) == list(range(13))


@pytest.mark.parametrize("gset", [0, 1])
def test_split_properties(gset):
    prof = c1_profiles().with_geometry_set(gset)
    G = 12 if gset == 0 else 37
    for n in range(1, G + 1):
        b = geometry_split(prof, n)
        assert b[0] == 0 and b[-1] == G and len(b) == n + 1
        assert all(x < y for x, y in zip(b, b[1:])), (n, b)
    if gset == 0:
        for n in (2, 3, 4):
            b = geometry_split(prof, n)
            loads = [sum(SLICES12[b[k]:b[k + 1]]) for k in range(n)]
            assert max(loads) - min(loads) <= max(SLICES12), (n, loads)
    for bad in (0, G + 1):
        with pytest.raises(_abi.ProteanError) as e:
            geometry_split(prof, bad)
        assert e.value.code == _abi.EINVAL


def test_merge_geometry_shards():
    R, E, N, G = 2, 3, 4, 12
    bounds = [0, 5, 12]
    rng = np.random.default_rng(0)
    full = rng.integers(0, 1 << 40, size=(R, E, N, G))
    outs = []
    for k in range(2):
        ck = np.full_like(full, 0)
        ck[..., bounds[k]:bounds[k + 1]] = full[..., bounds[k]:bounds[k + 1]]
        cnt = np.zeros((R, 10), np.int64)
        cnt[:, 0] = 7
        cnt[:, 8] = 10 * (k + 1)
        cnt[:, 9] = k + 1
        outs.append(dict(cand_keys=ck, counters=cnt, decisions=np.zeros((R, E, N), np.uint8)))
    m = merge_geometry_shards(outs, bounds)
    assert np.array_equal(m["cand_keys"], full)
    assert (m["counters"][:, 8] == 30).all() and (m["counters"][:, 9] == 3).all()
    assert (m["counters"][:, 0] == 7).all()


class _FakeHandle:
    """Stands in for the CUDA handle: export returns rank-tagged bytes, import records them."""

    def __init__(self):
        self.got = None

    def xchg_export(self, nranks, rank, max_replicas, max_gpus):
        return bytes([rank]) * 64

    def xchg_import(self, handles):
        self.got = handles


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from oracle import oracle as O
    from paper_conf_middleware_bhasisjgpkd24_b200.parallel import setup_geometry_sharding
    from protean_inputs import mix_a_params, synth_profiles, tick_trace
    h = _FakeHandle()
    setup_geometry_sharding(h, world, rank, 4, 8)
    wiring_ok = h.got == [bytes([k]) * 64 for k in range(world)]
    # min-loc over ranks of per-range minima == the full-range decision
    prof = synth_profiles()
    tr = tick_trace(mix_a_params(2, seed=5, seconds=12))
    o = O.replay(prof, tr, N=8, want_keys=True)
    keys = o["cand_keys"]                                 # [R][E][N][G], -1 = not scored
    b = geometry_split(prof, world)
    mine = keys[..., b[rank]:b[rank + 1]]
    big = np.iinfo(np.int64).max
    local = np.where(mine < 0, big, mine).min(axis=-1)
    t = torch.from_numpy(np.ascontiguousarray(local))
    dist.all_reduce(t, op=dist.ReduceOp.MIN)
    best = t.numpy()
    dec = o["decisions"]
    scored = dec != 255
    cur_tag = best & 255
    ok_dec = True
    for idx in zip(*np.nonzero(scored)):
        k = int(best[idx])
        full_min = int(keys[idx][keys[idx] >= 0].min())
        tag = k & 255
        ok_dec &= k == full_min and (tag == 0 or tag - 1 == int(dec[idx]))
    if rank == 0:
        q.put((wiring_ok, ok_dec, int(scored.sum()), int((cur_tag[scored] != 0).sum())))
    dist.barrier()
    dist.destroy_process_group()


def test_mode_g_wiring_and_minloc_gloo():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    wiring_ok, ok_dec, n_scored, n_switch = q.get(timeout=180)
    for p in procs:
        p.join(timeout=60)
    assert wiring_ok and ok_dec and n_scored > 0
