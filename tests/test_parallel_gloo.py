"""Mode R host logic with world_size 2 over gloo on CPU: sharded replay + gather is byte-identical
to a single-process replay (the CPU oracle stands in for the GPU backend here)."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

from paper_conf_middleware_bhasisjgpkd24_b200.parallel import replica_range


def test_replica_range_partitions():
    for n in range(0, 23):
        for w in range(1, 6):
            rs = [replica_range(n, w, k) for k in range(w)]
            assert rs[0][0] == 0 and rs[-1][1] == n
            assert all(a[1] == b[0] for a, b in zip(rs, rs[1:]))
            assert max(h - l for l, h in rs) - min(h - l for l, h in rs) <= 1


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from oracle import oracle as O
    from paper_conf_middleware_bhasisjgpkd24_b200.parallel import max_over_ranks, run_sharded
    from protean_inputs import random_profiles, uniform_trace
    rng = np.random.default_rng(42)
    prof = random_profiles(rng, 4)
    tr = uniform_trace(rng, 5, 4, 6_000_000, 300)
    tr.replica_base = 10

    def backend(sub, **cfg):
        return O.replay(prof, sub, N=3, vm_policy=2, p_rev=0.5, rev_interval=2_000_000,
                        notice=500_000, seed=3)
    got = run_sharded(backend, tr, world, rank)
    t = max_over_ranks(float(rank + 1))
    if rank == 0:
        full = backend(tr)
        ok = all(np.array_equal(got[k], full[k]) for k in got) and set(got) >= {"counters", "hist"}
        q.put((ok, t))
    dist.barrier()
    dist.destroy_process_group()


def test_mode_r_sharded_equals_single_process():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    ok, t = q.get(timeout=120)
    for p in procs:
        p.join(timeout=60)
    assert ok and t == 2.0
