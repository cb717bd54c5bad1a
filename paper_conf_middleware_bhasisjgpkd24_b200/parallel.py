"""Mode R (replica sharding): host-side logic for one process per GPU.

Replicas are independent, so rank k of n replays a contiguous replica range with no data-path
collective; global replica ids (replica_base) keep every VM draw rank-independent, so gathered
outputs are byte-identical to a 1-rank run.  torch.distributed is used only to gather results and
to take the max-over-ranks time.
"""
from __future__ import annotations

import numpy as np


def replica_range(n_total: int, world: int, rank: int) -> tuple[int, int]:
    """Balanced contiguous range [lo, hi) of rank `rank` among `world` ranks."""
    base, extra = divmod(n_total, world)
    lo = rank * base + min(rank, extra)
    return lo, lo + base + (1 if rank < extra else 0)


def shard_trace(trace, world: int, rank: int):
    """The rank's slice of a multi-replica trace (protean_inputs.Trace), replica ids preserved."""
    lo, hi = replica_range(trace.n_replicas, world, rank)
    sub = trace.subset(range(lo, hi)) if hi > lo else None
    if sub is not None:
        sub.replica_base = trace.replica_base + lo
    return sub, lo, hi


PER_REPLICA_KEYS = ("counters", "accum", "hist", "p50_p99", "cost", "util", "decisions", "n_batches")


def gather_rows(local: dict, world: int, keys=PER_REPLICA_KEYS):
    """Concatenate per-replica output rows of every rank in rank order (all ranks receive it)."""
    import torch.distributed as dist
    parts = [None] * world
    dist.all_gather_object(parts, {k: np.asarray(local[k]) for k in keys if k in local})
    out = {}
    for k in keys:
        rows = [p[k] for p in parts if p is not None and k in p and p[k].shape[0]]
        if rows:
            out[k] = np.concatenate(rows, axis=0)
    return out


def run_sharded(replay_fn, trace, world: int, rank: int, **cfg):
    """replay_fn(trace_slice, **cfg) -> dict of per-replica numpy rows; returns gathered rows."""
    sub, lo, hi = shard_trace(trace, world, rank)
    local = replay_fn(sub, **cfg) if sub is not None else {}
    return gather_rows(local, world)


def max_over_ranks(value: float) -> float:
    import torch
    import torch.distributed as dist
    t = torch.tensor([float(value)], dtype=torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


# ------------------------------------------------------------------------------------------------
# Mode G (geometry-range sharding): rank k scores geometries [b[k], b[k+1]) of
# protean_geometry_split and every rank runs the rest redundantly; the per-epoch min-loc exchange
# is fused into the replay kernel over peer memory (include/protean.h section 4).  The host side
# only wires the exchange buffers once: export -> all-gather of the 64-byte IPC handles -> import.

def setup_geometry_sharding(handle, world: int, rank: int, max_replicas: int, max_gpus: int):
    """Export this rank's exchange buffer, all-gather the IPC handles, map every peer's buffer."""
    import torch.distributed as dist
    mine = handle.xchg_export(world, rank, max_replicas, max_gpus)
    parts = [None] * world
    dist.all_gather_object(parts, (rank, mine))
    ordered = [h for _, h in sorted(parts)]
    assert [k for k, _ in sorted(parts)] == list(range(world))
    handle.xchg_import(ordered)
    return ordered


def merge_geometry_shards(outs: list, bounds: list[int]) -> dict:
    """Combine the per-rank outputs of one mode-G replay: every field is identical across ranks
    except counters 8/9 (each rank's own candidates: summed) and cand_keys (each rank's range)."""
    base = {k: (np.array(v, copy=True) if isinstance(v, np.ndarray) else v) for k, v in outs[0].items()}
    if "counters" in base:
        base["counters"][:, 8] = sum(np.asarray(o["counters"])[:, 8] for o in outs)
        base["counters"][:, 9] = sum(np.asarray(o["counters"])[:, 9] for o in outs)
    if "cand_keys" in base:
        for k, o in enumerate(outs):
            lo, hi = bounds[k], bounds[k + 1]
            base["cand_keys"][..., lo:hi] = np.asarray(o["cand_keys"])[..., lo:hi]
    return base
