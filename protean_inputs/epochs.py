"""Seeded synthetic GPU-epochs of dispatched batches (input generator only, no method arithmetic)
for protean_score_epoch / protean_sweep_assignments and their oracle twins.

``epoch_batches`` draws, per (replica, sim-GPU) unit, b ~ Poisson(mean_batches) clipped to
[0, max_batches] batches of one epoch [e W, (e+1) W): ready times iid uniform in the epoch, sorted;
model uniform over ``models``; strict ~ Bernoulli(strict_p); n members (``batch_size``, or
uniform in [1, batch_size] when ``ragged``) whose arrivals are iid uniform in
[ready - spread_us, ready] (clipped at 0), sorted, the last one at ready (a batch closes on its
last arrival).  The default shape is config 5's GPU-epoch (SURVEY §8 reference sizes: ~4.9
batches of 128 vision requests per sim-GPU and epoch).  cur_geom: iid uniform over G geometries.
"""
from __future__ import annotations

import numpy as np


def epoch_batches(seed: int, R: int, N: int, *, models=range(12), mean_batches: float = 4.9,
                  max_batches: int = 8, batch_size: int = 128, ragged: bool = False, epoch: int = 0,
                  W: int = 1_000_000, spread_us: int = 100_000, strict_p: float = 0.5, G: int = 12):
    rng = np.random.default_rng(seed)
    U = R * N
    b = np.minimum(rng.poisson(mean_batches, size=U), max_batches).astype(np.int64)
    batch_off = np.zeros(U + 1, np.int64)
    np.cumsum(b, out=batch_off[1:])
    nb = int(batch_off[-1])
    unit = np.repeat(np.arange(U), b)
    ready = (epoch * W + rng.integers(0, W, size=nb)).astype(np.int64)
    order = np.lexsort((ready, unit))  # sorted within each unit
    ready = ready[order]
    models = np.asarray(list(models), np.int64)
    model = models[rng.integers(0, models.shape[0], size=nb)]
    strict = (rng.random(nb) < strict_p).astype(np.int64)
    n = rng.integers(1, batch_size + 1, size=nb) if ragged else np.full(nb, batch_size, np.int64)
    req_off = np.zeros(nb + 1, np.int64)
    np.cumsum(n, out=req_off[1:])
    owner = np.repeat(np.arange(nb), n)
    lo = np.maximum(ready - spread_us, 0)
    arr = lo[owner] + (rng.random(owner.shape[0]) * (ready - lo + 1)[owner]).astype(np.int64)
    arr = np.minimum(arr, ready[owner])
    arr = arr[np.lexsort((arr, owner))]
    last = req_off[1:] - 1
    arr[last] = ready  # the member that closed the batch
    batches = dict(ready=ready.astype(np.uint32), req_off=req_off[:-1].astype(np.uint32), n=n.astype(np.int32),
                   model=model.astype(np.int32), strict=strict.astype(np.int32))
    cur_geom = rng.integers(0, G, size=U).astype(np.uint8)
    return batches, batch_off.astype(np.int32), arr.astype(np.uint32), cur_geom


def pack_batch_rows(batches) -> np.ndarray:
    """protean_batch rows (16 B: ready u32, req_off u32, n_req u16, model u8, strict u8, gpu u32)."""
    nb = batches["ready"].shape[0]
    dt = np.dtype([("ready", "<u4"), ("req_off", "<u4"), ("n", "<u2"), ("model", "u1"), ("strict", "u1"),
                   ("gpu", "<u4")])
    rows = np.zeros(nb, dt)
    rows["ready"] = batches["ready"]
    rows["req_off"] = batches["req_off"]
    rows["n"] = batches["n"]
    rows["model"] = batches["model"]
    rows["strict"] = batches["strict"]
    return rows.view(np.uint8).reshape(-1)
