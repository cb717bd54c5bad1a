"""Seeded synthetic request traces.  Input generator only.

Storage (5 B / request): per replica, `arrival_us` uint32 sorted non-decreasing, `meta` uint8
(bits 0-5 model id, bit 7 strict), concatenated with `replica_off` int64 [R+1].

Generators
----------
* ``c1_trace``  — config 1: 200 arrivals iid U[0, 1 s) sorted (a Poisson process conditioned on
  n = 200), model uniform over 3, strict ~ Bernoulli(0.5).
* ``uniform_trace`` — fuzzing: any valid trace (random rates, ties, sparse/dense streams).
* ``GEN-1`` tick generator (``tick_trace``) for mixes A and B: time is cut into 16-us ticks; in
  tick i of replica r, source s (0 vision, 1 language) emits one request iff
  ``h >> 32 < thr[r, s, second(i)]`` with ``h = splitmix64(seed ^ splitmix64(r<<40 ^ i<<2 ^ s))``
  (a Bernoulli thinning of a piecewise-constant-rate process, ~Poisson at p <= 0.08 per tick).
  Arrival = 16 i + (h & 15); strict = bit 4 of h; model from bits 5..31 of h.  Rate tables are
  computed here in float64 once and passed as integers to both this numpy generator and its CUDA
  twin (tools/tracegen.cu), which therefore produce identical bytes.
  - Mix A (configs 5, paper-literal P:L343): vision only; Wiki-shaped rate
    5000 (1 + 0.0429 sin(2 pi t / 600 s + phi_r)) rps (peak:mean 316:303); one fixed
    strict model per replica (uniform over the 12 vision models); the BE model is re-drawn every
    20 s from the opposite LI/HI class.
  - Mix B (configs 2-4): vision MMPP-2 Twitter-shaped (5000 / 2800 rps, mean sojourns 5 s / 19.2 s,
    peak:mean ~ 4561:2969) + language Poisson 128 rps, models Zipf(1.0)
    within each domain with per-replica rank permutations; strict ~ Bernoulli(0.5).
"""
from __future__ import annotations

import dataclasses
import numpy as np

TICK_US = 16
U27 = (1 << 27) - 1
_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)


@dataclasses.dataclass
class Trace:
    arrival_us: np.ndarray   # uint32 [n]
    meta: np.ndarray         # uint8 [n]
    replica_off: np.ndarray  # int64 [R+1]
    trace_len_us: int
    replica_base: int = 0

    @property
    def n_replicas(self) -> int:
        return int(self.replica_off.shape[0] - 1)

    def replica(self, r: int) -> tuple[np.ndarray, np.ndarray]:
        lo, hi = int(self.replica_off[r]), int(self.replica_off[r + 1])
        return self.arrival_us[lo:hi], self.meta[lo:hi]

    def subset(self, rs) -> "Trace":
        arrs, metas, off = [], [], [0]
        for r in rs:
            a, m = self.replica(r)
            arrs.append(a)
            metas.append(m)
            off.append(off[-1] + a.shape[0])
        return Trace(np.concatenate(arrs).astype(np.uint32), np.concatenate(metas).astype(np.uint8),
                     np.asarray(off, np.int64), self.trace_len_us, self.replica_base)


def concat(parts: list[tuple[np.ndarray, np.ndarray]], trace_len_us: int, base: int = 0) -> Trace:
    off = np.zeros(len(parts) + 1, np.int64)
    for i, (a, _) in enumerate(parts):
        off[i + 1] = off[i] + a.shape[0]
    arr = np.concatenate([a for a, _ in parts]).astype(np.uint32) if parts else np.zeros(0, np.uint32)
    meta = np.concatenate([m for _, m in parts]).astype(np.uint8) if parts else np.zeros(0, np.uint8)
    return Trace(arr, meta, off, trace_len_us, base)


def pack_meta(model, strict) -> np.ndarray:
    return (np.asarray(model, np.uint8) & 63) | (np.asarray(strict, np.uint8) << 7)


def c1_trace(seed: int = 1, n: int = 200, n_models: int = 3, trace_len_us: int = 1_000_000) -> Trace:
    rng = np.random.Generator(np.random.PCG64(seed))
    arr = np.sort(rng.integers(0, trace_len_us, size=n)).astype(np.uint32)
    model = rng.integers(0, n_models, size=n)
    strict = rng.random(n) < 0.5
    return concat([(arr, pack_meta(model, strict))], trace_len_us)


def uniform_trace(rng: np.random.Generator, R: int, n_models: int, trace_len_us: int,
                  mean_n: int, tie_frac: float = 0.1) -> Trace:
    """Fuzzing: per replica ~mean_n requests, some exact ties, random models/classes."""
    parts = []
    for _ in range(R):
        n = int(rng.integers(0, 2 * mean_n + 1))
        arr = np.sort(rng.integers(0, trace_len_us, size=n))
        if n > 1 and tie_frac > 0:
            dup = rng.random(n) < tie_frac
            dup[0] = False
            idx = np.nonzero(dup)[0]
            arr[idx] = arr[idx - 1]
            arr = np.maximum.accumulate(arr)
        hot = rng.integers(0, n_models, size=max(1, n_models // 2 + 1))
        model = np.where(rng.random(n) < 0.7, rng.choice(hot, size=n), rng.integers(0, n_models, size=n))
        strict = rng.random(n) < rng.uniform(0.2, 0.8)
        parts.append((arr.astype(np.uint32), pack_meta(model, strict)))
    return concat(parts, trace_len_us)


# ------------------------------------------------------------------------------------------------
# GEN-1 counter-based tick generator
# ------------------------------------------------------------------------------------------------
def splitmix64(x: np.ndarray) -> np.ndarray:
    x = np.asarray(x, dtype=np.uint64)
    with np.errstate(over="ignore"):
        x = x + np.uint64(0x9E3779B97F4A7C15)
        x = (x ^ (x >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        x = (x ^ (x >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        return x ^ (x >> np.uint64(31))


def _u01(x) -> float:
    return float(int(splitmix64(np.array([x], np.uint64))[0]) >> 11) / float(1 << 53)


def _h(seed: int, *parts: int) -> int:
    v = np.uint64(seed & 0xFFFFFFFFFFFFFFFF)
    for p in parts:
        v = splitmix64(np.array([int(v) ^ (p & 0xFFFFFFFFFFFFFFFF)], np.uint64))[0]
    return int(v)


@dataclasses.dataclass
class GenParams:
    """Integer parameter tables shared by the numpy generator and its CUDA twin."""
    kind: int                 # 0 = mix A, 1 = mix B
    seed: int
    replica_base: int
    n_replicas: int
    seconds: int
    thr: np.ndarray           # uint32 [R, 2, seconds]  per-tick probability * 2^32
    strict_model: np.ndarray  # uint8 [R]               (mix A)
    be_model: np.ndarray      # uint8 [R, nseg]         (mix A, one per 20 s)
    cdf: np.ndarray           # uint32 [R, 2, 16]       (mix B) first k with u27 < cdf[k]
    model_base: tuple = (0, 12)

    @property
    def trace_len_us(self) -> int:
        return self.seconds * 1_000_000


def _thr(rate_rps) -> np.ndarray:
    p = np.asarray(rate_rps, np.float64) * TICK_US * 1e-6
    return np.minimum(np.floor(p * 4294967296.0), 4294967295.0).astype(np.uint32)


def mix_a_params(n_replicas: int, seed: int = 1, seconds: int = 600, replica_base: int = 0,
                 mean_rps: float = 5000.0) -> GenParams:
    R = n_replicas
    nseg = (seconds + 19) // 20
    thr = np.zeros((R, 2, seconds), np.uint32)
    strict_model = np.zeros(R, np.uint8)
    be_model = np.zeros((R, nseg), np.uint8)
    t = np.arange(seconds, dtype=np.float64) + 0.5
    for i in range(R):
        r = replica_base + i
        phi = 2 * np.pi * _u01(_h(seed, 0xA5, r))
        thr[i, 0] = _thr(mean_rps * (1.0 + 0.0429 * np.sin(2 * np.pi * t / 600.0 + phi)))
        sm = (_h(seed, 0x51, r) >> 32) * 12 >> 32
        strict_model[i] = sm
        opposite = 1 - (sm & 1)          # LI (even) <-> HI (odd)
        for s in range(nseg):
            be_model[i, s] = 2 * ((_h(seed, 0xBE, r, s) >> 32) * 6 >> 32) + opposite
    return GenParams(0, seed, replica_base, R, seconds, thr, strict_model, be_model,
                     np.zeros((R, 2, 16), np.uint32))


def _zipf_cdf(n: int, perm_key: int) -> np.ndarray:
    w = 1.0 / np.arange(1, n + 1)
    keys = [(_h(perm_key, k), k) for k in range(n)]
    order = [k for _, k in sorted(keys)]        # rank -> model slot
    wm = np.zeros(n)
    for rank, slot in enumerate(order):
        wm[slot] = w[rank]
    c = np.cumsum(wm) / wm.sum()
    out = np.full(16, U27 + 1, np.uint32)
    out[:n] = np.minimum(np.rint(c * (U27 + 1)), U27 + 1).astype(np.uint32)
    out[n - 1] = U27 + 1
    return out


def mix_b_params(n_replicas: int, seed: int = 1, seconds: int = 3600, replica_base: int = 0,
                 scale: float = 1.0, n_vision: int = 12, n_language: int = 10) -> GenParams:
    R = n_replicas
    thr = np.zeros((R, 2, seconds), np.uint32)
    cdf = np.zeros((R, 2, 16), np.uint32)
    p_hl, p_lh, pi_hi = 1.0 / 5.0, 1.0 / 19.2, 0.207
    for i in range(R):
        r = replica_base + i
        hi = _u01(_h(seed, 0x3A, r)) < pi_hi
        rate = np.zeros(seconds)
        for s in range(seconds):
            rate[s] = 5000.0 if hi else 2800.0
            u = _u01(_h(seed, 0x3B, r, s))
            hi = (u >= p_hl) if hi else (u < p_lh)
        thr[i, 0] = _thr(rate * scale)
        thr[i, 1] = _thr(np.full(seconds, 128.0 * scale))
        cdf[i, 0] = _zipf_cdf(n_vision, _h(seed, 0x2F, r, 0))
        cdf[i, 1] = _zipf_cdf(n_language, _h(seed, 0x2F, r, 1))
    return GenParams(1, seed, replica_base, R, seconds, thr, np.zeros(R, np.uint8),
                     np.zeros((R, 1), np.uint8), cdf, (0, n_vision))


def _gen_replica(gp: GenParams, i: int, chunk: int = 1 << 22):
    r = np.uint64(gp.replica_base + i)
    seed = np.uint64(gp.seed & 0xFFFFFFFFFFFFFFFF)
    nt = gp.seconds * (1_000_000 // TICK_US)
    arrs, metas = [], []
    nsrc = 1 if gp.kind == 0 else 2
    for lo in range(0, nt, chunk):
        tick = np.arange(lo, min(nt, lo + chunk), dtype=np.uint64)
        sec = (tick * np.uint64(TICK_US) // np.uint64(1_000_000)).astype(np.int64)
        ev_t, ev_src, ev_meta = [], [], []
        for s in range(nsrc):
            h = splitmix64(seed ^ splitmix64((r << np.uint64(40)) ^ (tick << np.uint64(2)) ^ np.uint64(s)))
            hit = (h >> np.uint64(32)).astype(np.uint32) < gp.thr[i, s][sec]
            h = h[hit]
            t = (tick[hit] * np.uint64(TICK_US) + (h & np.uint64(15))).astype(np.int64)
            strict = ((h >> np.uint64(4)) & np.uint64(1)).astype(np.uint8)
            u = ((h >> np.uint64(5)) & np.uint64(U27)).astype(np.uint32)
            if gp.kind == 0:
                seg = sec[hit] // 20
                model = np.where(strict == 1, gp.strict_model[i], gp.be_model[i][seg]).astype(np.uint8)
            else:
                c = gp.cdf[i, s]
                model = (np.searchsorted(c, u, side="right") + gp.model_base[s]).astype(np.uint8)
            ev_t.append(t)
            ev_src.append(np.full(t.shape, s, np.int64))
            ev_meta.append(pack_meta(model, strict))
        t = np.concatenate(ev_t)
        src = np.concatenate(ev_src)
        meta = np.concatenate(ev_meta)
        order = np.lexsort((src, t))            # by time, then source
        arrs.append(t[order].astype(np.uint32))
        metas.append(meta[order])
    return np.concatenate(arrs), np.concatenate(metas)


def tick_trace(gp: GenParams, replicas=None) -> Trace:
    rs = range(gp.n_replicas) if replicas is None else replicas
    parts = [_gen_replica(gp, i) for i in rs]
    base = gp.replica_base if replicas is None else gp.replica_base + (list(rs)[0] if len(rs) else 0)
    return concat(parts, gp.trace_len_us, base)
