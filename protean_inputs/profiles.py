"""Seeded synthetic model-profile tables.

Input generator only: it holds none of the method's arithmetic (no Eq 1/2, no Alg 1/2).  Both the
CUDA library and the CPU oracle consume the tables it returns.  There is no real profiling data
(FBR estimation needs real GPUs), so the shapes are anchored to the paper:

* 22 models: 0-11 vision (batch 128), 12-21 language (batch 4); vision even = LI,
  odd = HI (F3); 12-19 VHI LLMs, 20-21 "GPT".
* solo on 7g ~ U[50, 200] ms; solo on profile p = round(solo7 * (7/compute_p)^gamma)
  with gamma ~ U[0.02, 1.26] (1g vs 3g up to 4x; ALBERT 2.15x).
* FBR on 7g: LI U[.15,.45], HI U[.45,.80], VHI U[.70,.95], GPT min(1, 1.42 x VHI draw)
  ("59% higher", "42% higher"); per profile scaled by compute fraction / cache
  fraction (T2).
* footprint per batch: LI U[2,6] GiB, HI U[4,10] GiB, language U[6,14] GiB.
* SLO = 3 x solo on 7g; batch timeout = SLO/3 (reading Q14).
"""
from __future__ import annotations

import dataclasses
import numpy as np

COMPUTE = np.array([1, 2, 3, 4, 7], dtype=np.float64)   # sevenths, T2
EIGHTHS = np.array([1, 2, 4, 4, 8], dtype=np.float64)   # cache eighths, T2


@dataclasses.dataclass
class Profiles:
    solo_us: np.ndarray      # int32 [M,5]
    fbr_ppm: np.ndarray      # int32 [M,5]
    mem_mib: np.ndarray      # int32 [M]
    batch_size: np.ndarray   # int32 [M]
    slo_us: np.ndarray       # int32 [M]
    timeout_us: np.ndarray   # int32 [M]
    geometry_set: int = 0
    geoms: np.ndarray | None = None   # uint8 [G,8] for geometry_set == 2
    names: tuple = ()
    gpu_mem_mib: int = 0              # N4c: GPU memory (0 = A100-40GB, 40960 MiB)

    @property
    def n_models(self) -> int:
        return int(self.solo_us.shape[0])

    def with_geometry_set(self, gs: int, geoms=None) -> "Profiles":
        return dataclasses.replace(self, geometry_set=gs,
                                   geoms=None if geoms is None else np.asarray(geoms, np.uint8))


def _finish(solo7, gamma, fbr7, mem, bsz, names):
    solo = np.rint(solo7[:, None] * (7.0 / COMPUTE[None, :]) ** gamma[:, None]).astype(np.int64)
    solo[:, 4] = solo7
    fbr = np.minimum(1e6, np.rint(fbr7[:, None] * (COMPUTE / 7.0) / (EIGHTHS / 8.0) * 1e6))
    slo = 3 * solo7
    return Profiles(solo_us=solo.astype(np.int32), fbr_ppm=fbr.astype(np.int32),
                    mem_mib=np.asarray(mem, np.int32), batch_size=np.asarray(bsz, np.int32),
                    slo_us=slo.astype(np.int32), timeout_us=(slo // 3).astype(np.int32),
                    names=tuple(names))


def synth_profiles(seed: int = 20241202, n_vision: int = 12, n_language: int = 10) -> Profiles:
    """The 22-model table of configs 2-5 (d.1)."""
    rng = np.random.Generator(np.random.PCG64(seed))
    M = n_vision + n_language
    solo7 = rng.integers(50_000, 200_001, size=M).astype(np.int64)
    gamma = rng.uniform(0.02, 1.26, size=M)
    fbr7 = np.zeros(M)
    mem = np.zeros(M, np.int64)
    names = []
    for m in range(M):
        if m < n_vision:
            if m % 2 == 0:
                fbr7[m] = rng.uniform(0.15, 0.45)
                mem[m] = rng.integers(2048, 6145)
                names.append(f"vision-LI-{m}")
            else:
                fbr7[m] = rng.uniform(0.45, 0.80)
                mem[m] = rng.integers(4096, 10241)
                names.append(f"vision-HI-{m}")
        else:
            v = rng.uniform(0.70, 0.95)
            if m < M - 2:
                fbr7[m] = v
                names.append(f"lang-VHI-{m}")
            else:
                fbr7[m] = min(1.0, 1.42 * v)
                names.append(f"lang-GPT-{m}")
            mem[m] = rng.integers(6144, 14337)
    bsz = np.array([128] * n_vision + [4] * n_language)
    return _finish(solo7, gamma, fbr7, mem, bsz, names)


def c1_profiles(seed: int = 1) -> Profiles:
    """Config 1: 3 models — vision-LI (B=8), vision-HI (B=8), VHI language (B=4) (d.2)."""
    rng = np.random.Generator(np.random.PCG64(seed + 7919))
    solo7 = rng.integers(50_000, 200_001, size=3).astype(np.int64)
    gamma = rng.uniform(0.02, 1.26, size=3)
    fbr7 = np.array([rng.uniform(0.15, 0.45), rng.uniform(0.45, 0.80), rng.uniform(0.70, 0.95)])
    mem = np.array([rng.integers(2048, 6145), rng.integers(4096, 10241), rng.integers(6144, 14337)])
    return _finish(solo7, gamma, fbr7, mem, [8, 8, 4], ["vision-LI", "vision-HI", "lang-VHI"])


def random_profiles(rng: np.random.Generator, M: int, *, small_time: bool = False,
                    max_batch: int = 8) -> Profiles:
    """Fuzzing tables: any valid values (wide FBR / footprint ranges, tiny batches)."""
    base = 300 if small_time else 50_000
    solo7 = rng.integers(base, 4 * base + 1, size=M).astype(np.int64)
    gamma = rng.uniform(0.0, 1.5, size=M)
    fbr7 = rng.uniform(0.05, 1.0, size=M)
    mem = rng.integers(512, 24_000, size=M)
    bsz = rng.integers(1, max_batch + 1, size=M)
    p = _finish(solo7, gamma, fbr7, mem, bsz, [f"m{i}" for i in range(M)])
    p.timeout_us[:] = rng.integers(0, 2 * base, size=M).astype(np.int32)
    return p
