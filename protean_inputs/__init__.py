"""Seeded synthetic inputs shared by the CUDA path and the CPU oracle (no method arithmetic)."""
from .profiles import Profiles, synth_profiles, c1_profiles, random_profiles  # noqa: F401
from .traces import (Trace, c1_trace, uniform_trace, concat, pack_meta, mix_a_params,  # noqa: F401
                     mix_b_params, tick_trace, GenParams)
from .epochs import epoch_batches, pack_batch_rows  # noqa: F401
