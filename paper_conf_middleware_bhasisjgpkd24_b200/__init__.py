"""B200-native PROTEAN placement scorer and trace replayer (C ABI: include/protean.h).

    load_profiles(profiles) -> Handle;  Handle.score_epoch(...);  Handle.replay_traces(...)
    geometry_split(profiles, nranks); Handle.xchg_export / xchg_import / xchg_attach (mode G)

All computation runs in libprotean.so (hand-written sm_100a CUDA).  There is no CPU fallback.
"""
from ._abi import ProteanError, load as load_library  # noqa: F401
from .api import Handle, geometry_split, load_profiles  # noqa: F401
