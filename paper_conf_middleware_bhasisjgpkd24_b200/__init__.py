"""B200-native PROTEAN placement scorer and trace replayer (C ABI: include/protean.h).

    load_profiles(profiles) -> Handle;  Handle.score_epoch(...);  Handle.replay_traces(...)
    geometry_split(profiles, nranks); Handle.xchg_export / xchg_import / xchg_attach (mode G)

All computation runs in libprotean.so (hand-written sm_100a CUDA).  There is no CPU fallback.
"""
import os as _os

# Mode-G ranks sharing one device run co-operating persistent kernels on separate streams; CUDA
# maps streams onto CUDA_DEVICE_MAX_CONNECTIONS hardware queues (default 8), and two streams on one
# queue serialise, which would hold a peer's kernel behind a spinning one.  Read at context
# creation: effective when this package is imported before CUDA is initialised.
_os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")

from ._abi import ProteanError, load as load_library  # noqa: E402,F401
from .api import Handle, geometry_split, load_profiles  # noqa: E402,F401
