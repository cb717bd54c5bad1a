"""Device-side twin of protean_inputs.traces GEN-1 (tools/tracegen.cu).  Input generation only:
builds a seeded synthetic trace directly in HBM (bench.py's 61 GB config-5 input).  Its bytes
equal the numpy generator's (checked by tests/test_tracegen.py on the GPU)."""
from __future__ import annotations

import ctypes as C

import numpy as np

from . import build_tools

_lib = None


def _load():
    global _lib
    if _lib is None:
        L = C.CDLL(build_tools.build())
        L.tracegen_scratch_elems.restype = C.c_int64
        L.tracegen_scratch_elems.argtypes = [C.c_int, C.c_int]
        args = [C.c_int, C.c_int, C.c_int, C.c_uint64, C.c_uint64, C.c_void_p, C.c_void_p, C.c_void_p,
                C.c_int, C.c_void_p, C.c_int]
        L.tracegen_count.argtypes = args + [C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p]
        L.tracegen_write.argtypes = args + [C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p]
        _lib = L
    return _lib


def generate_on_device(gp, device: int = 0):
    """Returns (arrival int32-view-of-uint32, meta uint8, replica_off int64) CUDA tensors."""
    import torch
    L = _load()
    dev = torch.device("cuda", device)
    thr = torch.from_numpy(np.ascontiguousarray(gp.thr).view(np.int32)).to(dev)
    sm = torch.from_numpy(np.ascontiguousarray(gp.strict_model)).to(dev)
    bm = torch.from_numpy(np.ascontiguousarray(gp.be_model)).to(dev)
    cdf = torch.from_numpy(np.ascontiguousarray(gp.cdf).view(np.int32)).to(dev)
    R = gp.n_replicas
    scratch = torch.empty(int(L.tracegen_scratch_elems(R, gp.seconds)), dtype=torch.int64, device=dev)
    roff = torch.empty(R + 1, dtype=torch.int64, device=dev)
    total = C.c_int64()
    st = torch.cuda.current_stream(dev).cuda_stream
    common = (gp.kind, R, gp.seconds, gp.seed & 0xFFFFFFFFFFFFFFFF, gp.replica_base, thr.data_ptr(),
              sm.data_ptr(), bm.data_ptr(), int(gp.be_model.shape[1]), cdf.data_ptr(), int(gp.model_base[1]))
    rc = L.tracegen_count(*common, scratch.data_ptr(), roff.data_ptr(), C.byref(total), C.c_void_p(st))
    if rc:
        raise RuntimeError(f"tracegen_count failed {rc}")
    n = int(total.value)
    arr = torch.empty(max(n, 1), dtype=torch.int32, device=dev)
    meta = torch.empty(max(n, 1), dtype=torch.uint8, device=dev)
    rc = L.tracegen_write(*common, scratch.data_ptr(), arr.data_ptr(), meta.data_ptr(), C.c_void_p(st))
    if rc:
        raise RuntimeError(f"tracegen_write failed {rc}")
    del scratch
    return arr[:n], meta[:n], roff
