"""ctypes mirror of include/protean.h (argument marshalling only).

Every step of the path runs in libprotean.so (hand-written sm_100a CUDA).  There is no CPU
fallback: if the shared library is missing, or no CUDA device is visible, loading fails loudly.
"""
from __future__ import annotations

import ctypes as C
import os

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "libprotean.so")

OK, EINVAL, ERANGE, ENOMEM, ECUDA, ENCCL, ESTATE, EUNSUP = 0, -1, -2, -3, -4, -5, -6, -7
ABI_VERSION = 1
NBUCKETS = 3328
MAX_LIVE = 64


class ProteanError(RuntimeError):
    def __init__(self, code: int, detail: str = ""):
        super().__init__(f"protean error {code} ({_strerror(code)}): {detail}")
        self.code = code


class Profiles(C.Structure):
    _fields_ = [("abi_version", C.c_int32), ("n_models", C.c_int32), ("solo_us", C.c_void_p),
                ("fbr_ppm", C.c_void_p), ("mem_mib", C.c_void_p), ("batch_size", C.c_void_p),
                ("slo_us", C.c_void_p), ("batch_timeout_us", C.c_void_p), ("geometry_set", C.c_int32),
                ("n_geoms", C.c_int32), ("geoms", C.c_void_p), ("device", C.c_int32),
                ("gpu_mem_mib", C.c_int32)]


class Batch(C.Structure):        # protean_batch, 16 B
    _fields_ = [("ready_us", C.c_uint32), ("req_off", C.c_uint32), ("n_req", C.c_uint16),
                ("model", C.c_uint8), ("strict", C.c_uint8), ("gpu", C.c_uint32)]


class Resident(C.Structure):     # protean_resident, 24 B
    _fields_ = [("start_us", C.c_int64), ("end_us", C.c_int64), ("mem_mib", C.c_int32),
                ("slice", C.c_uint8), ("model", C.c_uint8), ("strict", C.c_uint8), ("pad", C.c_uint8)]


class GpuState(C.Structure):     # protean_gpu_state
    _fields_ = [("geom", C.c_uint8), ("target", C.c_uint8), ("wait_ctr", C.c_uint8), ("n_live", C.c_uint8),
                ("has_vm", C.c_uint8), ("vm_type", C.c_uint8), ("pad", C.c_uint8 * 2),
                ("recfg_start_us", C.c_int64), ("recfg_end_us", C.c_int64),
                ("last_start_us", C.c_int64 * 7), ("busy_until_us", C.c_int64 * 7),
                ("busy_us", C.c_int64 * 7), ("live", Resident * MAX_LIVE)]


class Placement(C.Structure):    # protean_placement, 24 B
    _fields_ = [("start_us", C.c_int64), ("end_us", C.c_int64), ("slice", C.c_uint8),
                ("dropped", C.c_uint8), ("pad", C.c_uint8 * 6)]


class EpochIn(C.Structure):
    _fields_ = [("n_replicas", C.c_int32), ("n_gpus", C.c_int32), ("epoch", C.c_int32),
                ("max_live", C.c_int32), ("epoch_len_us", C.c_int64), ("horizon_us", C.c_int64),
                ("batches", C.c_void_p), ("batch_off", C.c_void_p), ("arrival_us", C.c_void_p),
                ("state", C.c_void_p), ("geom_lo", C.c_int32), ("geom_hi", C.c_int32),
                ("price_od_node_hr", C.c_double), ("price_spot_node_hr", C.c_double)]


class EpochOut(C.Structure):
    _fields_ = [("best_key", C.c_void_p), ("cand_key", C.c_void_p), ("placement", C.c_void_p),
                ("counters", C.c_void_p), ("accum", C.c_void_p), ("cost_usd", C.c_void_p)]


class ReplayCfg(C.Structure):
    _fields_ = [("n_replicas", C.c_int32), ("n_gpus", C.c_int32), ("replica_base", C.c_int64),
                ("trace_len_us", C.c_int64), ("epoch_len_us", C.c_int64), ("arrival_us", C.c_void_p),
                ("meta", C.c_void_p), ("replica_off", C.c_void_p), ("policy", C.c_int32),
                ("wait_limit", C.c_int32), ("reconfig_cap_pct", C.c_int32), ("init_geom", C.c_int32),
                ("max_live", C.c_int32), ("vm_policy", C.c_int32), ("reconfig_us", C.c_int64),
                ("p_rev", C.c_double), ("price_od_node_hr", C.c_double), ("price_spot_node_hr", C.c_double),
                ("rev_interval_us", C.c_int64), ("notice_us", C.c_int64), ("seed", C.c_uint64),
                ("shard_mode", C.c_int32), ("rank", C.c_int32), ("nranks", C.c_int32),
                ("max_ctas", C.c_int32), ("ewma_alpha_pm", C.c_int32), ("t_low_milli", C.c_int64),
                ("t_high_milli", C.c_int64), ("cold_start_us", C.c_int64), ("keepalive_epochs", C.c_int32),
                ("prewarm", C.c_int32), ("ctas_per_replica", C.c_int32), ("reserved2", C.c_int32)]


class SweepIn(C.Structure):      # protean_sweep_in
    _fields_ = [("n_replicas", C.c_int32), ("n_gpus", C.c_int32), ("max_live", C.c_int32),
                ("max_batches", C.c_int32), ("batches", C.c_void_p), ("batch_off", C.c_void_p),
                ("arrival_us", C.c_void_p), ("cur_geom", C.c_void_p), ("geom_lo", C.c_int32),
                ("geom_hi", C.c_int32)]


class SweepOut(C.Structure):     # protean_sweep_out
    _fields_ = [("sweep_key", C.c_void_p), ("assign", C.c_void_p), ("best_key", C.c_void_p),
                ("n_assign", C.c_void_p)]


class DepthOut(C.Structure):
    _fields_ = [("depth_key", C.c_void_p), ("depth_code", C.c_void_p), ("best_key", C.c_void_p),
                ("n_eval", C.c_void_p)]


class BatchRec(C.Structure):     # protean_batch_rec, 32 B
    _fields_ = [("ready_us", C.c_uint32), ("epoch", C.c_uint32), ("n_req", C.c_uint16), ("model", C.c_uint8),
                ("strict", C.c_uint8), ("gpu", C.c_uint8), ("slice", C.c_uint8), ("dropped", C.c_uint8),
                ("pad", C.c_uint8), ("start_us", C.c_int64), ("end_us", C.c_int64)]


class ReplayOut(C.Structure):
    _fields_ = [("counters", C.c_void_p), ("accum", C.c_void_p), ("hist", C.c_void_p),
                ("p50_p99_us", C.c_void_p), ("cost_usd", C.c_void_p), ("util", C.c_void_p),
                ("decisions", C.c_void_p), ("cand_keys", C.c_void_p), ("batch_log", C.c_void_p),
                ("batch_log_cap", C.c_int64), ("n_batches", C.c_void_p), ("cold_starts", C.c_void_p)]


assert C.sizeof(Batch) == 16 and C.sizeof(Resident) == 24 and C.sizeof(Placement) == 24
assert C.sizeof(BatchRec) == 32

EXPORTS = ["protean_load_profiles", "protean_free", "protean_strerror", "protean_last_error",
           "protean_get_geometries", "protean_num_epochs", "protean_score_epoch", "protean_score_epoch_status",
           "protean_replay_traces", "protean_replay_traces_host", "protean_replay_cfg_defaults", "protean_last_timings", "protean_last_search_ms",
           "protean_sweep_depths", "protean_geometry_split", "protean_xchg_export", "protean_xchg_import", "protean_xchg_attach"]
IPC_HANDLE_BYTES = 64

_lib = None


def load(path: str = None, require_cuda: bool = True):
    """Load libprotean.so (or the in-tree debug build named by PROTEAN_LIB, e.g. the racecheck
    variant).  Raises if the library (or, with require_cuda, a GPU) is missing."""
    global _lib
    if _lib is not None:
        return _lib
    if path is None:
        v = os.environ.get("PROTEAN_LIB")
        path = os.path.join(os.path.dirname(LIB_PATH), v) if v else LIB_PATH
    if not os.path.exists(path):
        raise ImportError(f"{path} is missing: run __graft_entry__.build() (nvcc, sm_100a)")
    L = C.CDLL(path)
    L.protean_load_profiles.argtypes = [C.c_void_p, C.c_void_p]
    L.protean_free.argtypes = [C.c_void_p]
    L.protean_free.restype = None
    L.protean_strerror.argtypes = [C.c_int]
    L.protean_strerror.restype = C.c_char_p
    L.protean_last_error.argtypes = [C.c_void_p]
    L.protean_last_error.restype = C.c_char_p
    L.protean_get_geometries.argtypes = [C.c_void_p, C.c_void_p, C.c_void_p]
    L.protean_num_epochs.argtypes = [C.c_void_p, C.c_int64, C.c_int64, C.c_void_p]
    L.protean_score_epoch.argtypes = [C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p]
    if hasattr(L, "protean_score_epoch_status"):
        L.protean_score_epoch_status.argtypes = [C.c_void_p]
    L.protean_sweep_assignments.argtypes = [C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p]
    if hasattr(L, "protean_sweep_depths"):  # (older experiment builds loaded by path lack it)
        L.protean_sweep_depths.argtypes = [C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p]
    L.protean_form_batches.argtypes = [C.c_void_p, C.c_void_p, C.c_int32, C.c_int32, C.c_void_p, C.c_void_p,
                                       C.c_void_p, C.c_void_p, C.c_void_p, C.c_int64, C.c_void_p]
    L.protean_replay_traces.argtypes = [C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p]
    if hasattr(L, "protean_replay_traces_host"):
        L.protean_replay_traces_host.argtypes = [C.c_void_p, C.c_void_p, C.c_void_p, C.c_int32, C.c_void_p]
    L.protean_replay_cfg_defaults.argtypes = [C.c_void_p]
    L.protean_replay_cfg_defaults.restype = None
    L.protean_last_timings.argtypes = [C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p]
    if hasattr(L, "protean_last_search_ms"):  # tolerant of older experiment builds
        L.protean_last_search_ms.argtypes = [C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p]
    L.protean_geometry_split.argtypes = [C.c_void_p, C.c_int32, C.c_void_p]
    L.protean_xchg_export.argtypes = [C.c_void_p, C.c_int32, C.c_int32, C.c_int32, C.c_int32, C.c_void_p]
    L.protean_xchg_import.argtypes = [C.c_void_p, C.c_void_p]
    L.protean_xchg_attach.argtypes = [C.c_void_p, C.c_int32, C.c_int32, C.c_int32]
    _lib = L
    return L


def _strerror(code: int) -> str:
    try:
        return load(require_cuda=False).protean_strerror(code).decode()
    except Exception:
        return str(code)
