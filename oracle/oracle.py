"""oracle/oracle.py — TEST INFRASTRUCTURE ONLY.

ctypes wrapper of oracle/liboracle.so (the plain C++17 CPU oracle of the PROTEAN epoch model).
Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may import
this module.  The product package never imports it.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
LIB = os.path.join(HERE, "liboracle.so")
NB = 3328


def build(force: bool = False) -> str:
    srcs = [os.path.join(HERE, f) for f in os.listdir(HERE) if f.endswith((".cpp", ".hpp", ".h"))]
    if force or not os.path.exists(LIB) or max(os.path.getmtime(s) for s in srcs) > os.path.getmtime(LIB):
        subprocess.check_call(["make", "-s", "-C", HERE, "-B" if force else "liboracle.so"])
    return LIB


class Tables(C.Structure):
    _fields_ = [("M", C.c_int32), ("solo", C.c_void_p), ("fbr", C.c_void_p), ("mem", C.c_void_p),
                ("bsz", C.c_void_p), ("slo", C.c_void_p), ("tmo", C.c_void_p),
                ("geometry_set", C.c_int32), ("n_geoms", C.c_int32), ("geoms", C.c_void_p),
                ("gpu_mem_mib", C.c_int32)]


class Res(C.Structure):
    _fields_ = [("start", C.c_int64), ("end", C.c_int64), ("mem", C.c_int32), ("slice", C.c_int32),
                ("model", C.c_int32), ("strict", C.c_int32)]


class State(C.Structure):
    _fields_ = [("geom", C.c_int32), ("target", C.c_int32), ("wait_ctr", C.c_int32),
                ("has_vm", C.c_int32), ("recfg_start", C.c_int64), ("recfg_end", C.c_int64),
                ("last_start", C.c_int64 * 7), ("busy_until", C.c_int64 * 7), ("busy_us", C.c_int64 * 7),
                ("vm_type", C.c_int32), ("n_res", C.c_int32), ("res", Res * 64)]


class ReplayIn(C.Structure):
    _fields_ = [("R", C.c_int32), ("N", C.c_int32), ("replica_base", C.c_int64),
                ("trace_len", C.c_int64), ("W", C.c_int64), ("arrival", C.c_void_p),
                ("meta", C.c_void_p), ("replica_off", C.c_void_p), ("policy", C.c_int32),
                ("wait_limit", C.c_int32), ("cap_pct", C.c_int32), ("init_geom", C.c_int32),
                ("max_live", C.c_int32), ("vm_policy", C.c_int32), ("reconfig_us", C.c_int64),
                ("p_rev", C.c_double), ("price_od", C.c_double), ("price_spot", C.c_double),
                ("rev_interval", C.c_int64), ("notice", C.c_int64), ("seed", C.c_uint64),
                ("shard_mode", C.c_int32), ("nthreads", C.c_int32),
                ("ewma_alpha_pm", C.c_int32), ("pad", C.c_int32), ("t_low", C.c_int64),
                ("t_high", C.c_int64), ("cold_us", C.c_int64), ("keepalive_epochs", C.c_int32),
                ("prewarm", C.c_int32)]


class BatchRec(C.Structure):
    _fields_ = [("ready", C.c_uint32), ("epoch", C.c_uint32), ("n", C.c_int32), ("model", C.c_int32),
                ("strict", C.c_int32), ("gpu", C.c_int32), ("slice", C.c_int32),
                ("dropped", C.c_int32), ("start", C.c_int64), ("end", C.c_int64)]


class ReplayOut(C.Structure):
    _fields_ = [("counters", C.c_void_p), ("accum", C.c_void_p), ("hist", C.c_void_p),
                ("p50_p99", C.c_void_p), ("cost", C.c_void_p), ("util", C.c_void_p),
                ("decisions", C.c_void_p), ("cand_keys", C.c_void_p), ("log", C.c_void_p),
                ("log_cap", C.c_int64), ("n_batches", C.c_void_p), ("cold_starts", C.c_void_p),
                ("stats", C.c_void_p)]


BATCH_REC_DTYPE = np.dtype([("ready", "<u4"), ("epoch", "<u4"), ("n", "<i4"), ("model", "<i4"),
                            ("strict", "<i4"), ("gpu", "<i4"), ("slice", "<i4"), ("dropped", "<i4"),
                            ("start", "<i8"), ("end", "<i8")])


def _p(a):
    return None if a is None else a.ctypes.data


class OracleError(RuntimeError):
    def __init__(self, code, what=""):
        super().__init__(f"oracle error {code} {what}")
        self.code = code


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(LIB)
        L.orc_exec_us.restype = C.c_int64
        L.orc_exec_us.argtypes = [C.c_int64, C.c_int64]
        L.orc_bucket.restype = C.c_int32
        L.orc_bucket.argtypes = [C.c_uint64]
        L.orc_bucket_lower.restype = C.c_uint64
        L.orc_bucket_lower.argtypes = [C.c_int32]
        L.orc_percentile.restype = C.c_uint64
        L.orc_percentile.argtypes = [C.c_void_p, C.c_int32]
        L.orc_vm_draw.restype = C.c_uint64
        L.orc_vm_draw.argtypes = [C.c_uint64] * 5
        L.orc_key.restype = C.c_int64
        L.orc_key.argtypes = [C.c_int64, C.c_int64, C.c_int32]
        L.orc_num_epochs.restype = C.c_int64
        L.orc_num_epochs.argtypes = [C.c_void_p, C.c_int64, C.c_int64]
        L.orc_form_batches.restype = C.c_int64
        L.orc_form_batches.argtypes = [C.c_void_p, C.c_void_p, C.c_void_p, C.c_int64] + [C.c_void_p] * 5 + [C.c_int64]
        L.orc_place.argtypes = [C.c_void_p, C.c_void_p, C.c_int64, C.c_int32, C.c_int32, C.c_int32,
                                C.c_int64] + [C.c_void_p] * 9
        L.orc_tick_simulate.argtypes = [C.c_void_p, C.c_int32, C.c_int32] + [C.c_void_p] * 5
        L.orc_enumerate.argtypes = [C.c_int32, C.c_void_p, C.c_void_p, C.c_void_p]
        L.orc_table_geometries.argtypes = [C.c_void_p, C.c_void_p, C.c_void_p]
        L.orc_replay.argtypes = [C.c_void_p, C.c_void_p, C.c_void_p]
        L.orc_score_epoch.argtypes = ([C.c_void_p] + [C.c_int32] * 4 + [C.c_int64] * 2 +
                                      [C.c_void_p] * 8 + [C.c_int32] * 2 + [C.c_void_p] * 8 +
                                      [C.c_double, C.c_double, C.c_void_p])
        L.orc_form_dispatch.argtypes = ([C.c_void_p, C.c_int32, C.c_int32, C.c_int64, C.c_int64] + [C.c_void_p] * 3 +
                                       [C.c_int32, C.c_int32] + [C.c_void_p] * 10 + [C.c_int64])
        L.orc_sweep.argtypes = ([C.c_void_p] + [C.c_int32] * 4 + [C.c_void_p] * 8 + [C.c_int32] * 2 +
                                [C.c_void_p] * 4)
        L.orc_sweep_depths.argtypes = ([C.c_void_p] + [C.c_int32] * 3 + [C.c_void_p] * 8 + [C.c_int32] * 2 +
                                       [C.c_void_p] * 4)
        _lib = L
    return _lib


class OTables:
    """Keeps the numpy buffers alive while the C struct points at them."""

    def __init__(self, prof):
        self.arrs = [np.ascontiguousarray(x, np.int32) for x in
                     (prof.solo_us, prof.fbr_ppm, prof.mem_mib, prof.batch_size, prof.slo_us, prof.timeout_us)]
        self.geoms = None if prof.geoms is None else np.ascontiguousarray(prof.geoms, np.uint8)
        self.s = Tables(int(self.arrs[0].shape[0]), *[a.ctypes.data for a in self.arrs],
                        int(prof.geometry_set), 0 if self.geoms is None else int(self.geoms.shape[0]),
                        _p(self.geoms), int(getattr(prof, "gpu_mem_mib", 0)))

    @property
    def ref(self):
        return C.byref(self.s)


def enumerate_geometries(set_: int):
    n = C.c_int32()
    out = np.zeros((64, 8), np.uint8)
    stats = np.zeros(4, np.int32)
    rc = lib().orc_enumerate(set_, C.byref(n), _p(out), _p(stats))
    if rc:
        raise OracleError(rc)
    return out[: n.value].copy(), dict(zip(["feasible", "maximal_placements",
                                            "placement_maximal_multisets", "multiset_maximal"],
                                           stats.tolist()))


def table_geometries(prof):
    t = OTables(prof)
    n = C.c_int32()
    out = np.zeros((256, 8), np.uint8)
    rc = lib().orc_table_geometries(t.ref, C.byref(n), _p(out))
    if rc:
        raise OracleError(rc)
    return out[: n.value].copy()


def exec_us(solo, F):
    return lib().orc_exec_us(int(solo), int(F))


def bucket(x):
    return lib().orc_bucket(int(x))


def bucket_lower(b):
    return lib().orc_bucket_lower(int(b))


def percentile(hist, q):
    h = np.ascontiguousarray(hist, np.uint32)
    return lib().orc_percentile(_p(h), int(q))


def vm_draw(seed, replica, node, k, d):
    return lib().orc_vm_draw(seed, replica, node, k, d)


def key(misses, tail, tag):
    return lib().orc_key(int(misses), int(tail), int(tag))


def num_epochs(prof, trace_len, W):
    t = OTables(prof)
    v = lib().orc_num_epochs(t.ref, int(trace_len), int(W))
    if v < 0:
        raise OracleError(v)
    return v


def new_state(geom: int, residents=(), last_start=None, has_vm=1, target=-1, recfg_start=0, recfg_end=0):
    s = State()
    s.geom = geom
    s.target = target
    s.has_vm = has_vm
    s.recfg_start = recfg_start
    s.recfg_end = recfg_end
    for i, r in enumerate(residents):
        s.res[i] = Res(*r)
    s.n_res = len(residents)
    if last_start is not None:
        for i, v in enumerate(last_start):
            s.last_start[i] = v
    return s


def place(prof, state: State, t, model, strict, max_live=64, H=1 << 62):
    T = OTables(prof)
    sl, st, en, dr = C.c_int32(), C.c_int64(), C.c_int64(), C.c_int32()
    s_start = np.zeros(7, np.int64)
    s_end = np.zeros(7, np.int64)
    feas = np.zeros(7, np.int32)
    elig = np.zeros(7, np.int32)
    acc = np.zeros(2, np.int64)
    rc = lib().orc_place(T.ref, C.byref(state), int(t), int(model), int(strict), int(max_live), int(H),
                         C.byref(sl), C.byref(st), C.byref(en), C.byref(dr), _p(s_start), _p(s_end),
                         _p(feas), _p(elig), _p(acc))
    if rc:
        raise OracleError(rc)
    return dict(slice=sl.value, start=st.value, end=en.value, dropped=dr.value, s_start=s_start,
                s_end=s_end, feasible=feas.astype(bool), eligible=elig.astype(bool), accum=acc)


def form_batches(prof, arrival, meta):
    T = OTables(prof)
    a = np.ascontiguousarray(arrival, np.uint32)
    m = np.ascontiguousarray(meta, np.uint8)
    cap = max(1, a.shape[0])
    ready = np.zeros(cap, np.uint32)
    n = np.zeros(cap, np.int32)
    model = np.zeros(cap, np.int32)
    strict = np.zeros(cap, np.int32)
    first = np.zeros(cap, np.int64)
    nb = lib().orc_form_batches(T.ref, _p(a), _p(m), a.shape[0], _p(ready), _p(n), _p(model),
                                _p(strict), _p(first), cap)
    if nb < 0:
        raise OracleError(nb)
    return dict(ready=ready[:nb], n=n[:nb], model=model[:nb], strict=strict[:nb], first_raw=first[:nb])


def tick_simulate(prof, geom, t, model, slice_):
    T = OTables(prof)
    t = np.ascontiguousarray(t, np.int64)
    model = np.ascontiguousarray(model, np.int32)
    slice_ = np.ascontiguousarray(slice_, np.int32)
    start = np.zeros(t.shape[0], np.int64)
    end = np.zeros(t.shape[0], np.int64)
    rc = lib().orc_tick_simulate(T.ref, int(geom), int(t.shape[0]), _p(t), _p(model), _p(slice_),
                                 _p(start), _p(end))
    if rc:
        raise OracleError(rc)
    return start, end


DEFAULT_CFG = dict(N=8, W=1_000_000, policy=0, wait_limit=3, cap_pct=30, init_geom=2, max_live=64,
                   vm_policy=0, reconfig_us=2_000_000, p_rev=0.0, price_od=32.7726 / 8,
                   price_spot=9.8318 / 8, rev_interval=300_000_000, notice=30_000_000, seed=0,
                   shard_mode=0, ewma_alpha_pm=500, t_low=500, t_high=4000, cold_us=0, keepalive_epochs=600,
                   prewarm=0)


def replay(prof, trace, *, nthreads=1, want_keys=False, want_log=False, log_cap=None, **cfg):
    c = dict(DEFAULT_CFG)
    c.update(cfg)
    T = OTables(prof)
    R = trace.n_replicas
    N = c["N"]
    arr = np.ascontiguousarray(trace.arrival_us, np.uint32)
    meta = np.ascontiguousarray(trace.meta, np.uint8)
    off = np.ascontiguousarray(trace.replica_off, np.int64)
    rin = ReplayIn(R, N, int(trace.replica_base), int(trace.trace_len_us), int(c["W"]), _p(arr) or 0,
                   _p(meta) or 0, _p(off), c["policy"], c["wait_limit"], c["cap_pct"], c["init_geom"],
                   c["max_live"], c["vm_policy"], c["reconfig_us"], c["p_rev"], c["price_od"],
                   c["price_spot"], c["rev_interval"], c["notice"], c["seed"], c["shard_mode"], nthreads,
                   c["ewma_alpha_pm"], 0, c["t_low"], c["t_high"], c["cold_us"], c["keepalive_epochs"],
                   c["prewarm"])
    if arr.shape[0] == 0:  # keep pointers non-NULL for empty traces
        arr = np.zeros(1, np.uint32)
        meta = np.zeros(1, np.uint8)
        rin.arrival, rin.meta = arr.ctypes.data, meta.ctypes.data
    G = table_geometries(prof).shape[0] if want_keys else 0
    E = num_epochs(prof, trace.trace_len_us, c["W"])
    out = dict(counters=np.zeros((R, 10), np.int64), accum=np.zeros((R, 4), np.int64),
               hist=np.zeros((R, 2, NB), np.uint32), p50_p99=np.zeros((R, 2, 2), np.int64),
               cost=np.zeros(R, np.float64), util=np.zeros((R, 2), np.float64),
               decisions=np.zeros((R, E, N), np.uint8), n_batches=np.zeros(R, np.int64),
               cold_starts=np.zeros(R, np.int64), stats=np.zeros((R, 4), np.int64))
    if want_keys:
        out["cand_keys"] = np.zeros((R, E, N, G), np.int64)
    if want_log:
        if log_cap is None:
            log_cap = max(1, int(np.max(np.diff(off))) if R else 1)
        out["log"] = np.zeros((R, log_cap), BATCH_REC_DTYPE)
    ro = ReplayOut(_p(out["counters"]), _p(out["accum"]), _p(out["hist"]), _p(out["p50_p99"]),
                   _p(out["cost"]), _p(out["util"]), _p(out["decisions"]), _p(out.get("cand_keys")),
                   _p(out.get("log")), int(log_cap or 0), _p(out["n_batches"]), _p(out["cold_starts"]),
                   _p(out["stats"]))
    rc = lib().orc_replay(T.ref, C.byref(rin), C.byref(ro))
    if rc:
        raise OracleError(rc)
    out["E"] = E
    return out


def score_epoch(prof, *, R, N, epoch, batches, batch_off, arrival, states, geom_lo=0, geom_hi=None,
                W=1_000_000, H=1 << 62, max_live=64, price_od=32.7726 / 8, price_spot=9.8318 / 8):
    """batches: dict of arrays ready, req_off, n, model, strict (ordered by (replica, gpu, id));
    states: ctypes array of State (modified in place)."""
    T = OTables(prof)
    G = table_geometries(prof).shape[0]
    if geom_hi is None:
        geom_hi = G
    nb = len(batches["ready"])
    arrs = {k: np.ascontiguousarray(batches[k], np.uint32 if k in ("ready", "req_off") else np.int32)
            for k in ("ready", "req_off", "n", "model", "strict")}
    boff = np.ascontiguousarray(batch_off, np.int32)
    arrival = np.ascontiguousarray(arrival, np.uint32)
    if arrival.shape[0] == 0:
        arrival = np.zeros(1, np.uint32)
    nc = geom_hi - geom_lo
    out = dict(best_key=np.zeros(R * N, np.int64), cand_key=np.zeros(R * N * max(nc, 0), np.int64),
               start=np.zeros(max(nb, 1), np.int64), end=np.zeros(max(nb, 1), np.int64),
               slice=np.zeros(max(nb, 1), np.int32), dropped=np.zeros(max(nb, 1), np.int32),
               counters=np.zeros((R, 10), np.int64), accum=np.zeros((R, 4), np.int64),
               cost=np.zeros(R * N, np.float64))
    rc = lib().orc_score_epoch(T.ref, R, N, epoch, max_live, C.c_int64(W), C.c_int64(H), _p(arrs["ready"]), _p(arrs["req_off"]),
                               _p(arrs["n"]), _p(arrs["model"]), _p(arrs["strict"]), _p(boff),
                               _p(arrival), C.addressof(states), geom_lo, geom_hi, _p(out["best_key"]),
                               _p(out["cand_key"]), _p(out["start"]), _p(out["end"]), _p(out["slice"]),
                               _p(out["dropped"]), _p(out["counters"]), _p(out["accum"]),
                               C.c_double(price_od), C.c_double(price_spot), _p(out["cost"]))
    if rc:
        raise OracleError(rc)
    for k in ("start", "end", "slice", "dropped"):
        out[k] = out[k][:nb]
    return out


def sweep(prof, *, R, N, batches, batch_off, arrival, cur_geom, geom_lo=0, geom_hi=None, max_live=64,
          max_batches=8):
    """N4a exhaustive assignment sweep (orc_sweep); batches as for score_epoch."""
    T = OTables(prof)
    G = table_geometries(prof).shape[0]
    if geom_hi is None:
        geom_hi = G
    arrs = {k: np.ascontiguousarray(batches[k], np.uint32 if k in ("ready", "req_off") else np.int32)
            for k in ("ready", "req_off", "n", "model", "strict")}
    for k in arrs:
        if arrs[k].shape[0] == 0:
            arrs[k] = np.zeros(1, arrs[k].dtype)
    boff = np.ascontiguousarray(batch_off, np.int32)
    arrival = np.ascontiguousarray(arrival, np.uint32)
    if arrival.shape[0] == 0:
        arrival = np.zeros(1, np.uint32)
    cg = np.ascontiguousarray(cur_geom, np.uint8)
    nc = geom_hi - geom_lo
    out = dict(sweep_key=np.zeros(R * N * max(nc, 0), np.int64), assign=np.zeros(R * N * max(nc, 0), np.uint32),
               best_key=np.zeros(R * N, np.int64), n_assign=np.zeros(1, np.int64))
    rc = lib().orc_sweep(T.ref, R, N, max_live, max_batches, _p(arrs["ready"]), _p(arrs["req_off"]),
                         _p(arrs["n"]), _p(arrs["model"]), _p(arrs["strict"]), _p(boff), _p(arrival),
                         _p(cg), geom_lo, geom_hi, _p(out["sweep_key"]), _p(out["assign"]),
                         _p(out["best_key"]), _p(out["n_assign"]))
    if rc:
        raise OracleError(rc)
    out["n_assign"] = int(out["n_assign"][0])
    return out


def sweep_depths(prof, *, R, N, batches, batch_off, arrival, cur_geom, geom_lo=0, geom_hi=None, max_live=64):
    """N4b BE-reserve depth sweep (orc_sweep_depths); batches as for score_epoch.  depth_key is
    [R*N, nc, 8]: code 0 = Alg 1's tag walk, 1 + d = reserve depth d (-1 beyond the slice count)."""
    T = OTables(prof)
    G = table_geometries(prof).shape[0]
    if geom_hi is None:
        geom_hi = G
    arrs = {k: np.ascontiguousarray(batches[k], np.uint32 if k in ("ready", "req_off") else np.int32)
            for k in ("ready", "req_off", "n", "model", "strict")}
    for k in arrs:
        if arrs[k].shape[0] == 0:
            arrs[k] = np.zeros(1, arrs[k].dtype)
    boff = np.ascontiguousarray(batch_off, np.int32)
    arrival = np.ascontiguousarray(arrival, np.uint32)
    if arrival.shape[0] == 0:
        arrival = np.zeros(1, np.uint32)
    cg = np.ascontiguousarray(cur_geom, np.uint8)
    nc = geom_hi - geom_lo
    out = dict(depth_key=np.zeros((R * N, max(nc, 0), 8), np.int64), depth_code=np.zeros((R * N, max(nc, 0)), np.uint8),
               best_key=np.zeros(R * N, np.int64), n_eval=np.zeros(1, np.int64))
    rc = lib().orc_sweep_depths(T.ref, R, N, max_live, _p(arrs["ready"]), _p(arrs["req_off"]), _p(arrs["n"]),
                                _p(arrs["model"]), _p(arrs["strict"]), _p(boff), _p(arrival), _p(cg), geom_lo,
                                geom_hi, _p(out["depth_key"]), _p(out["depth_code"]), _p(out["best_key"]),
                                _p(out["n_eval"]))
    if rc:
        raise OracleError(rc)
    out["n_eval"] = int(out["n_eval"][0])
    return out


def form_dispatch(prof, trace, *, N, e_lo, e_hi, avail=None, W=1_000_000):
    """O3 + O5.2 for epochs [e_lo, e_hi) (orc_form_dispatch); rows as a dict of arrays."""
    T = OTables(prof)
    R = trace.n_replicas
    arr = np.ascontiguousarray(trace.arrival_us, np.uint32)
    meta = np.ascontiguousarray(trace.meta, np.uint8)
    off = np.ascontiguousarray(trace.replica_off, np.int64)
    if arr.shape[0] == 0:
        arr, meta = np.zeros(1, np.uint32), np.zeros(1, np.uint8)
    cap = max(1, int(arr.shape[0]))
    out = dict(ready=np.zeros(cap, np.uint32), req_off=np.zeros(cap, np.uint32), n=np.zeros(cap, np.int32),
               model=np.zeros(cap, np.int32), strict=np.zeros(cap, np.int32), gpu=np.zeros(cap, np.int32))
    boff = np.zeros(R * (e_hi - e_lo) * N + 1, np.int32)
    members = np.zeros(cap, np.uint32)
    nrows = np.array([cap], np.int64)
    av = None if avail is None else np.ascontiguousarray(avail, np.int64)
    rc = lib().orc_form_dispatch(T.ref, R, N, W, int(trace.trace_len_us), _p(arr), _p(meta), _p(off), e_lo, e_hi,
                                _p(av), _p(out["ready"]), _p(out["req_off"]), _p(out["n"]), _p(out["model"]),
                                _p(out["strict"]), _p(out["gpu"]), _p(boff), _p(nrows), _p(members), cap)
    if rc:
        raise OracleError(rc)
    k = int(nrows[0])
    res = {kk: v[:k] for kk, v in out.items()}
    res["batch_off"] = boff
    res["members"] = members
    return res
