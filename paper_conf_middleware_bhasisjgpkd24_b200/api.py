"""Thin Python binding of the C ABI (same names as include/protean.h).

torch is used for device memory and streams only; every computation runs in libprotean.so.
"""
from __future__ import annotations

import ctypes as C

import numpy as np

from . import _abi as A

_REPLAY_DEFAULTS = dict(n_gpus=8, epoch_len_us=1_000_000, policy=0, wait_limit=3, reconfig_cap_pct=30,
                        init_geom=2, max_live=64, vm_policy=0, reconfig_us=2_000_000, p_rev=0.0,
                        price_od_node_hr=32.7726 / 8, price_spot_node_hr=9.8318 / 8,
                        rev_interval_us=300_000_000, notice_us=30_000_000, seed=0, shard_mode=0,
                        rank=0, nranks=1, max_ctas=0, replica_base=0, ewma_alpha_pm=500, t_low_milli=500,
                        t_high_milli=4000, cold_start_us=0, keepalive_epochs=600, prewarm=0,
                        ctas_per_replica=0)


def _torch():
    import torch
    if not torch.cuda.is_available():
        raise RuntimeError("paper_conf_middleware_bhasisjgpkd24_b200 needs a CUDA device (no CPU fallback)")
    return torch


def _check(h, rc):
    if rc != A.OK:
        detail = A.load().protean_last_error(h).decode() if h else ""
        raise A.ProteanError(rc, detail)


def _profiles_struct(profiles, device: int = 0):
    """protean_profiles for `profiles` (+ the numpy arrays it points into, to keep alive)."""
    arrs = [np.ascontiguousarray(x, np.int32) for x in
            (profiles.solo_us, profiles.fbr_ppm, profiles.mem_mib, profiles.batch_size,
             profiles.slo_us, profiles.timeout_us)]
    geoms = None if profiles.geoms is None else np.ascontiguousarray(profiles.geoms, np.uint8)
    p = A.Profiles(A.ABI_VERSION, int(arrs[0].shape[0]), *[a.ctypes.data for a in arrs],
                   int(profiles.geometry_set), 0 if geoms is None else int(geoms.shape[0]),
                   None if geoms is None else geoms.ctypes.data, int(device),
                   int(getattr(profiles, "gpu_mem_mib", 0)))
    return p, (arrs, geoms)


def geometry_split(profiles, nranks: int) -> list[int]:
    """protean_geometry_split: slot-balanced geometry range bounds [nranks + 1] (host only)."""
    lib = A.load(require_cuda=False)
    p, keep = _profiles_struct(profiles)
    b = (C.c_int32 * (nranks + 1))()
    rc = lib.protean_geometry_split(C.byref(p), int(nranks), b)
    if rc != A.OK:
        raise A.ProteanError(rc, "protean_geometry_split")
    del keep
    return list(b)


class Handle:
    """protean_load_profiles(): validated tables + geometry set resident on `device`."""

    def __init__(self, profiles, device: int = 0):
        self._lib = A.load()
        self.device = device
        p, keep = _profiles_struct(profiles, device)
        self._h = C.c_void_p()
        rc = self._lib.protean_load_profiles(C.byref(p), C.byref(self._h))
        if rc != A.OK:
            raise A.ProteanError(rc, "protean_load_profiles")
        del keep
        n = C.c_int32()
        self._lib.protean_get_geometries(self._h, C.byref(n), None)
        self.n_geoms = n.value

    # ------------------------------------------------------------------ mode G exchange set-up
    def xchg_export(self, nranks: int, rank: int, max_replicas: int, max_gpus: int) -> bytes:
        """protean_xchg_export: allocate this rank's exchange buffer; returns its IPC handle."""
        buf = (C.c_char * A.IPC_HANDLE_BYTES)()
        _check(self._h, self._lib.protean_xchg_export(self._h, int(nranks), int(rank), int(max_replicas),
                                                      int(max_gpus), buf))
        return bytes(buf)

    def xchg_import(self, handles: list[bytes]):
        """protean_xchg_import: map every rank's buffer (handles in rank order)."""
        blob = b"".join(handles)
        assert len(blob) == A.IPC_HANDLE_BYTES * len(handles)
        buf = (C.c_char * len(blob)).from_buffer_copy(blob)
        _check(self._h, self._lib.protean_xchg_import(self._h, buf))

    @staticmethod
    def xchg_attach(handles: list["Handle"], max_replicas: int, max_gpus: int):
        """protean_xchg_attach: every rank in this process, handles[k] = rank k."""
        lib = A.load()
        arr = (C.c_void_p * len(handles))(*[h._h.value for h in handles])
        rc = lib.protean_xchg_attach(arr, len(handles), int(max_replicas), int(max_gpus))
        if rc != A.OK:
            raise A.ProteanError(rc, "protean_xchg_attach: "
                                 + " | ".join(lib.protean_last_error(h._h).decode() for h in handles))

    def close(self):
        if getattr(self, "_h", None):
            self._lib.protean_free(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def geometries(self) -> np.ndarray:
        n = C.c_int32()
        out = np.zeros((self.n_geoms, 8), np.uint8)
        _check(self._h, self._lib.protean_get_geometries(self._h, C.byref(n), out.ctypes.data))
        return out

    def num_epochs(self, trace_len_us: int, epoch_len_us: int = 1_000_000) -> int:
        E = C.c_int64()
        _check(self._h, self._lib.protean_num_epochs(self._h, int(trace_len_us), int(epoch_len_us), C.byref(E)))
        return E.value

    def last_timings(self):
        """(prepass_ms, replay_kernel_ms, {grid, block, smem, per_sm}) of the last replay call."""
        a, b = C.c_float(), C.c_float()
        launch = (C.c_int32 * 4)()
        _check(self._h, self._lib.protean_last_timings(self._h, C.byref(a), C.byref(b), launch))
        return a.value, b.value, dict(zip(("grid", "block", "smem", "per_sm"), list(launch)))

    def last_search_ms(self):
        """(search_ms, walk_ms, acct_ms): device time of the candidate search (cand.cu) the last
        replay ran ahead of its chain, of its cursor pass alone, and of the accounting pass after
        the lean chain (chain.cu; 0 when the fused engine ran)."""
        a, b, d = C.c_float(), C.c_float(), C.c_float()
        if not hasattr(self._lib, "protean_last_search_ms"):
            return 0.0, 0.0, 0.0
        _check(self._h, self._lib.protean_last_search_ms(self._h, C.byref(a), C.byref(b), C.byref(d)))
        return a.value, b.value, d.value

    # -------------------------------------------------------------------------------- replay
    def alloc_replay_out(self, R: int, E: int, N: int, *, decisions=True, cand_keys=False, log_cap=0):
        torch = _torch()
        dev = torch.device("cuda", self.device)
        out = dict(counters=torch.zeros((R, 10), dtype=torch.int64, device=dev),
                   accum=torch.zeros((R, 4), dtype=torch.int64, device=dev),
                   hist=torch.zeros((R, 2, A.NBUCKETS), dtype=torch.int32, device=dev),
                   p50_p99=torch.zeros((R, 2, 2), dtype=torch.int64, device=dev),
                   cost=torch.zeros(R, dtype=torch.float64, device=dev),
                   util=torch.zeros((R, 2), dtype=torch.float64, device=dev),
                   n_batches=torch.zeros(R, dtype=torch.int64, device=dev),
                   cold_starts=torch.zeros(R, dtype=torch.int64, device=dev))
        if decisions:
            out["decisions"] = torch.zeros((R, E, N), dtype=torch.uint8, device=dev)
        if cand_keys:
            out["cand_keys"] = torch.zeros((R, E, N, self.n_geoms), dtype=torch.int64, device=dev)
        if log_cap:
            out["log"] = torch.zeros((R, log_cap, C.sizeof(A.BatchRec)), dtype=torch.uint8, device=dev)
        out["log_cap"] = int(log_cap)
        return out

    def _cfg(self, R: int, trace_len_us: int, c: dict, arrival_ptr: int, meta_ptr: int, off_ptr: int):
        cf = A.ReplayCfg()
        self._lib.protean_replay_cfg_defaults(C.byref(cf))
        cf.n_replicas, cf.n_gpus = R, int(c["n_gpus"])
        cf.replica_base = int(c["replica_base"])
        cf.trace_len_us = int(trace_len_us)
        cf.epoch_len_us = int(c["epoch_len_us"])
        cf.arrival_us, cf.meta, cf.replica_off = arrival_ptr, meta_ptr, off_ptr
        for k in ("policy", "wait_limit", "reconfig_cap_pct", "init_geom", "max_live", "vm_policy",
                  "reconfig_us", "rev_interval_us", "notice_us", "seed", "shard_mode", "rank", "nranks",
                  "max_ctas", "ewma_alpha_pm", "t_low_milli", "t_high_milli", "cold_start_us",
                  "keepalive_epochs", "prewarm", "ctas_per_replica"):
            setattr(cf, k, int(c[k]))
        for k in ("p_rev", "price_od_node_hr", "price_spot_node_hr"):
            setattr(cf, k, float(c[k]))
        return cf

    @staticmethod
    def _check_out(out: dict, R: int, E: int, N: int, G: int, device=None):
        """The C ABI cannot check caller buffer sizes: assert every output's shape (and device)."""
        want = dict(counters=(R, 10), accum=(R, 4), hist=(R, 2, A.NBUCKETS), p50_p99=(R, 2, 2), cost=(R,),
                    util=(R, 2), n_batches=(R,), cold_starts=(R,), decisions=(R, E, N), cand_keys=(R, E, N, G))
        for k, shp in want.items():
            if k not in out:
                continue
            t = out[k]
            assert tuple(t.shape) == shp, f"out[{k!r}] has shape {tuple(t.shape)}, expected {shp}"
            assert t.is_contiguous(), f"out[{k!r}] is not contiguous"
            if device is not None:
                assert t.is_cuda and t.device.index == device, f"out[{k!r}] is not on cuda:{device}"
            else:
                assert not t.is_cuda, f"out[{k!r}] must be a host tensor"
        if "log" in out:
            assert out["log"].shape[0] == R and out["log"].shape[1] >= out.get("log_cap", 0)

    def _out_struct(self, out: dict):
        return A.ReplayOut(out["counters"].data_ptr(), out["accum"].data_ptr(), out["hist"].data_ptr(),
                           out["p50_p99"].data_ptr(), out["cost"].data_ptr(), out["util"].data_ptr(),
                           out["decisions"].data_ptr() if "decisions" in out else None,
                           out["cand_keys"].data_ptr() if "cand_keys" in out else None,
                           out["log"].data_ptr() if "log" in out else None, out.get("log_cap", 0),
                           out["n_batches"].data_ptr() if "n_batches" in out else None,
                           out["cold_starts"].data_ptr() if "cold_starts" in out else None)

    def replay_traces(self, arrival_us, meta, replica_off, *, trace_len_us: int, out=None,
                      want_decisions=True, want_cand_keys=False, log_cap=0, stream=None, **cfg):
        """protean_replay_traces on device tensors (arrival uint32/int32, meta uint8, off int64)."""
        torch = _torch()
        c = dict(_REPLAY_DEFAULTS)
        c.update(cfg)
        R = int(replica_off.shape[0]) - 1
        N = int(c["n_gpus"])
        E = self.num_epochs(trace_len_us, c["epoch_len_us"])
        if out is None:
            out = self.alloc_replay_out(R, E, N, decisions=want_decisions, cand_keys=want_cand_keys,
                                        log_cap=log_cap)
        self._check_out(out, R, E, N, self.n_geoms, device=self.device)
        assert arrival_us.element_size() == 4 and meta.element_size() == 1 and replica_off.element_size() == 8
        for t in (arrival_us, meta, replica_off):
            assert t.is_cuda and t.is_contiguous() and t.device.index == self.device
        cf = self._cfg(R, trace_len_us, c, arrival_us.data_ptr() if arrival_us.numel() else replica_off.data_ptr(),
                       meta.data_ptr() if meta.numel() else replica_off.data_ptr(), replica_off.data_ptr())
        o = self._out_struct(out)
        st = stream if stream is not None else torch.cuda.current_stream(self.device)
        _check(self._h, self._lib.protean_replay_traces(self._h, C.byref(cf), C.byref(o),
                                                        C.c_void_p(st.cuda_stream)))
        out["E"] = E
        return out

    def replay_traces_host(self, trace, *, pinned=None, stream=None, **cfg):
        """A Trace (numpy) through the device call: H2D of the trace, the replay, D2H of results.
        (Test convenience; the C-ABI host-buffer entry point is replay_traces_pinned.)"""
        torch = _torch()
        dev = torch.device("cuda", self.device)
        arr = torch.from_numpy(np.ascontiguousarray(trace.arrival_us).view(np.int32))
        meta = torch.from_numpy(np.ascontiguousarray(trace.meta))
        off = torch.from_numpy(np.ascontiguousarray(trace.replica_off, np.int64))
        if pinned is not None:
            arr, meta, off = pinned
        d = [x.to(dev, non_blocking=True) for x in (arr, meta, off)]
        cfg.setdefault("replica_base", trace.replica_base)
        out = self.replay_traces(d[0], d[1], d[2], trace_len_us=trace.trace_len_us, stream=stream, **cfg)
        return {k: (v.cpu().numpy() if hasattr(v, "cpu") else v) for k, v in out.items()}

    def alloc_host_out(self, R: int, E: int, N: int, *, decisions=True):
        """Page-locked host output tensors for replay_traces_pinned."""
        torch = _torch()
        d = self.alloc_replay_out(1, 1, 1, decisions=False)
        out = {k: torch.empty((R,) + tuple(v.shape[1:]), dtype=v.dtype).pin_memory() for k, v in d.items()
               if hasattr(v, "shape")}
        if decisions:
            out["decisions"] = torch.empty((R, E, N), dtype=torch.uint8).pin_memory()
        return out

    def replay_traces_pinned(self, arrival_h, meta_h, off_h, *, trace_len_us: int, chunks: int = 4,
                             out_host=None, stream=None, **cfg):
        """protean_replay_traces_host (include/protean.h 3c): the end-to-end call on HOST tensors
        (arrival int32/uint32 [n], meta uint8 [n], off int64 [R+1]; page-locked for overlap).  The
        library cuts the replicas into `chunks` ranges and overlaps chunk k+1's H2D and chunk k-1's
        D2H with chunk k's replay.  Returns the host output tensors (out_host, allocated pinned if
        None)."""
        torch = _torch()
        c = dict(_REPLAY_DEFAULTS)
        c.update(cfg)
        R = int(off_h.shape[0]) - 1
        N = int(c["n_gpus"])
        E = self.num_epochs(trace_len_us, c["epoch_len_us"])
        for t in (arrival_h, meta_h, off_h):
            assert not t.is_cuda and t.is_contiguous()
        assert arrival_h.element_size() == 4 and meta_h.element_size() == 1 and off_h.element_size() == 8
        if out_host is None:
            out_host = self.alloc_host_out(R, E, N)
        self._check_out(out_host, R, E, N, self.n_geoms, device=None)
        assert "cand_keys" not in out_host and "log" not in out_host
        cf = self._cfg(R, trace_len_us, c, arrival_h.data_ptr() if arrival_h.numel() else off_h.data_ptr(),
                       meta_h.data_ptr() if meta_h.numel() else off_h.data_ptr(), off_h.data_ptr())
        o = self._out_struct(out_host)
        st = stream if stream is not None else torch.cuda.current_stream(self.device)
        _check(self._h, self._lib.protean_replay_traces_host(self._h, C.byref(cf), C.byref(o), int(chunks),
                                                             C.c_void_p(st.cuda_stream)))
        return out_host

    # -------------------------------------------------------------------------------- score_epoch
    def score_epoch(self, *, n_replicas, n_gpus, epoch, batches, batch_off, arrival_us, state,
                    geom_lo=0, geom_hi=None, epoch_len_us=1_000_000, horizon_us=1 << 62, max_live=64,
                    counters=None, accum=None, want_cand_keys=True, price_od_node_hr=32.7726 / 8,
                    price_spot_node_hr=9.8318 / 8, stream=None, sync=True):
        """protean_score_epoch.  batches: uint8 device tensor of protean_batch rows (16 B each);
        state: uint8 device tensor of protean_gpu_state rows (modified in place).  The C call only
        enqueues; with sync=True (default) the stream is synchronised and
        protean_score_epoch_status raises the kernel's validation verdict, if any."""
        torch = _torch()
        dev = torch.device("cuda", self.device)
        geom_hi = self.n_geoms if geom_hi is None else geom_hi
        R, N = int(n_replicas), int(n_gpus)
        nb = batches.numel() // 16
        nc = geom_hi - geom_lo
        out = dict(best_key=torch.zeros(R * N, dtype=torch.int64, device=dev),
                   placement=torch.zeros((max(nb, 1), 24), dtype=torch.uint8, device=dev),
                   counters=counters if counters is not None else torch.zeros((R, 10), dtype=torch.int64, device=dev),
                   accum=accum if accum is not None else torch.zeros((R, 4), dtype=torch.int64, device=dev),
                   cost=torch.zeros(R * N, dtype=torch.float64, device=dev))
        if want_cand_keys:
            out["cand_key"] = torch.zeros(R * N * max(nc, 1), dtype=torch.int64, device=dev)
        ei = A.EpochIn(R, N, int(epoch), int(max_live), int(epoch_len_us), int(horizon_us),
                       batches.data_ptr() if nb else out["placement"].data_ptr(), batch_off.data_ptr(),
                       arrival_us.data_ptr() if arrival_us.numel() else batch_off.data_ptr(),
                       state.data_ptr(), int(geom_lo), int(geom_hi), float(price_od_node_hr),
                       float(price_spot_node_hr))
        eo = A.EpochOut(out["best_key"].data_ptr(), out["cand_key"].data_ptr() if want_cand_keys else None,
                        out["placement"].data_ptr(), out["counters"].data_ptr(), out["accum"].data_ptr(),
                        out["cost"].data_ptr())
        st = stream if stream is not None else torch.cuda.current_stream(self.device)
        _check(self._h, self._lib.protean_score_epoch(self._h, C.byref(ei), C.byref(eo),
                                                      C.c_void_p(st.cuda_stream)))
        if sync:
            st.synchronize()
            self.score_epoch_status()
        out["placement"] = out["placement"][:nb]
        return out

    def score_epoch_status(self):
        """protean_score_epoch_status: raise the latched verdict of enqueued score_epoch calls."""
        _check(self._h, self._lib.protean_score_epoch_status(self._h))

    def form_batches(self, arrival_us, meta, replica_off, *, trace_len_us: int, n_gpus: int, e_lo: int,
                     e_hi: int, avail=None, epoch_len_us: int = 1_000_000, stream=None):
        """protean_form_batches on device tensors: rows (uint8 [n, 16] protean_batch), batch_off
        (int32 CSR over (replica, epoch - e_lo, gpu)) and members (uint32 as int32)."""
        torch = _torch()
        dev = torch.device("cuda", self.device)
        R = int(replica_off.shape[0]) - 1
        cf = A.ReplayCfg()
        self._lib.protean_replay_cfg_defaults(C.byref(cf))
        cf.n_replicas, cf.n_gpus = R, int(n_gpus)
        cf.trace_len_us, cf.epoch_len_us = int(trace_len_us), int(epoch_len_us)
        cf.arrival_us = arrival_us.data_ptr() if arrival_us.numel() else replica_off.data_ptr()
        cf.meta = meta.data_ptr() if meta.numel() else replica_off.data_ptr()
        cf.replica_off = replica_off.data_ptr()
        n_req = int(arrival_us.numel())
        mcap = n_req + 4 * R
        members = torch.zeros(max(mcap, 1), dtype=torch.int32, device=dev)
        boff = torch.zeros(R * (e_hi - e_lo) * int(n_gpus) + 1, dtype=torch.int32, device=dev)
        st = stream if stream is not None else torch.cuda.current_stream(self.device)
        cap = C.c_int64(0)  # first call sizes the rows
        rc = self._lib.protean_form_batches(self._h, C.byref(cf), int(e_lo), int(e_hi),
                                            avail.data_ptr() if avail is not None else None, None,
                                            boff.data_ptr(), C.byref(cap), members.data_ptr(), mcap,
                                            C.c_void_p(st.cuda_stream))
        if rc not in (A.OK, A.ERANGE) or (rc == A.ERANGE and cap.value == 0):
            _check(self._h, rc)
        rows = torch.zeros((max(cap.value, 1), 16), dtype=torch.uint8, device=dev)
        _check(self._h, self._lib.protean_form_batches(self._h, C.byref(cf), int(e_lo), int(e_hi),
                                                       avail.data_ptr() if avail is not None else None,
                                                       rows.data_ptr(), boff.data_ptr(), C.byref(cap),
                                                       members.data_ptr(), mcap, C.c_void_p(st.cuda_stream)))
        return dict(rows=rows[: cap.value], batch_off=boff, members=members, n=cap.value)

    def sweep_assignments(self, *, n_replicas, n_gpus, batches, batch_off, arrival_us, cur_geom,
                          geom_lo=0, geom_hi=None, max_live=64, max_batches=8, want_sweep_keys=True,
                          out=None, stream=None):
        """protean_sweep_assignments (N4a).  batches: uint8 device tensor of protean_batch rows
        (16 B each); batch_off int32 [R*N+1]; arrival_us uint32/int32; cur_geom uint8 [R*N]."""
        torch = _torch()
        dev = torch.device("cuda", self.device)
        geom_hi = self.n_geoms if geom_hi is None else geom_hi
        R, N = int(n_replicas), int(n_gpus)
        nc = geom_hi - geom_lo
        if out is None:
            out = dict(best_key=torch.zeros(R * N, dtype=torch.int64, device=dev),
                       n_assign=torch.zeros(1, dtype=torch.int64, device=dev))
            if want_sweep_keys:
                out["sweep_key"] = torch.zeros(R * N * max(nc, 1), dtype=torch.int64, device=dev)
                out["assign"] = torch.zeros(R * N * max(nc, 1), dtype=torch.int32, device=dev)
        nb = batches.numel() // 16
        si = A.SweepIn(R, N, int(max_live), int(max_batches),
                       batches.data_ptr() if nb else batch_off.data_ptr(), batch_off.data_ptr(),
                       arrival_us.data_ptr() if arrival_us.numel() else batch_off.data_ptr(),
                       cur_geom.data_ptr(), int(geom_lo), int(geom_hi))
        so = A.SweepOut(out["sweep_key"].data_ptr() if "sweep_key" in out else None,
                        out["assign"].data_ptr() if "assign" in out else None,
                        out["best_key"].data_ptr(), out["n_assign"].data_ptr())
        st = stream if stream is not None else torch.cuda.current_stream(self.device)
        _check(self._h, self._lib.protean_sweep_assignments(self._h, C.byref(si), C.byref(so),
                                                            C.c_void_p(st.cuda_stream)))
        return out

    def sweep_depths(self, *, n_replicas, n_gpus, batches, batch_off, arrival_us, cur_geom, geom_lo=0,
                     geom_hi=None, max_live=64, out=None, stream=None):
        """protean_sweep_depths (N4b, BE-reserve depth codes).  Inputs as sweep_assignments.
        Returns depth_key [R*N, nc, 8], depth_code [R*N, nc] (uint8), best_key [R*N], n_eval [1]."""
        torch = _torch()
        dev = torch.device("cuda", self.device)
        geom_hi = self.n_geoms if geom_hi is None else geom_hi
        R, N = int(n_replicas), int(n_gpus)
        nc = geom_hi - geom_lo
        if out is None:
            out = dict(depth_key=torch.zeros((R * N, max(nc, 1), 8), dtype=torch.int64, device=dev),
                       depth_code=torch.zeros((R * N, max(nc, 1)), dtype=torch.uint8, device=dev),
                       best_key=torch.zeros(R * N, dtype=torch.int64, device=dev),
                       n_eval=torch.zeros(1, dtype=torch.int64, device=dev))
        nb = batches.numel() // 16
        si = A.SweepIn(R, N, int(max_live), 8, batches.data_ptr() if nb else batch_off.data_ptr(),
                       batch_off.data_ptr(), arrival_us.data_ptr() if arrival_us.numel() else batch_off.data_ptr(),
                       cur_geom.data_ptr(), int(geom_lo), int(geom_hi))
        do = A.DepthOut(out["depth_key"].data_ptr(), out["depth_code"].data_ptr(), out["best_key"].data_ptr(),
                        out["n_eval"].data_ptr())
        st = stream if stream is not None else torch.cuda.current_stream(self.device)
        _check(self._h, self._lib.protean_sweep_depths(self._h, C.byref(si), C.byref(do), C.c_void_p(st.cuda_stream)))
        return out


def load_profiles(profiles, device: int = 0) -> Handle:
    return Handle(profiles, device)
