"""Request validation inside the fused replay (count pass) and unaligned trace buffers.  -m gpu.

Every request is checked once per window it appears in: model id < M and no reserved bit, arrival <
trace_len, arrival >= its predecessor (a malformed trace is PROTEAN_EINVAL, no
partial result).  The body of the count pass reads 16 requests per lane with 16-byte loads, so the
faults are planted at positions that cover the unaligned head, the vector body (inside a 16-entry
group, across groups, across lanes) and the tail of several windows.  Unaligned device pointers take
the scalar path and must give the oracle's result bit for bit."""
import numpy as np
import pytest

from gpu_common import compare, gpu_replay, oracle_replay
from protean_inputs import concat, pack_meta, random_profiles
from protean_inputs.traces import Trace

pytestmark = pytest.mark.gpu


def _trace(rng, n=6000, M=4, T=3_000_000):
    a = np.sort(rng.integers(0, T, n)).astype(np.uint32)
    return a, pack_meta(rng.integers(0, M, n), rng.integers(0, 2, n)), T


def _code(prof, tr):
    import paper_conf_middleware_bhasisjgpkd24_b200 as pkg
    try:
        h = pkg.load_profiles(prof)
        h.replay_traces_host(tr, n_gpus=2)
    except pkg.ProteanError as e:
        return e.code
    return 0


@pytest.mark.parametrize("kind", ["unsorted", "model", "reserved_bit", "beyond_trace"])
def test_planted_faults(oracle, kind):
    rng = np.random.default_rng({"unsorted": 1, "model": 2, "reserved_bit": 3, "beyond_trace": 4}[kind])
    prof = random_profiles(rng, 4)
    a0, m0, T = _trace(rng)
    assert _code(prof, concat([(a0, m0)], T)) == 0
    positions = sorted({1, 2, 15, 16, 17, 31, 32, 33, 511, 512, 513, 1999, 2000, 2001, 4095, 4096,
                        len(a0) - 2, len(a0) - 1, *rng.integers(1, len(a0), 8).tolist()})
    for p in positions:
        a, m = a0.copy(), m0.copy()
        if kind == "unsorted":
            if a[p] == 0:
                continue
            a[p] = a[p - 1] - 1 if a[p - 1] > 0 else 0
            if a[p] >= a[p - 1]:
                continue
        elif kind == "model":
            m[p] = (m[p] & 0x80) | 9          # model 9 >= M = 4
        elif kind == "reserved_bit":
            m[p] |= 0x40
        else:
            if p != len(a) - 1:
                continue
            a[p] = T                          # arrival == trace_len
        tr = concat([(a, m)], T)
        g = _code(prof, tr)
        o = 0
        try:
            oracle_replay(oracle, prof, tr, want_keys=False, want_log=False, n_gpus=2)
        except oracle.OracleError as e:
            o = e.code
        assert o != 0 and g == o, (kind, p, g, o)


@pytest.mark.parametrize("shift", [(1, 3), (2, 0), (0, 5)])
def test_unaligned_device_buffers(oracle, shift):
    """arrival/meta views at 4-byte / 1-byte offsets: the scalar count path, same results."""
    import torch
    import paper_conf_middleware_bhasisjgpkd24_b200 as pkg
    rng = np.random.default_rng(11)
    prof = random_profiles(rng, 3)
    parts = []
    for _ in range(3):
        a, m, T = _trace(rng, n=int(rng.integers(2000, 5000)), M=3)
        parts.append((a, m))
    tr = concat(parts, T)
    sa, sm = shift
    n = tr.arrival_us.shape[0]
    abuf = torch.zeros(n + 8, dtype=torch.int32, device="cuda")
    mbuf = torch.zeros(n + 16, dtype=torch.uint8, device="cuda")
    arr = abuf[sa:sa + n]
    meta = mbuf[sm:sm + n]
    arr.copy_(torch.from_numpy(tr.arrival_us.view(np.int32)))
    meta.copy_(torch.from_numpy(tr.meta))
    off = torch.from_numpy(tr.replica_off).cuda()
    h = pkg.load_profiles(prof)
    out = h.replay_traces(arr, meta, off, trace_len_us=T, n_gpus=3, want_cand_keys=True, log_cap=n)
    g = {k: (v.cpu().numpy() if hasattr(v, "cpu") else v) for k, v in out.items()}
    g["hist"] = g["hist"].view(np.uint32)
    from gpu_common import GPU_LOG_DTYPE
    g["log"] = g["log"].reshape(3, n, 32).view(GPU_LOG_DTYPE).reshape(3, n)
    compare(g, oracle_replay(oracle, prof, tr, n_gpus=3), 3)
    ref = gpu_replay(prof, tr, n_gpus=3)
    for k in ("counters", "hist", "cand_keys"):
        assert np.array_equal(g[k], ref[k]), k


def test_score_epoch_enqueue_only_verdict(oracle):
    """protean_score_epoch only enqueues: an invalid state (geometry >= G) or batch_off[0] != 0 is
    latched in the handle's device word and raised by protean_score_epoch_status after the sync
    (SURVEY.md §8(b) "score_epoch enqueues on stream and returns"); the oracle rejects the same
    input with the same code; a valid call afterwards reports OK (the word is cleared)."""
    import torch
    import paper_conf_middleware_bhasisjgpkd24_b200 as pkg
    from paper_conf_middleware_bhasisjgpkd24_b200 import _abi as A
    from helpers import w1
    _, P, _ = w1()
    dev = torch.device("cuda", 0)
    h = pkg.load_profiles(P)
    rows = np.zeros((4, 16), np.uint8)
    for i, (rd, off, m, s) in enumerate([(5000, 0, 1, 0), (10000, 2, 0, 1), (30000, 4, 1, 0), (45000, 6, 0, 1)]):
        rows[i] = np.frombuffer(bytes(A.Batch(rd, off, 2, m, s, 0)), np.uint8)
    arr = torch.tensor(np.array([0, 5000, 0, 10000, 20000, 30000, 40000, 45000], np.int32), device=dev)

    def call(geom, off0):
        st = A.GpuState()
        st.geom, st.target, st.has_vm, st.vm_type = geom, 255, 1, 1
        t_state = torch.from_numpy(np.frombuffer(bytes(st), np.uint8).copy()).to(dev)
        t_off = torch.tensor([off0, 4], dtype=torch.int32, device=dev)
        out = h.score_epoch(n_replicas=1, n_gpus=1, epoch=0, batches=torch.from_numpy(rows.reshape(-1)).to(dev),
                            batch_off=t_off, arrival_us=arr, state=t_state, sync=False)
        torch.cuda.synchronize()
        try:
            h.score_epoch_status()
        except pkg.ProteanError as e:
            return e.code, out
        return 0, out

    code, _ = call(h.n_geoms, 0)
    assert code == A.EINVAL
    code, _ = call(2, 1)
    assert code == A.EINVAL
    code, out = call(2, 0)
    assert code == 0
    assert out["cand_key"].cpu().tolist() == [56320001, 64000002, 78080000]  # W1 golden
    assert out["cost"].cpu().tolist() == [(32.7726 / 8 * 1e6) / 3.6e9]
    ostate = (oracle.State * 1)()
    ostate[0].geom, ostate[0].target, ostate[0].has_vm = P.geoms.shape[0], -1, 1
    with pytest.raises(oracle.OracleError) as ei:
        oracle.score_epoch(P, R=1, N=1, epoch=0, batches=dict(ready=[5000], req_off=[0], n=[2], model=[1], strict=[0]),
                           batch_off=[0, 1], arrival=np.array([0, 5000], np.uint32), states=ostate)
    assert ei.value.code == A.EINVAL


def test_replica_off_checked_on_device(oracle):
    """replica_off is validated and scanned on the device (roff_scan_kernel; no host readback
    before the prepass): replica_off[0] != 0 or a decreasing entry is PROTEAN_EINVAL like the
    oracle's host check, with nothing else launched on the bad offsets; a valid trace of more
    replicas than the scan's 1024-wide chunk (empty replicas included) matches the oracle."""
    import torch
    import paper_conf_middleware_bhasisjgpkd24_b200 as pkg
    from paper_conf_middleware_bhasisjgpkd24_b200 import _abi as A
    rng = np.random.default_rng(21)
    prof = random_profiles(rng, 3)
    T = 2_000_000
    parts = []
    for r in range(1100):
        n = 0 if r % 7 == 3 else int(rng.integers(1, 12))
        a, m, _ = _trace(rng, n=n, M=3, T=T)
        parts.append((a, m))
    tr = concat(parts, T)
    h = pkg.load_profiles(prof)
    arr = torch.from_numpy(tr.arrival_us.view(np.int32)).cuda()
    meta = torch.from_numpy(tr.meta).cuda()
    R = len(parts)
    out = h.replay_traces(arr, meta, torch.from_numpy(tr.replica_off).cuda(), trace_len_us=T, n_gpus=2)
    o = oracle_replay(oracle, prof, tr, want_keys=False, want_log=False, n_gpus=2)
    assert np.array_equal(out["counters"].cpu().numpy(), o["counters"])
    assert np.array_equal(out["hist"].cpu().numpy().view(np.uint32), o["hist"])
    for bad in ("first", "decreasing"):
        off = tr.replica_off.copy()
        if bad == "first":
            off[0] = 1
        else:
            off[600] = off[599] - 1 if off[599] > 0 else off[601] + 5
        with pytest.raises(pkg.ProteanError) as ei:
            h.replay_traces(arr, meta, torch.from_numpy(off).cuda(), trace_len_us=T, n_gpus=2)
        assert ei.value.code == A.EINVAL
        with pytest.raises(oracle.OracleError) as eo:
            oracle_replay(oracle, prof, Trace(tr.arrival_us, tr.meta, off, T),
                          want_keys=False, want_log=False, n_gpus=2)
        assert eo.value.code == A.EINVAL
    # the handle is usable afterwards
    out2 = h.replay_traces(arr, meta, torch.from_numpy(tr.replica_off).cuda(), trace_len_us=T, n_gpus=2)
    assert np.array_equal(out2["counters"].cpu().numpy(), o["counters"])
