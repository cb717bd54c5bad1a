"""Mode G across PROCESSES (-m gpu): two ranks, each its own process and CUDA context on cuda:0,
wired exactly as on a multi-GPU box — protean_xchg_export -> all-gather of the 64-byte CUDA IPC
handles over a torch.distributed (gloo) group -> protean_xchg_import (parallel.setup_geometry_sharding)
— then one replay per rank with shard_mode = 1.  Each kernel stores its (best, current) key pairs
into BOTH ranks' exchange buffers (its own and the peer's cudaIpcOpenMemHandle mapping) and
acquires the peer's flags at system scope every epoch.  Two contexts on one GPU time-slice, so
the exchange also proves progress under preemption.  Every rank's outputs must equal the oracle's
1-rank result (counters 8/9 and cand_keys per rank's range, merged)."""
import os
import subprocess
import sys

import numpy as np
import pytest

from gpu_common import GPU_LOG_DTYPE, compare, oracle_replay

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _workload():
    from protean_inputs import mix_a_params, synth_profiles, tick_trace
    return synth_profiles(), tick_trace(mix_a_params(3, seed=9, seconds=30, replica_base=40))


def _worker(rank: int, world: int, port: int, outdir: str):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), PROTEAN_XCHG_TIMEOUT_S="120")
    sys.path.insert(0, ROOT)
    import torch
    import torch.distributed as dist
    import paper_conf_middleware_bhasisjgpkd24_b200 as pkg
    from paper_conf_middleware_bhasisjgpkd24_b200.parallel import setup_geometry_sharding
    dist.init_process_group("gloo", rank=rank, world_size=world)
    prof, tr = _workload()
    N, R = 8, tr.n_replicas
    h = pkg.load_profiles(prof, device=0)
    setup_geometry_sharding(h, world, rank, R, N)
    dist.barrier()
    dev = torch.device("cuda", 0)
    arr = torch.from_numpy(np.ascontiguousarray(tr.arrival_us).view(np.int32)).to(dev)
    meta = torch.from_numpy(np.ascontiguousarray(tr.meta)).to(dev)
    off = torch.from_numpy(np.ascontiguousarray(tr.replica_off, np.int64)).to(dev)
    E = h.num_epochs(tr.trace_len_us)
    log_cap = int(np.max(np.diff(tr.replica_off)))
    out = h.alloc_replay_out(R, E, N, cand_keys=True, log_cap=log_cap)
    for call in range(2):  # two calls: sequence numbers continue across calls
        h.replay_traces(arr, meta, off, trace_len_us=tr.trace_len_us, out=out, n_gpus=N, shard_mode=1,
                        rank=rank, nranks=world, replica_base=tr.replica_base)
        torch.cuda.synchronize()
        np.savez(os.path.join(outdir, f"rank{rank}_call{call}.npz"),
                 **{k: v.cpu().numpy() for k, v in out.items() if hasattr(v, "cpu")})
    dist.barrier()
    h.close()
    dist.destroy_process_group()


def _compute_mode() -> str:
    try:
        return subprocess.run(["nvidia-smi", "--id=0", "--query-gpu=compute_mode", "--format=csv,noheader"],
                              capture_output=True, text=True, timeout=30).stdout.strip()
    except Exception:
        return ""


def test_two_process_ipc_exchange(oracle, tmp_path):
    if "Exclusive" in _compute_mode():
        pytest.skip("GPU in an exclusive compute mode: a second process cannot open a context")
    import socket
    import paper_conf_middleware_bhasisjgpkd24_b200 as pkg
    from paper_conf_middleware_bhasisjgpkd24_b200.parallel import merge_geometry_shards
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    world = 2
    code = ("import sys; sys.path.insert(0, {root!r}); sys.path.insert(0, {tests!r}); "
            "import test_gpu_modeg_ipc as t; t._worker({rank}, {world}, {port}, {out!r})")
    procs = [subprocess.Popen([sys.executable, "-c", code.format(root=ROOT, tests=os.path.join(ROOT, "tests"),
                                                                 rank=k, world=world, port=port, out=str(tmp_path))],
                              cwd=ROOT, stdout=subprocess.PIPE, stderr=subprocess.STDOUT, text=True)
             for k in range(world)]
    logs = []
    for p in procs:
        try:
            logs.append(p.communicate(timeout=600)[0])
        except subprocess.TimeoutExpired:
            for q in procs:
                q.kill()
            raise AssertionError("mode G processes did not finish")
    assert all(p.returncode == 0 for p in procs), "\n".join(l[-3000:] for l in logs)
    prof, tr = _workload()
    R = tr.n_replicas
    bounds = pkg.geometry_split(prof, world)
    o = oracle_replay(oracle, prof, tr, n_gpus=8, want_keys=True, want_log=True)
    log_cap = int(np.max(np.diff(tr.replica_off)))
    for call in range(2):
        host = []
        for k in range(world):
            d = dict(np.load(tmp_path / f"rank{k}_call{call}.npz"))
            d["hist"] = d["hist"].view(np.uint32)
            d["log"] = d["log"].reshape(R, log_cap, 32).view(GPU_LOG_DTYPE).reshape(R, log_cap)
            host.append(d)
            assert np.array_equal(d["decisions"], o["decisions"])
            assert np.array_equal(d["counters"][:, :8], o["counters"][:, :8])
        compare(merge_geometry_shards(host, bounds), o, R)
