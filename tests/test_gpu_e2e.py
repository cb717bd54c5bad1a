"""The pipelined end-to-end call (Handle.replay_traces_pinned: chunked H2D overlapped with the
replay, results copied back per chunk) returns exactly what one device-resident call returns,
which the parity tests pin to the oracle.  -m gpu."""
import numpy as np
import pytest

from protean_inputs import mix_a_params, synth_profiles, tick_trace

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("chunks", [1, 3, 7])
def test_pinned_pipeline_equals_single_call(chunks):
    import torch
    import paper_conf_middleware_bhasisjgpkd24_b200 as pkg
    tr = tick_trace(mix_a_params(7, seed=4, seconds=20, replica_base=100))
    h = pkg.load_profiles(synth_profiles())
    ref = h.replay_traces_host(tr, n_gpus=8)
    arr = torch.from_numpy(np.ascontiguousarray(tr.arrival_us).view(np.int32)).pin_memory()
    meta = torch.from_numpy(np.ascontiguousarray(tr.meta)).pin_memory()
    off = torch.from_numpy(np.ascontiguousarray(tr.replica_off, np.int64)).pin_memory()
    got = h.replay_traces_pinned(arr, meta, off, trace_len_us=tr.trace_len_us, chunks=chunks, n_gpus=8,
                                 replica_base=tr.replica_base)
    for k in ("counters", "accum", "hist", "p50_p99", "cost", "util", "decisions", "n_batches"):
        assert np.array_equal(got[k].numpy(), np.asarray(ref[k]).reshape(got[k].shape)), k
