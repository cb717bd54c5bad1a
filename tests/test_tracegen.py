"""The CUDA twin of the GEN-1 input generator produces the numpy generator's bytes (-m gpu)."""
import numpy as np
import pytest

from protean_inputs import mix_a_params, mix_b_params, tick_trace

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("kind", ["a", "b"])
def test_tracegen_twin_bytes(kind):
    from tools import tracegen
    gp = mix_a_params(3, seed=5, seconds=25, replica_base=7) if kind == "a" else \
        mix_b_params(2, seed=9, seconds=20, replica_base=3)
    ref = tick_trace(gp)
    arr, meta, off = tracegen.generate_on_device(gp, 0)
    assert np.array_equal(off.cpu().numpy(), ref.replica_off)
    assert np.array_equal(arr.cpu().numpy().view(np.uint32), ref.arrival_us)
    assert np.array_equal(meta.cpu().numpy(), ref.meta)
