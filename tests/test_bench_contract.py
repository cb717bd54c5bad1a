"""bench.py's JSON line keeps the driver's contract: the reference arm (the CPU oracle, runs here)
and, on a B200, our arm on a reduced config-5 shape for the replay, alg2 and sweep paths."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
BASE = ["metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
        "vs_baseline", "dtype", "data", "config", "cpu_baseline", "e2e"]


def _run(args, timeout=900):
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], capture_output=True, text=True,
                         timeout=timeout, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-2000:]
    return json.loads(out.stdout.strip().splitlines()[-1])


def test_reference_arm_line():
    d = _run(["--impl", "reference", "--replicas", "2", "--seconds", "10", "--steps", "1", "--warmup", "0"])
    for k in BASE + ["impl"]:
        assert k in d, k
    assert d["impl"] == "reference" and d["value"] > 0
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["cpu_baseline"]["kind"] == "oracle"


@pytest.mark.gpu
@pytest.mark.parametrize("extra", [[], ["--policy", "alg2"], ["--path", "sweep", "--replicas", "64"]])
def test_our_arm_line(extra):
    args = ["--replicas", "256", "--seconds", "30", "--steps", "3", "--warmup", "3", "--cpu-sample", "2",
            "--e2e-replicas", "16"] + extra
    d = _run(args)
    for k in BASE + ["roofline", "gpu_launches", "clocks"]:
        assert k in d, k
    assert d["value"] > 0 and d["n_gpus"] == 1 and d["steps"] == 3
    r = d["roofline"]
    assert r["bound"] in ("hbm", "alu") and 0 < r["frac"] < 1 and r["peak"] > 0
    assert d["e2e"]["value"] > 0 and d["e2e"]["h2d_bytes_per_step"] > 0
    assert d["gpu_launches"] > 0 and "sm_mhz" in d["clocks"]


def test_gpus_flag_relaunches_one_process_per_rank():
    """--gpus N outside torchrun re-launches bench.py through torch.distributed.run (ADVICE r1:
    the flag used to be parsed and ignored); the reference arm prints one line from rank 0 with
    n_gpus = N.  A WORLD_SIZE that contradicts --gpus fails loudly."""
    d = _run(["--impl", "reference", "--gpus", "2", "--replicas", "2", "--seconds", "5", "--steps", "1",
              "--warmup", "0"])
    assert d["impl"] == "reference" and d["n_gpus"] == 2
    env = dict(os.environ, WORLD_SIZE="3", RANK="0", LOCAL_RANK="0")
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--gpus", "2"],
                         capture_output=True, text=True, timeout=300, cwd=ROOT, env=env)
    assert out.returncode != 0 and "WORLD_SIZE" in out.stderr
