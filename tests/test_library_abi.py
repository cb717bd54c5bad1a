"""Not-GPU checks of the boundary: the C-ABI library builds for sm_100a, loads, and exports every
entry point include/protean.h declares; the binding refuses to run without a GPU."""
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def lib():
    from paper_conf_middleware_bhasisjgpkd24_b200 import build
    path = build.build()
    from paper_conf_middleware_bhasisjgpkd24_b200 import _abi
    return _abi.load(path, require_cuda=False), path


def test_exports_every_declared_symbol(lib):
    L, path = lib
    hdr = open(os.path.join(ROOT, "include", "protean.h")).read()
    declared = set(re.findall(r"\b(protean_[a-z_0-9]+)\s*\(", hdr))
    assert declared >= {"protean_load_profiles", "protean_score_epoch", "protean_replay_traces"}
    nm = subprocess.run(["nm", "-D", "--defined-only", path], capture_output=True, text=True).stdout
    exported = set(re.findall(r"\bT (protean_[a-z_0-9]+)", nm))
    assert declared <= exported, declared - exported
    for s in declared:
        getattr(L, s)


def test_sm100a_cubin_only(lib):
    _, path = lib
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", path], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_strerror_and_no_cpu_fallback(lib):
    L, _ = lib
    assert L.protean_strerror(-1) == b"invalid argument"
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    import paper_conf_middleware_bhasisjgpkd24_b200 as pkg
    from protean_inputs import c1_profiles
    with pytest.raises(Exception):
        h = pkg.load_profiles(c1_profiles())
        h.replay_traces_host(__import__("protean_inputs").c1_trace(), n_gpus=1)


def test_product_does_not_import_oracle():
    pkg_dir = os.path.join(ROOT, "paper_conf_middleware_bhasisjgpkd24_b200")
    for dp, _, fs in os.walk(pkg_dir):
        for f in fs:
            if f.endswith((".py", ".cu", ".cuh", ".cpp", ".h")):
                src = open(os.path.join(dp, f)).read()
                assert "oracle" not in re.sub(r"//.*|#.*", "", src).replace("Oracle", ""), f
