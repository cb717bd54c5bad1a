"""Run one replay with the phase-timing debug build (libprotean_phase.so) and print the share of
CTA wall cycles per epoch phase (thread 0 clock64 between barriers)."""
import ctypes as C
import os
import shutil
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
PKG = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "paper_conf_middleware_bhasisjgpkd24_b200")
import paper_conf_middleware_bhasisjgpkd24_b200._abi as A  # noqa: E402

A.LIB_PATH = os.path.join(PKG, os.environ.get("PHASE_LIB", "libprotean_phase.so"))
import torch  # noqa: E402

import paper_conf_middleware_bhasisjgpkd24_b200 as pkg  # noqa: E402
from protean_inputs import mix_a_params, synth_profiles  # noqa: E402
from tools import tracegen  # noqa: E402

R = int(sys.argv[1]) if len(sys.argv) > 1 else 444
S = int(sys.argv[2]) if len(sys.argv) > 2 else 60
MIX = os.environ.get("PHASE_MIX", "a")
NG = int(os.environ.get("PHASE_N", "8"))
GS = 0
if MIX == "b":
    from protean_inputs import mix_b_params
    gp = mix_b_params(R, seed=2, seconds=S)
elif MIX == "b8":  # the C4 shape: Mix B x 8, 37 geometries (use PHASE_N=64)
    from protean_inputs import mix_b_params
    gp, GS = mix_b_params(R, seed=4, seconds=S, scale=8.0), 1
else:
    gp = mix_a_params(R, seed=1, seconds=S)
arr, meta, roff = tracegen.generate_on_device(gp, 0)
A._lib = None
L = A.load(A.LIB_PATH)
h = pkg.load_profiles(synth_profiles().with_geometry_set(GS))
POL = int(sys.argv[3]) if len(sys.argv) > 3 else 0
out = h.replay_traces(arr, meta, roff, trace_len_us=gp.trace_len_us, n_gpus=NG, policy=POL)
torch.cuda.synchronize()
buf = (C.c_ulonglong * 13)()
L.protean_debug_phase_cycles(buf)
names = ["-", "A vm/install + B window layout", "-", "B window TMA wait", "C formation",
         "C rank (+ closed-form dispatch)", "D dispatch", "E units + F accounting", "G decide",
         "G cap + epoch barrier"]
tot = sum(buf[:10]) or 1
print("kernel ms", h.last_timings()[1])
for n, v in zip(names, buf):
    print(f"{100 * v / tot:5.1f}%  {n}")
tt = sum(buf[10:13]) or 1
ntask = (R * (gp.seconds + 1))
for n, v in zip(["actual units", "candidate units", "accounting tasks"], buf[10:13]):
    print(f"task time {100 * v / tt:5.1f}%  {n}  ({v / ntask:.0f} warp-cycles per replica-epoch)")
