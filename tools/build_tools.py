"""Builds the input-generator twin (tools/tracegen.cu -> tools/libtracegen.so), sm_100a."""
import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
OUT = os.path.join(HERE, "libtracegen.so")


def build(force: bool = False) -> str:
    src = os.path.join(HERE, "tracegen.cu")
    if not os.path.exists(src):
        return ""
    if force or not os.path.exists(OUT) or os.path.getmtime(src) > os.path.getmtime(OUT):
        subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-gencode", "arch=compute_100a,code=sm_100a",
                               "-O3", "-lineinfo", "-Xcompiler", "-fPIC", "-shared", "-cudart", "static",
                               "-o", OUT, src])
    return OUT
