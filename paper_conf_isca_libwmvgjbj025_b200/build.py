"""Build libtriosim.so in-tree with nvcc for sm_100a (no torch extension machinery)."""
from __future__ import annotations

import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
SRC = [os.path.join(HERE, "csrc", f) for f in ("ts_host.cu", "ts_kernels.cu", "ts_k3.cu", "ts_k3h.cu")]
HDR = [os.path.join(HERE, "csrc", "ts_internal.h"), os.path.join(ROOT, "include", "triosim.h")]
OUT = os.path.join(HERE, "libtriosim.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-lineinfo", "-O3", "--fmad=false", "-std=c++17",
         "-Xcompiler", "-fPIC", "-shared", "-I" + os.path.join(ROOT, "include")]


def stale() -> bool:
    if not os.path.exists(OUT):
        return True
    t = os.path.getmtime(OUT)
    return any(os.path.getmtime(f) > t for f in SRC + HDR)


def build(force=False, verbose=False) -> str:
    if force or stale():
        tmp = OUT + f".tmp{os.getpid()}"
        cmd = [NVCC, *FLAGS, *SRC, "-o", tmp]
        if verbose:
            print(" ".join(cmd), file=sys.stderr)
        subprocess.check_call(cmd)
        os.replace(tmp, OUT)
    return OUT


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))
