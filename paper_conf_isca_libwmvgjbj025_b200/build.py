"""Build libtriosim.so in-tree with nvcc for sm_100a (no torch extension machinery).  Each .cu is
compiled to an object in parallel (no relocatable device code crosses files), then linked."""
from __future__ import annotations

import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
SRC = [os.path.join(HERE, "csrc", f) for f in ("ts_host.cu", "ts_kernels.cu", "ts_k3.cu", "ts_k3h.cu", "ts_timeline.cu")]
HDR = [os.path.join(HERE, "csrc", "ts_internal.h"), os.path.join(ROOT, "include", "triosim.h")]
OUT = os.environ.get("TS_BUILD_OUT", os.path.join(HERE, "libtriosim.so"))   # override: A/B variants
OBJ = os.path.join(HERE, "csrc", "build")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = [*ARCH, "-lineinfo", "-O3", "--fmad=false", "-std=c++17", "-Xcompiler", "-fPIC",
         "-I" + os.path.join(ROOT, "include")] + os.environ.get("TS_NVCC_EXTRA", "").split()


def stale() -> bool:
    if not os.path.exists(OUT):
        return True
    t = os.path.getmtime(OUT)
    return any(os.path.getmtime(f) > t for f in SRC + HDR)


def build(force=False, verbose=False) -> str:
    if force or stale():
        os.makedirs(OBJ, exist_ok=True)
        tag = os.getpid()
        objs, procs = [], []
        for f in SRC:
            o = os.path.join(OBJ, os.path.basename(f)[:-3] + f".{tag}.o")
            cmd = [NVCC, *FLAGS, "-c", f, "-o", o]
            if verbose:
                print(" ".join(cmd), file=sys.stderr)
            objs.append(o)
            procs.append((cmd, subprocess.Popen(cmd)))
        bad = [cmd for cmd, p in procs if p.wait() != 0]
        try:
            if bad:
                raise subprocess.CalledProcessError(1, bad[0])
            tmp = OUT + f".tmp{tag}"
            link = [NVCC, *ARCH, "-shared", *objs, "-o", tmp]
            if verbose:
                print(" ".join(link), file=sys.stderr)
            subprocess.check_call(link)
            os.replace(tmp, OUT)
        finally:
            for o in objs:
                if os.path.exists(o):
                    os.remove(o)
    return OUT


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))
