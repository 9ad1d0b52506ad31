"""Build libtid.so in-tree for sm_100a (nvcc; no GPU needed to compile)."""
from __future__ import annotations

import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libtid.so")
SOURCES = [os.path.join(CSRC, f) for f in ("tid_api.cu", "tid_kernels.cu", "tid_f16.cu", "tid_geom.cu")]
DEPS = SOURCES + [os.path.join(CSRC, "tid_kernels.cuh"), os.path.join(ROOT, "include", "tid.h")]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17",
         "-Xcompiler", "-fPIC", "-shared", "-Xptxas", "-warn-spills"]


def stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(d) > t for d in DEPS)


def build(force: bool = False, verbose: bool = False, out: str | None = None, defines=()) -> str:
    """Compile libtid.so (or a variant at `out` with extra -D defines, for experiments)."""
    target = out or LIB
    if force or out or stale():
        tmp = target + ".tmp%d" % os.getpid()
        cmd = [NVCC, *FLAGS, *[f"-D{d}" for d in defines], "-o", tmp, *SOURCES, "-ldl"]
        if verbose:
            print(" ".join(cmd), file=sys.stderr)
        subprocess.check_call(cmd)
        os.replace(tmp, target)
    return target


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))
