"""Build libsptrsv_b200.so in-tree with nvcc for sm_100a (B200) only."""
from __future__ import annotations

import os
import shutil
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
INCLUDE = os.path.join(ROOT, "include")
LIB = os.path.join(HERE, "libsptrsv_b200.so")
BUILD = os.path.join(ROOT, "build", "sptrsv")

SOURCES = ["analyse.cpp", "analyse_dev.cu", "capi.cpp", "exec.cu"]
HEADERS = ["internal.h", "kernels.cuh"]

NVCC = os.environ.get("NVCC", shutil.which("nvcc") or "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
COMMON = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC,-fvisibility=hidden,-O3",
          "-I", INCLUDE, "-I", CSRC]
# extra nvcc flags for instrumented builds (e.g. -DSPTRSV_WAVE_TRACE); never set by the driver
COMMON += os.environ.get("SPTRSV_NVCC_FLAGS", "").split()


def _stale(out: str, deps: list[str]) -> bool:
    if not os.path.exists(out):
        return True
    t = os.path.getmtime(out)
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False) -> str:
    os.makedirs(BUILD, exist_ok=True)
    # a change of the compile flags (SPTRSV_NVCC_FLAGS) rebuilds everything
    stamp = os.path.join(BUILD, "flags.txt")
    flags = " ".join(COMMON)
    if not os.path.exists(stamp) or open(stamp).read() != flags:
        force = True
        with open(stamp, "w") as f:
            f.write(flags)
    hdrs = [os.path.join(CSRC, h) for h in HEADERS] + [os.path.join(INCLUDE, "sptrsv.h")]
    objs = []
    for src in SOURCES:
        s = os.path.join(CSRC, src)
        o = os.path.join(BUILD, src + ".o")
        objs.append(o)
        if force or _stale(o, [s] + hdrs):
            lang = ["-x", "cu"] if src.endswith(".cu") else ["-x", "c++"]
            extra = ["-Xptxas", "-v"] if (verbose and src.endswith(".cu")) else []
            cmd = [NVCC, *ARCH, *COMMON, *extra, *lang, "-c", s, "-o", o]
            subprocess.check_call(cmd)
    if force or _stale(LIB, objs):
        tmp = LIB + f".tmp{os.getpid()}"
        cmd = [NVCC, *ARCH, "-shared", "-o", tmp, *objs, "-cudart", "static", "-lpthread"]
        subprocess.check_call(cmd)
        os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
