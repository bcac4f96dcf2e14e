"""Build the oracle's plain-C library (TEST INFRASTRUCTURE ONLY)."""
from __future__ import annotations

import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "csrc", "oracle.c")
LIB = os.path.join(HERE, "liboracle.so")

# -ffp-contract=off: no FMA contraction, so Algorithm 1's "left_sum + val*x"
# rounds exactly as written; no -ffast-math, no vector intrinsics, no OpenMP.
CFLAGS = ["-O2", "-ffp-contract=off", "-fno-fast-math", "-fno-tree-vectorize",
          "-shared", "-fPIC", "-pthread"]


def build(force: bool = False) -> str:
    if (not force and os.path.exists(LIB)
            and os.path.getmtime(LIB) >= os.path.getmtime(SRC)):
        return LIB
    tmp = LIB + f".tmp{os.getpid()}"
    subprocess.check_call(["gcc", *CFLAGS, SRC, "-o", tmp])
    os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    print(build(force=True))
