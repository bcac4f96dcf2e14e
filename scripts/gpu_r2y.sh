#!/bin/bash
# recursion depth probe (C3, C4, C5 one RHS) with the B200 kernels
O=gpurun_out/r2y
mkdir -p $O
export SPTRSV_GEN_CACHE=/tmp/gencache
timeout 1200 python scripts/depth_probe.py C3 0 1 2 3 4 2>&1 | grep depth
timeout 600 python scripts/depth_probe.py C5 0 1 2 3 2>&1 | grep depth
timeout 600 python scripts/depth_probe.py C4 0 1 2 2>&1 | grep depth
