#!/bin/bash
# depth probe at 512 RHS (C5) and C3 again
export SPTRSV_GEN_CACHE=/tmp/gencache
PROBE_NRHS=512 timeout 1200 python scripts/depth_probe.py C5 0 1 2 2>&1 | grep depth
timeout 1200 python scripts/depth_probe.py C3 1 2 3 2>&1 | grep depth
