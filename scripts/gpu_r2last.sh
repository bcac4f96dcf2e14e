#!/bin/bash
# depth re-check with the final sync-free kernel; piece size 128 with the threshold 64
export SPTRSV_GEN_CACHE=/tmp/gencache
timeout 900 python scripts/depth_probe.py C3 0 1 2 3 2>&1 | grep depth
PROBE_NRHS=512 timeout 900 python scripts/depth_probe.py C5 0 1 2>&1 | grep depth
SPTRSV_NVCC_FLAGS="-DSPTRSV_SF_NB=128" python -c "import __graft_entry__ as g; g.build()" > /tmp/b.log 2>&1 && { echo "== SF_NB 128"; timeout 600 python scripts/sweep_sf.py C3 2>&1 | tail -1; }
python -c "import __graft_entry__ as g; g.build()" > /tmp/b.log 2>&1; echo "== default"; timeout 600 python scripts/sweep_sf.py C3 2>&1 | tail -1
