#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2j_build.log 2>&1 || { echo BUILD FAILED; tail gpurun_out/r2j_build.log; exit 1; }
export SPTRSV_GEN_CACHE=/tmp/gencache
timeout 600 python scripts/chain_probe.py 2>&1 | tail -6
echo "== WROW C3"; SPTRSV_SF_WROW=1 timeout 900 python scripts/sweep_sf.py C3 2>&1 | tail -1
echo "== MIXED C3"; SPTRSV_SF_MIXED=1 timeout 900 python scripts/sweep_sf.py C3 2>&1 | tail -1
