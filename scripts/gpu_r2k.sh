#!/bin/bash
mkdir -p gpurun_out
export SPTRSV_GEN_CACHE=/tmp/gencache
for cfg in "1 64" "2 64" "3 64" "4 48" "2 128"; do
  set -- $cfg
  SPTRSV_NVCC_FLAGS="-DSPTRSV_SF_POLLS=$1 -DSPTRSV_SF_GAP=$2" python -c "from paper_conf_icpp_lun020_b200 import build; build.build(force=True)" > /dev/null 2>&1 || { echo BUILD FAILED; exit 1; }
  echo "== POLLS=$1 GAP=$2"
  SPTRSV_SF_MIXED=1 timeout 600 python scripts/sweep_sf.py C3 2>&1 | tail -1
done
