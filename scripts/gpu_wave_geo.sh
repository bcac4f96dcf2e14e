#!/bin/bash
# C2 triangle times under wave geometries / wait back-offs (tuning)
mkdir -p gpurun_out
for geo in ${GEOS:-"16,2,12,4" "16,2,6,4"}; do
  SPTRSV_WAVE=$geo timeout 300 python scripts/time_segs.py --config C2 --tag "geo=$geo" 2>&1 | tail -1
done
for ns in ${WAITS:-}; do
  SPTRSV_NVCC_FLAGS="-DSPTRSV_WAVE_WAIT_NS=$ns" python -c "from paper_conf_icpp_lun020_b200 import build; build.build(force=True)" > gpurun_out/build_exp.log 2>&1
  for geo in ${GEOS:-"16,2,12,4" "16,2,6,4"}; do
    SPTRSV_WAVE=$geo timeout 300 python scripts/time_segs.py --config C2 --tag "wait=$ns geo=$geo" 2>&1 | tail -1
  done
done
[ -n "$WAITS" ] && python -c "from paper_conf_icpp_lun020_b200 import build; build.build(force=True)" > /dev/null 2>&1
true
