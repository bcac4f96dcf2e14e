#!/bin/bash
mkdir -p gpurun_out
for geo in ${GEOS:-"1,1,12,4" "1,1,6,4" "2,1,12,4" "1,2,12,4" "4,2,12,4" "16,2,12,4"}; do
  SPTRSV_WAVE=$geo timeout 120 python scripts/wave_iso.py --nx ${NX:-32} --ny ${NY:-20000} --tag "geo=$geo" 2>&1 | tail -1
done
