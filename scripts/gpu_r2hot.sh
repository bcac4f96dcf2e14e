#!/bin/bash
# tri_sf_mixed "hot front" polling sweep on C3 (and C5 one RHS)
export SPTRSV_GEN_CACHE=/tmp/gencache

timeout 1500 python scripts/sweep_sf.py C3 "SPTRSV_SF_HOT=0:1:0" "SPTRSV_SF_HOT=128:2:100" "SPTRSV_SF_HOT=128:3:80" "SPTRSV_SF_HOT=256:2:150" "SPTRSV_SF_HOT=256:3:100" "SPTRSV_SF_HOT=512:2:100" "SPTRSV_SF_HOT=1024:2:200" "SPTRSV_SF_HOT=64:4:60" 2>&1 | grep -v Warn | tail -9
