#!/bin/bash
export SPTRSV_GEN_CACHE=/tmp/sptrsv_gen
for d in -1 0 2; do timeout 300 python scripts/time_segs.py --config C2 --depth $d --tag "C2 depth=$d" 2>&1 | tail -1; done
for d in -1 1 2 4; do timeout 600 python scripts/time_segs.py --config C3 --depth $d --tag "C3 depth=$d" 2>&1 | tail -1 | cut -c1-60; done
for d in -1 1 3; do timeout 600 python scripts/time_segs.py --config C5 --nrhs 512 --reps 3 --depth $d --tag "C5 depth=$d" 2>&1 | tail -1 | cut -c1-60; done
