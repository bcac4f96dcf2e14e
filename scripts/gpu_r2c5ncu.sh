#!/bin/bash
# C5 (512 RHS, depth 0 under R33): full ncu capture of the dominant tri_syncfree_multi, summarised on the box
O=gpurun_out/r2c5
mkdir -p $O
export SPTRSV_GEN_CACHE=/tmp/gencache
timeout 600 python scripts/prof_solve.py --config C5 --nrhs 512 --reps 1 > $O/plain.log 2>&1 && \
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:tri_syncfree_multi -c 1 -o /tmp/prof_C5 -f python scripts/prof_solve.py --config C5 --nrhs 512 --reps 1 > $O/ncu_C5.log 2>&1; echo "ncu C5 rc=$?"
python scripts/ncu_summary.py --rep /tmp/prof_C5.ncu-rep --out $O/r02_C5_final --impl C5:TRI_SYNCFREE --json $O/ncu_summary.json --title "C5 512 RHS (round 2 final, depth 0)" > /dev/null 2>&1; echo "summary rc=$?"
ncu -i /tmp/prof_C5.ncu-rep --page source --csv --print-source sass > /tmp/src_C5.csv 2>/dev/null
python scripts/sass_hot.py /tmp/src_C5.csv > $O/r02_C5_final_sass_hot.md 2>/dev/null; rm -f /tmp/prof_C5.ncu-rep /tmp/src_C5.csv
