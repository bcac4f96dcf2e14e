#!/bin/bash
# C5 seg0 (tri_syncfree_multi) ncu: round-1 tree vs HEAD; HEAD bench C5 with the untiled SpMM default
O=gpurun_out/r2t
mkdir -p $O
export SPTRSV_GEN_CACHE=/tmp/gencache
timeout 900 python bench.py --config C5 --steps 5 --warmup 3 --no-cpu-baseline > $O/bench_C5.log 2>&1; echo "bench rc=$?"
python -c "
import json
for l in open('$O/bench_C5.log'):
    if l.startswith('{'): d=json.loads(l); print(d['ms_per_step'], {k: round(v,3) for k,v in d['segment_ms'].items()})"
(cd _r1 && timeout 900 ncu --set full --clock-control none -k regex:tri_syncfree_multi -c 1 -o ../$O/r1_sfm -f python scripts/prof_solve.py --config C5 --nrhs 512 --reps 1 > ../$O/ncu_r1.log 2>&1); echo "ncu r1 rc=$?"
timeout 900 ncu --set full --clock-control none -k regex:tri_syncfree_multi -c 1 -o $O/head_sfm -f python scripts/prof_solve.py --config C5 --nrhs 512 --reps 1 > $O/ncu_head.log 2>&1; echo "ncu head rc=$?"
