#!/bin/bash
# ncu captures: launch list of a bench run + full sets of the top kernels
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c2.csv python scripts/prof_solve.py --config C2 --reps 2 > /dev/null 2>&1; echo "launches rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tri_chain_tma -s 2 -c 1 -o gpurun_out/prof_c2_chain -f python scripts/prof_solve.py --config C2 --reps 3 > gpurun_out/ncu_c2.log 2>&1; echo "ncu c2 rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tri_syncfree -s 2 -c 1 -o gpurun_out/prof_c3_sf -f python scripts/prof_solve.py --config C3 --reps 1 > gpurun_out/ncu_c3.log 2>&1; echo "ncu c3 rc=$?"
ls -la gpurun_out/
