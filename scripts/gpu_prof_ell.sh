#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
SPTRSV_ELL_GEOM=2048,4096,4 timeout 600 ncu --set full --warp-sampling-interval 0 --clock-control none --import-source on -k regex:tri_chain_ell -s 2 -c 1 -o gpurun_out/prof_c2_ell -f python scripts/prof_solve.py --config C2 --reps 3 > gpurun_out/ncu_ell.log 2>&1; echo "ncu rc=$?"
tail -3 gpurun_out/ncu_ell.log
