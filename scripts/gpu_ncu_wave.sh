#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 600 ncu --section SourceCounters --section WarpStateStats --warp-sampling-interval 0 --clock-control none --import-source on -k regex:tri_wave -s 2 -c 1 -o gpurun_out/prof_wave_src -f python scripts/prof_solve.py --config C2 --reps 2 > gpurun_out/ncu_wave.log 2>&1; echo "ncu rc=$?"
tail -3 gpurun_out/ncu_wave.log
