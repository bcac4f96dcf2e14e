#!/bin/bash
# t_lvl microbenchmarks, C5 through the NCCL sharded path at world 1, and ncu
# full captures of the top kernels of C3 / C4 / C5.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/t_lvl scripts/microbench/t_lvl.cu && /tmp/t_lvl > gpurun_out/t_lvl.txt 2>&1; echo "t_lvl rc=$?"; cat gpurun_out/t_lvl.txt
timeout 900 python bench.py --config C5 --steps 5 --warmup 3 --dist --no-cpu-baseline > gpurun_out/bench_C5_dist.log 2>&1; echo "bench C5 dist rc=$?"; grep '^{' gpurun_out/bench_C5_dist.log | cut -c1-400; tail -3 gpurun_out/bench_C5_dist.log | cut -c1-300
timeout 600 python bench.py --steps 20 --warmup 3 > gpurun_out/bench_C2.log 2>&1; echo "bench C2 rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:tri_syncfree -s 2 -c 1 -o gpurun_out/prof_c3_sf -f python scripts/prof_solve.py --config C3 --reps 1 > gpurun_out/ncu_c3.log 2>&1; echo "ncu c3 rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:tri_syncfree -c 1 -o gpurun_out/prof_c4_sf -f python scripts/prof_solve.py --config C4 --reps 1 > gpurun_out/ncu_c4.log 2>&1; echo "ncu c4 rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"sq_multi|perm_in_cm|tri_syncfree_multi|tri_level_multi" -c 6 -o gpurun_out/prof_c5 -f python scripts/prof_solve.py --config C5 --nrhs 512 --reps 1 > gpurun_out/ncu_c5.log 2>&1; echo "ncu c5 rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c3.csv python scripts/prof_solve.py --config C3 --reps 2 > /dev/null 2>&1; echo "launch c3 rc=$?"
ls -la gpurun_out
