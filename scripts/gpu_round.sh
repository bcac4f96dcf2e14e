#!/bin/bash
# One gpurun session: smoke, GPU parity tests, bench of every config, ncu
# launch list of the default bench, one full ncu capture of the top kernel.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,driver_version --format=csv > gpurun_out/gpu.txt 2>&1
nproc > gpurun_out/nproc.txt; lscpu | grep "Model name" >> gpurun_out/nproc.txt
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"
tail -2 gpurun_out/smoke.log
if [ -z "$NO_TESTS" ]; then
timeout ${TEST_TIMEOUT:-1500} python -m pytest tests -m gpu -q ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"
tail -15 gpurun_out/pytest_gpu.log
fi
for c in ${CONFIGS:-C2 C1 C3 C4 C5}; do
  steps=30; [ $c = C5 ] && steps=5
  timeout 900 python bench.py --config $c --steps $steps --warmup 3 ${BENCH_ARGS} > gpurun_out/bench_$c.log 2>&1; echo "bench $c rc=$?"
  grep '^{' gpurun_out/bench_$c.log | cut -c1-700
done
if [ -z "$NO_NCU" ]; then
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c2.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_launch_bench.log 2>&1; echo "ncu launches rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:${NCU_KERNEL:-tri_wave} -s 2 -c 1 -o gpurun_out/prof_c2_top -f python scripts/prof_solve.py --config C2 --reps 3 > gpurun_out/ncu_c2.log 2>&1; echo "ncu full rc=$?"
fi
ls -la gpurun_out/
