#!/bin/bash
# C5 allocator probe; solve-only launch list of C3; compute-sanitizer on the spin-wait kernels
O=gpurun_out/r2r
mkdir -p $O
export SPTRSV_GEN_CACHE=/tmp/gencache
timeout 900 python scripts/alloc_probe.py C5 2>&1 | tail -4
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k "regex:tri_|sq_|perm_" -c 400 --csv --log-file $O/launches_C3_solve.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > $O/ncu_launch.log 2>&1; echo "ncu launches rc=$?"
for tool in memcheck racecheck synccheck; do
  timeout 1200 compute-sanitizer --tool $tool --print-limit 20 python -m pytest tests/test_gpu_parity.py -q -x -k "test_forced_kernels and (C1 or C3) and SQ_ADAPT" > $O/sanitize_$tool.log 2>&1; echo "sanitizer $tool rc=$?"; grep -E "ERROR SUMMARY|passed|failed" $O/sanitize_$tool.log | tail -3
done
