#!/bin/bash
# Iteration run: GPU tests (optional), selected benches, optional ncu capture.
#   CONFIGS="C3 C5" TESTS=1 NCU_CFG=C3 NCU_K=sq_adapt NCU_S=3 bash scripts/gpu_iter.sh
mkdir -p gpurun_out
if [ -n "$TESTS" ]; then
  timeout 1500 python -m pytest tests -m gpu -q -x ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"
  tail -4 gpurun_out/pytest_gpu.log
fi
for c in ${CONFIGS}; do
  steps=30; [ $c = C5 ] && steps=5
  timeout 900 python bench.py --config $c --steps $steps --warmup 3 --no-cpu-baseline ${BENCH_ARGS} > gpurun_out/bench_$c.log 2>&1; echo "bench $c rc=$?"
  grep '^{' gpurun_out/bench_$c.log | python -c "
import json,sys
d=json.loads(sys.stdin.read())
print('$c ms=%.4f pre=%.1f' % (d['ms_per_step'], d['preprocess_ms']), {k: round(v,4) for k,v in d['segment_ms'].items()})
"
done
if [ -n "$NCU_CFG" ]; then
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:${NCU_K} -s ${NCU_S:-0} -c 1 -o gpurun_out/prof_${NCU_CFG}_${NCU_K} -f python scripts/prof_solve.py --config ${NCU_CFG} --reps 2 ${PROF_ARGS} > gpurun_out/ncu_${NCU_CFG}.log 2>&1; echo "ncu rc=$?"
  tail -3 gpurun_out/ncu_${NCU_CFG}.log
fi
