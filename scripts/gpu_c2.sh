#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
timeout 600 python -m pytest tests -m gpu -x -q -k "CHAIN or chain or C2 or C1 or adversarial" > gpurun_out/pytest_chain.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/pytest_chain.log
for w in ${WARPS:-auto 4 6 8 12}; do
 for eg in ${EGEOMS:-"2048,4096,4"}; do
  echo "== ell geom $eg warps $w"
  if [ "$w" != "auto" ]; then export SPTRSV_ELL_WARPS=$w; else unset SPTRSV_ELL_WARPS; fi
  SPTRSV_ELL_GEOM=$eg SPTRSV_TRACE=1 python scripts/prof_solve.py --config C2 --reps 2 2>&1 | grep trace | tail -1
  SPTRSV_ELL_GEOM=$eg python bench.py --config C2 --steps 20 --warmup 3 --no-cpu-baseline 2>&1 | python -c "import json,sys; d=json.loads([l for l in sys.stdin if l.startswith('{')][0]); print('GFLOPS %.2f ms %.3f' % (d['value'], d['ms_per_step']), d['segment_ms'])"
 done
done
