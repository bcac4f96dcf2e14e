#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
timeout 600 python -m pytest tests -m gpu -x -q -k "CHAIN or chain or C2 or smoke or adversarial" > gpurun_out/pytest_chain.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_chain.log
for geom in ${GEOMS:-"4,1024,2048,4096,256" "5,1024,2048,2048,256" "6,768,1536,2048,256"}; do
  echo "== geom $geom"
  SPTRSV_TRACE=1 SPTRSV_CHAIN_GEOM=$geom python scripts/prof_solve.py --config C2 --reps 2 2>&1 | grep trace | tail -2
  SPTRSV_CHAIN_GEOM=$geom python bench.py --config C2 --steps 20 --warmup 3 --no-cpu-baseline 2>&1 | python -c "import json,sys; d=json.loads([l for l in sys.stdin if l.startswith('{')][0]); print('GFLOPS %.2f ms %.3f' % (d['value'], d['ms_per_step']), d['segment_ms'])"
done
