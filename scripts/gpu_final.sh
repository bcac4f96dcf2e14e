#!/bin/bash
# Round-end measurement: smoke, GPU suite, bench of every config (with the
# oracle baseline), ncu launch lists and one full capture per config.
O=gpurun_out/${OUTDIR:-final}
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,driver_version --format=csv > $O/gpu.txt 2>&1
nproc > $O/nproc.txt
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
if [ -z "$NO_TESTS" ]; then
timeout 1500 python -m pytest tests -m gpu -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest_gpu.log
fi
for c in ${CONFIGS:-C2 C1 C3 C4 C5}; do
  steps=30; [ $c = C5 ] && steps=5
  timeout 900 python bench.py --config $c --steps $steps --warmup 3 > $O/bench_$c.log 2>&1; echo "bench $c rc=$?"
  grep '^{' $O/bench_$c.log | python -c "
import json,sys
d=json.loads(sys.stdin.read())
print('$c ms=%.4f GFLOPS=%.2f pre=%.1f' % (d['ms_per_step'], d['value'], d['preprocess_ms']), 'roof', d['roofline'].get('kernel'), round(d['roofline']['frac'],4))
"
done
if [ -z "$NO_NCU" ]; then
for c in ${NCU_CONFIGS:-C2 C3 C4 C5}; do
  steps=2; nr=""; [ $c = C5 ] && nr="--nrhs 512"
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_$c.csv python bench.py --config $c --steps 2 --warmup 3 --no-cpu-baseline > $O/ncu_launch_$c.log 2>&1; echo "ncu launches $c rc=$?"
  case $c in
    C2) K=tri_wave; S=1;; C3) K=tri_syncfree; S=0;; C4) K=tri_supernode; S=0;; C5) K=sq_multi; S=1;;
  esac
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$K -s $S -c 1 -o $O/prof_$c -f python scripts/prof_solve.py --config $c --reps 2 $nr > $O/ncu_$c.log 2>&1; echo "ncu full $c rc=$?"
  # summarise on the box (gpurun brings back <= 64 MiB): launch list, full-set
  # summary, DRAM bytes per launch; the .ncu-rep stays only if small
  IMPL=$c:$(python - "$c" <<'PY'
import sys
print({"C2": "TRI_PIPE", "C3": "TRI_SYNCFREE", "C4": "TRI_SUPERNODE", "C5": "SQ_SPMM"}[sys.argv[1]])
PY
)
  python scripts/ncu_summary.py --launches $O/launches_$c.csv --rep $O/prof_$c.ncu-rep --out $O/${TAG:-r01}_${c}_final --impl $IMPL --json $O/ncu_summary_part.json > /dev/null 2>&1; echo "summary $c rc=$?"
  ncu -i $O/prof_$c.ncu-rep --page source --csv --print-source sass > $O/src_$c.csv 2>/dev/null
  python scripts/sass_hot.py $O/src_$c.csv > $O/${TAG:-r01}_${c}_final_sass_hot.md 2>/dev/null; rm -f $O/src_$c.csv
  [ $(stat -c %s $O/prof_$c.ncu-rep 2>/dev/null || echo 0) -gt 12000000 ] && rm -f $O/prof_$c.ncu-rep
done
fi
ls $O
