#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
for geo in "8,4,8,4" "16,2,8,4" "8,2,8,4" "4,4,8,4" "16,1,8,4" "8,4,2,4"; do
  SPTRSV_WAVE=$geo timeout 300 python bench.py --config C2 --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/bench_w.log 2>&1
  echo "geo $geo: $(grep '^{' gpurun_out/bench_w.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['ms_per_step'],4), {k:round(v,4) for k,v in d['segment_ms'].items()})")"
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tri_wave -s 2 -c 1 -o gpurun_out/prof_wave -f python scripts/prof_solve.py --config C2 --reps 2 > gpurun_out/ncu_wave.log 2>&1; echo "ncu rc=$?"
