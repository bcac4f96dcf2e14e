#!/bin/bash
# full GPU parity suite, benches of all configs, ncu of the C2 chain kernel
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/smoke.log
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -8 gpurun_out/pytest_gpu.log
summ() { python - "$1" <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith("{"):
        d=json.loads(l); print("GFLOPS=%.3f ms=%.4f" % (d["value"], d["ms_per_step"]), {k: round(v,4) for k,v in d["segment_ms"].items()}, "err", d["parity"]["rel_err"])
PY
}
for c in C2 C3 C4 C5; do steps=20; [ $c = C5 ] && steps=5
timeout 600 python bench.py --config $c --steps $steps --warmup 3 --no-cpu-baseline > gpurun_out/bench_$c.log 2>&1; echo "$c rc=$?"; summ gpurun_out/bench_$c.log; done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tri_chain -s 2 -c 1 -o gpurun_out/prof_c2_v2 -f python scripts/prof_solve.py --config C2 --reps 3 > gpurun_out/ncu_c2.log 2>&1; echo "ncu c2 rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tri_supernode -c 1 -o gpurun_out/prof_c4_sn -f python scripts/prof_solve.py --config C4 --reps 1 > gpurun_out/ncu_c4.log 2>&1; echo "ncu c4 rc=$?"
