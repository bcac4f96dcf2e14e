#!/bin/bash
# Round-2 checkpoint on B200: smoke, full GPU suite, bench all configs (C3 default),
# ncu launch list of the default bench and full captures of the top kernels.
O=gpurun_out/r2p
mkdir -p $O
export SPTRSV_GEN_CACHE=/tmp/gencache
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
timeout 2400 python -m pytest tests -m gpu -q -x > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -4 $O/pytest_gpu.log
summ() { python - "$1" <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith("{"):
        d=json.loads(l); print(sys.argv[1].split('/')[-1], "GFLOPS=%.3f ms=%.4f pre=%.1f frac=%.4f" % (d["value"], d["ms_per_step"], d.get("preprocess_ms",-1), d["roofline"]["frac"]), d["roofline"].get("kernel"), {k: round(v,4) for k,v in d.get("segment_ms",{}).items()}, "err", d.get("parity",{}).get("rel_err"), "e2e", d.get("e2e",{}).get("value"))
PY
}
for c in C3 C1 C2 C4 C5; do steps=20; [ $c = C5 ] && steps=5
timeout 900 python bench.py --config $c --steps $steps --warmup 3 --cpu-seconds 5 > $O/bench_$c.log 2>&1; echo "$c rc=$?"; summ $O/bench_$c.log; done
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > $O/bench_ref.log 2>&1; echo "ref rc=$?"; tail -c 600 $O/bench_ref.log
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file $O/launches_C3.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > $O/ncu_launch.log 2>&1; echo "ncu launches rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:tri_sf_mixed -c 1 -o $O/prof_C3_sf -f python scripts/prof_solve.py --config C3 --reps 1 > $O/ncu_c3.log 2>&1; echo "ncu c3 rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sq_ -c 2 -o $O/prof_C3_sq -f python scripts/prof_solve.py --config C3 --reps 1 > $O/ncu_c3sq.log 2>&1; echo "ncu c3 sq rc=$?"
