#!/bin/bash
# Round-2 final evidence at HEAD: smoke, full GPU suite, every config's bench
# line, the oracle arm, launch lists and the C3 / C2 / C4 captures (summarised on the box)
O=gpurun_out/r2final3
mkdir -p $O
export SPTRSV_GEN_CACHE=/tmp/gencache
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
timeout 2400 python -m pytest tests -m gpu -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 $O/pytest_gpu.log
summ() { python - "$1" <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith("{"):
        d=json.loads(l); print(sys.argv[1].split('/')[-1], "ms=%.4f GFLOPS=%.2f frac=%.4f" % (d["ms_per_step"], d["value"], d["roofline"]["frac"]), d["roofline"].get("kernel"), "pre=%.1f" % d["preprocess_ms"], "e2e=%.2f" % d["e2e"]["value"], "err", d["parity"]["rel_err"])
PY
}
for c in C3 C1 C2 C4 C5; do steps=20; [ $c = C5 ] && steps=5
timeout 900 python bench.py --config $c --steps $steps --warmup 3 --cpu-seconds 10 > $O/bench_$c.log 2>&1; echo "$c rc=$?"; summ $O/bench_$c.log; done
timeout 900 python bench.py --config C4 --nrhs 64 --steps 10 --warmup 3 --cpu-seconds 5 > $O/bench_C4_k64.log 2>&1; echo "C4 k64 rc=$?"; summ $O/bench_C4_k64.log
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > $O/bench_ref.log 2>&1; echo "ref rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k "regex:tri_|sq_|perm_" -c 300 --csv --log-file $O/launches_C3.csv python scripts/prof_solve.py --config C3 --reps 3 > $O/ncu_launch_C3.log 2>&1; echo "launches C3 rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:tri_sf_mixed -c 1 -o /tmp/prof_C3 -f python scripts/prof_solve.py --config C3 --reps 1 > $O/ncu_C3.log 2>&1; echo "ncu C3 rc=$?"
python scripts/ncu_summary.py --launches $O/launches_C3.csv --rep /tmp/prof_C3.ncu-rep --out $O/r02_C3 --impl C3:TRI_SYNCFREE --json $O/ncu_summary.json --title "C3 (round 2 final, depth 1, SF_LONG 64)" > /dev/null 2>&1; echo "summary rc=$?"
ncu -i /tmp/prof_C3.ncu-rep --page source --csv --print-source sass > /tmp/src_C3.csv 2>/dev/null
python scripts/sass_hot.py /tmp/src_C3.csv > $O/r02_C3_sass_hot.md 2>/dev/null; rm -f /tmp/prof_C3.ncu-rep /tmp/src_C3.csv
