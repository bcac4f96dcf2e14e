#!/bin/bash
# Round-2 evidence on B200: smoke, full GPU suite, every config's bench line,
# the oracle arm, solve-kernel launch lists and full ncu captures of each
# config's dominant kernel, DMMA vs DFMA A/B of the supernodal SpTRSM.
O=gpurun_out/r2final
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
for c in C2 C3 C4 C5; do
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k "regex:tri_|sq_|perm_" -c 300 --csv --log-file $O/launches_$c.csv python scripts/prof_solve.py --config $c --reps 3 $( [ $c = C5 ] && echo "--nrhs 512" ) > $O/ncu_launch_$c.log 2>&1; echo "launches $c rc=$?"
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:tri_wave -c 1 -o $O/prof_C2 -f python scripts/prof_solve.py --config C2 --reps 1 > $O/ncu_C2.log 2>&1; echo "ncu C2 rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:tri_sf_mixed -c 1 -o $O/prof_C3 -f python scripts/prof_solve.py --config C3 --reps 1 > $O/ncu_C3.log 2>&1; echo "ncu C3 rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:tri_supernode -c 1 -o $O/prof_C4 -f python scripts/prof_solve.py --config C4 --reps 1 > $O/ncu_C4.log 2>&1; echo "ncu C4 rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sq_multi -s 1 -c 1 -o $O/prof_C5 -f python scripts/prof_solve.py --config C5 --nrhs 512 --reps 1 > $O/ncu_C5.log 2>&1; echo "ncu C5 rc=$?"
SPTRSV_NVCC_FLAGS=-DSPTRSV_SNM_DMMA=0 python -c "import __graft_entry__ as g; g.build()" > $O/build_dfma.log 2>&1; echo "build dfma rc=$?"
timeout 900 python bench.py --config C4 --nrhs 64 --steps 10 --warmup 3 --no-cpu-baseline > $O/bench_C4_k64_dfma.log 2>&1; echo "C4 k64 dfma rc=$?"; summ $O/bench_C4_k64_dfma.log
timeout 900 python bench.py --config C4 --nrhs 256 --steps 10 --warmup 3 --no-cpu-baseline > $O/bench_C4_k256_dfma.log 2>&1; echo "C4 k256 dfma rc=$?"; summ $O/bench_C4_k256_dfma.log
python -c "import __graft_entry__ as g; g.build()" > $O/build_default.log 2>&1
