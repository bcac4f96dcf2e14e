#!/bin/bash
# Session check: transposed-solve + PCG tests, transposed and multi-RHS C4 bench lines
O=gpurun_out/r1end
mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
timeout 900 python -m pytest tests -m gpu -q -k "transpose or pcg or supernode_multi or (test_multi_rhs and SUPERNODE) or test_full_size_configs" > $O/pytest_new.log 2>&1; echo "pytest new rc=$?"; tail -2 $O/pytest_new.log
summ() { python - "$1" <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith("{"):
        d=json.loads(l); print(sys.argv[1].split('/')[-1], "GFLOPS=%.3f ms=%.4f pre=%.1f frac=%.4f" % (d["value"], d["ms_per_step"], d["preprocess_ms"], d["roofline"]["frac"]), d["roofline"].get("kernel"), {k: round(v,4) for k,v in d["segment_ms"].items()}, "err", d["parity"]["rel_err"], "e2e", round(d["e2e"]["ms_per_step"],3))
PY
}
for c in C2 C4; do
  timeout 600 python bench.py --config $c --transpose --steps 20 --warmup 3 --cpu-seconds 2 > $O/bench_${c}_T.log 2>&1; echo "bench $c T rc=$?"; summ $O/bench_${c}_T.log
done
for k in 16 64 256; do
  timeout 600 python bench.py --config C4 --nrhs $k --steps 10 --warmup 3 --cpu-seconds 2 > $O/bench_C4_k$k.log 2>&1; echo "bench C4 k=$k rc=$?"; summ $O/bench_C4_k$k.log
  SPTRSV_NO_SN_MULTI=1 timeout 600 python bench.py --config C4 --nrhs $k --steps 10 --warmup 3 --no-cpu-baseline > $O/bench_C4_k${k}_sf.log 2>&1; echo "bench C4 k=$k syncfree rc=$?"; summ $O/bench_C4_k${k}_sf.log
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tri_supernode_multi -s 1 -c 1 -o $O/prof_C4_k64 -f python scripts/prof_solve.py --config C4 --reps 2 --nrhs 64 > $O/ncu_C4_k64.log 2>&1; echo "ncu C4 k64 rc=$?"
ncu -i $O/prof_C4_k64.ncu-rep --page raw --csv > $O/prof_C4_k64_raw.csv 2>/dev/null
ncu -i $O/prof_C4_k64.ncu-rep --page details --csv > $O/prof_C4_k64_details.csv 2>/dev/null
timeout 300 python examples/ic0_pcg.py > $O/pcg.log 2>&1; echo "pcg rc=$?"; grep -v Warn $O/pcg.log | tail -4
