#!/bin/bash
# tri_supernode_multi iteration: parity tests, C4 multi-RHS bench lines, one ncu capture
O=gpurun_out/${OUTDIR:-snm}
mkdir -p $O
timeout 900 python -m pytest tests -m gpu -q -k "supernode_multi or test_multi_rhs or test_supernodal or epoch or pipelined or layouts or full_size_c5" > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
summ() { python - "$1" <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith("{"):
        d=json.loads(l); print(sys.argv[1].split('/')[-1], "GFLOPS=%.3f ms=%.4f frac=%.4f" % (d["value"], d["ms_per_step"], d["roofline"]["frac"]), d["roofline"].get("kernel"), {k: round(v,4) for k,v in d["segment_ms"].items()}, "err", d["parity"]["rel_err"], "e2e", round(d["e2e"]["ms_per_step"],3))
PY
}
for k in 16 64 256; do
  timeout 600 python bench.py --config C4 --nrhs $k --steps 10 --warmup 3 --cpu-seconds 2 > $O/bench_C4_k$k.log 2>&1; echo "bench C4 k=$k rc=$?"; summ $O/bench_C4_k$k.log
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tri_supernode_multi -s 1 -c 1 -o $O/prof_C4_k64 -f python scripts/prof_solve.py --config C4 --reps 2 --nrhs 64 > $O/ncu_C4_k64.log 2>&1; echo "ncu C4 k64 rc=$?"
ncu -i $O/prof_C4_k64.ncu-rep --page raw --csv > $O/prof_C4_k64_raw.csv 2>/dev/null
ncu -i $O/prof_C4_k64.ncu-rep --page details --csv > $O/prof_C4_k64_details.csv 2>/dev/null
ncu -i $O/prof_C4_k64.ncu-rep --page source --csv --print-source sass > $O/src.csv 2>/dev/null; python scripts/sass_hot.py $O/src.csv > $O/sass_hot.md 2>/dev/null; rm -f $O/src.csv
