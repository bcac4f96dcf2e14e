#!/bin/bash
# Round-2 evidence (second pass; ncu reports summarised on the box, not copied back):
# every config's bench line, the oracle arm, solve-kernel launch lists, full ncu
# captures of each config's dominant kernel.
O=gpurun_out/r2final2
mkdir -p $O
export SPTRSV_GEN_CACHE=/tmp/gencache
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
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
for c in C1 C2 C3 C4 C5; do
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k "regex:tri_|sq_|perm_" -c 300 --csv --log-file $O/launches_$c.csv python scripts/prof_solve.py --config $c --reps 3 $( [ $c = C5 ] && echo "--nrhs 512" ) > $O/ncu_launch_$c.log 2>&1; echo "launches $c rc=$?"
done
cap() {  # cap <cfg> <kernel regex> <impl key> [extra prof_solve args]
  local c=$1 k=$2 key=$3; shift 3
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$k -c 1 -o /tmp/prof_$c -f python scripts/prof_solve.py --config $c --reps 1 "$@" > $O/ncu_$c.log 2>&1; echo "ncu $c rc=$?"
  python scripts/ncu_summary.py --launches $O/launches_$c.csv --rep /tmp/prof_$c.ncu-rep --out $O/r02_${c} --impl "$key" --json $O/ncu_summary.json --title "$c (round 2 final)" > /dev/null 2>&1; echo "summary $c rc=$?"
  ncu -i /tmp/prof_$c.ncu-rep --page source --csv --print-source sass > /tmp/src_$c.csv 2>/dev/null
  python scripts/sass_hot.py /tmp/src_$c.csv > $O/r02_${c}_sass_hot.md 2>/dev/null; rm -f /tmp/src_$c.csv
  rm -f /tmp/prof_$c.ncu-rep
}
cap C1 tri_chain C1:TRI_CHAIN
cap C2 tri_wave C2:TRI_PIPE
cap C3 tri_sf_mixed C3:TRI_SYNCFREE
cap C4 tri_supernode C4:TRI_SUPERNODE
cap C5 sq_multi C5:SQ_SPMM --nrhs 512
