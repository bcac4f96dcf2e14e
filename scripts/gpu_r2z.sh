#!/bin/bash
# fp64 supernodal SpTRSM product on the tensor cores (DMMA) vs DFMA
O=gpurun_out/r2z
mkdir -p $O
export SPTRSV_GEN_CACHE=/tmp/gencache
summ() { python - "$1" <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith("{"):
        d=json.loads(l); print(sys.argv[1].split('/')[-1], "ms=%.4f GFLOPS=%.1f" % (d["ms_per_step"], d["value"]), {k: round(v,3) for k,v in d.get("segment_ms",{}).items()}, "err", d["parity"]["rel_err"])
PY
}
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -x -k "supernode_multi or (multi_rhs and SUPERNODE) or full_size_c4" > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
for k in 16 64 256; do
timeout 600 python bench.py --config C4 --nrhs $k --steps 10 --warmup 3 --no-cpu-baseline > $O/bench_C4_k${k}_dmma.log 2>&1; echo "k=$k dmma rc=$?"; summ $O/bench_C4_k${k}_dmma.log
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tri_supernode_multi -c 1 -o $O/prof_C4_k64_dmma -f python scripts/prof_solve.py --config C4 --reps 1 --nrhs 64 > $O/ncu.log 2>&1; echo "ncu rc=$?"
SPTRSV_NVCC_FLAGS=-DSPTRSV_SNM_DMMA=0 python -c "import __graft_entry__ as g; g.build()" > $O/build0.log 2>&1; echo "build dfma rc=$?"
for k in 16 64 256; do
timeout 600 python bench.py --config C4 --nrhs $k --steps 10 --warmup 3 --no-cpu-baseline > $O/bench_C4_k${k}_dfma.log 2>&1; echo "k=$k dfma rc=$?"; summ $O/bench_C4_k${k}_dfma.log
done
