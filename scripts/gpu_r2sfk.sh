#!/bin/bash
# tri_sf_mixed compile-time knobs on C3 (depth 1 default): long-row threshold, piece size
export SPTRSV_GEN_CACHE=/tmp/gencache
for f in "" "-DSPTRSV_SF_LONG=16" "-DSPTRSV_SF_LONG=64" "-DSPTRSV_SF_NB=128" "-DSPTRSV_SF_NB=512"; do
  SPTRSV_NVCC_FLAGS="$f" python -c "import __graft_entry__ as g; g.build()" > /tmp/b.log 2>&1 || { echo "build '$f' failed"; tail -3 /tmp/b.log; continue; }
  echo "== flags '$f'"; timeout 600 python scripts/sweep_sf.py C3 2>&1 | tail -1
done
python -c "import __graft_entry__ as g; g.build()" > /tmp/b.log 2>&1
