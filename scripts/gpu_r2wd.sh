#!/bin/bash
# watchdog test alone, then the boundary file, then the tiny C1 bench
export SPTRSV_GEN_CACHE=/tmp/gencache
timeout 400 python -m pytest tests/test_gpu_boundary.py -q -x -k watchdog 2>&1 | tail -3
timeout 900 python -m pytest tests/test_gpu_boundary.py -q -x 2>&1 | tail -3
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "cluster or tiny" 2>&1 | tail -2
