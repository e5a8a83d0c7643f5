#!/bin/bash
# Register-pressure refactor (warp context in shared memory): GPU tests, then variant timings
# (occupancy 12 vs 10 blocks/SM, L2 residency-hint builds) on configs 2, 4 (1/64 shard) and 5 (1/16 shard).
export PYTHONPATH=$PWD
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_r02m.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_r02m.log
REPS=3 bash scripts/variants.sh 2 triangle,c4,diamond,tailed_triangle,k4 base mb10 h1 h3 h7 h1mb10 > gpurun_out/var_c2_r02m.log 2>&1
for v in base mb10 h1 h3 h7; do
  d=/tmp/var_$v; echo "== $v"
  PYTHONPATH=$d:$PWD timeout 600 python scripts/variant_time.py 4 prism,w5 1 64
  PYTHONPATH=$d:$PWD timeout 600 python scripts/variant_time.py 5 k4 1 16
done > gpurun_out/var_c45_r02m.log 2>&1
cat gpurun_out/var_c2_r02m.log gpurun_out/var_c45_r02m.log
