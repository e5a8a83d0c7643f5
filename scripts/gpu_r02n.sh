#!/bin/bash
# One DFS call site (kernel loop takes batch edges / queue tasks / chunks): old (HEAD~) vs new vs new at
# 10 blocks/SM on configs 2, 4 (1/64 shard), 5 (1/16 shard); then the GPU test suite on the new library.
export PYTHONPATH=$PWD
mkdir -p gpurun_out
REPS=5 bash scripts/variants.sh 2 triangle,c4,diamond,tailed_triangle,k4 old base mb10 > gpurun_out/var_c2_r02n.log 2>&1
for v in old base mb10; do
  d=/tmp/var_$v; echo "== $v"
  PYTHONPATH=$d:$PWD timeout 600 python scripts/variant_time.py 4 prism,w5 1 64
  PYTHONPATH=$d:$PWD timeout 600 python scripts/variant_time.py 5 k4 1 16
done > gpurun_out/var_c45_r02n.log 2>&1
cat gpurun_out/var_c2_r02n.log gpurun_out/var_c45_r02n.log | grep -v "^lib"
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_r02n.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_r02n.log
