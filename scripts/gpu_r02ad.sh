#!/bin/bash
# Leaf-stage capacity 512 (base) vs 1024 / 2048 ids per warp on C5 k4 (1/16, tau 100, 1 GB) and C2.
export PYTHONPATH=$PWD
mkdir -p gpurun_out
REPS=5 bash scripts/variants.sh 2 c4,diamond,tailed_triangle,k4,triangle base lf1024 lf2048 > gpurun_out/var_c2_r02ad.log 2>&1
grep -v "^lib" gpurun_out/var_c2_r02ad.log
{
for v in base lf1024 lf2048; do
  echo "== $v"; TAU=100 PYTHONPATH=/tmp/var_$v:$PWD timeout 900 python scripts/variant_time.py 5 k4 1 16 1024
done
} > gpurun_out/c5_r02ad.log 2>&1
grep -v "^lib" gpurun_out/c5_r02ad.log
