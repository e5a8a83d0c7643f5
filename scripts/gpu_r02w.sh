#!/bin/bash
# Stream A with two 16-byte groups per lane per round (8 hub-bitmap probes in flight, variant a2) vs base, on C2,
# C5 k4 (1/16 shard, tau 100, 1 GB bitmaps) and C4 prism/w5 (1/64, tau 1, 1 GB).
export PYTHONPATH=$PWD
mkdir -p gpurun_out
REPS=5 bash scripts/variants.sh 2 c4,diamond,tailed_triangle,k4,triangle base a2 > gpurun_out/var_c2_r02w.log 2>&1
grep -v "^lib" gpurun_out/var_c2_r02w.log
{
for v in base a2 base a2; do
  echo "== $v"
  TAU=100 PYTHONPATH=/tmp/var_$v:$PWD timeout 900 python scripts/variant_time.py 5 k4 1 16 1024
  TAU=1 PYTHONPATH=/tmp/var_$v:$PWD timeout 900 python scripts/variant_time.py 4 prism,w5 1 64 1024
done
} > gpurun_out/c45_r02w.log 2>&1
grep -v "^lib" gpurun_out/c45_r02w.log
