#!/bin/bash
# Initial-task chunk size on the HBM-sized configs (measured 1 best on C2): C5 k4 1/16 (tau 100, 1 GB), C4 prism/w5 1/64.
export PYTHONPATH=$PWD
mkdir -p gpurun_out
{
for ch in 1 4 16 64; do
  echo "== chunk $ch"
  CHUNK=$ch TAU=100 timeout 900 python scripts/variant_time.py 5 k4 1 16 1024
  CHUNK=$ch TAU=1 timeout 900 python scripts/variant_time.py 4 prism,w5 1 64 1024
done
} > gpurun_out/chunk_r02z.log 2>&1
grep -v "^lib" gpurun_out/chunk_r02z.log
