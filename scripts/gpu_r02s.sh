#!/bin/bash
# Hub-bitmap budget on the HBM-sized configs (round-1 verdict: tuned on C2 only): 256 MB (default) / 1 / 4 / 16 GB
# on C5 k4 (1/16 shard, tau 100), C4 prism + w5 (1/64 shard, tau 1), C3 k5 + house (1/64 shard); plus the new
# hub-graph c4 parity test.
export PYTHONPATH=$PWD
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "hub_bitmaps" > gpurun_out/pytest_r02s.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/pytest_r02s.log
{
for mb in 256 1024 4096 16384; do
  echo "== hub_mb $mb"
  TAU=100 timeout 900 python scripts/variant_time.py 5 k4 1 16 $mb
  TAU=1 timeout 900 python scripts/variant_time.py 4 prism,w5 1 64 $mb
  timeout 900 python scripts/variant_time.py 3 k5,c5 1 64 $mb
done
} > gpurun_out/hub_budget_r02s.log 2>&1
cat gpurun_out/hub_budget_r02s.log
