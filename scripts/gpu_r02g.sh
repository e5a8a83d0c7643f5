#!/bin/bash
# Multi-GPU shard imbalance (8 shards run one after another on one GPU, both partitions), the tau
# sweep on config 3 (Tables II/III) and E10 (paged vs array stacks) on configs 3/4.
export PYTHONPATH=$PWD
P=scripts/configs_probe.py
timeout 1200 python $P 4 prism,w5 8 0,1,2,3,4,5,6,7 0 > gpurun_out/imb_c4_rr.log 2>&1; tail -4 gpurun_out/imb_c4_rr.log
timeout 1200 python $P 4 prism,w5 8 0,1,2,3,4,5,6,7 1 > gpurun_out/imb_c4_db.log 2>&1; tail -4 gpurun_out/imb_c4_db.log
timeout 900 python $P 5 k4 8 0,1,2,3,4,5,6,7 0 > gpurun_out/imb_c5_rr.log 2>&1; tail -2 gpurun_out/imb_c5_rr.log
timeout 900 python $P 5 k4 8 0,1,2,3,4,5,6,7 1 > gpurun_out/imb_c5_db.log 2>&1; tail -2 gpurun_out/imb_c5_db.log
for tau in 1 10 100 1000 -1; do
  timeout 900 python $P 3 house,c5 64 0 0 $tau 0 stats > gpurun_out/tau_c3_$tau.log 2>&1; grep "shard" gpurun_out/tau_c3_$tau.log
done
timeout 900 python $P 3 house,c5 64 0 0 10 128 > gpurun_out/e10_c3_array.log 2>&1; grep shard gpurun_out/e10_c3_array.log
timeout 900 python $P 4 prism,w5 64 0 0 10 128 > gpurun_out/e10_c4_array.log 2>&1; grep shard gpurun_out/e10_c4_array.log
timeout 900 python $P 4 prism,w5 64 0 0 10 0 > gpurun_out/e10_c4_paged.log 2>&1; grep shard gpurun_out/e10_c4_paged.log
