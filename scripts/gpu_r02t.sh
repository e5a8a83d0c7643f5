#!/bin/bash
# Bench lines for configs 4 and 5 with the per-config hub-bitmap budget (1 GB) and tau.
export PYTHONPATH=$PWD
mkdir -p gpurun_out
for c in 5 4; do
  timeout 1500 python bench.py --config $c --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/bench_r02t_config$c.json 2> gpurun_out/bench_r02t_config$c.err; echo "config $c rc=$?"
  tail -c 300 gpurun_out/bench_r02t_config$c.err
done
