#!/bin/bash
export PYTHONPATH=$PWD
mkdir -p gpurun_out
timeout 900 python bench.py --config 3 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_r02ab_config3.json 2> gpurun_out/bench_r02ab_config3.err; echo "config 3 rc=$?"
tail -c 300 gpurun_out/bench_r02ab_config3.err
