#!/bin/bash
# Session-3 baseline evidence: default bench line, then profile_round (launch list, per-query ncu --set full, L2 peak)
export PYTHONPATH=$PWD
mkdir -p gpurun_out
timeout 900 python bench.py > gpurun_out/bench_r02l.json 2> gpurun_out/bench_r02l.err; echo "bench rc=$?"
tail -c 600 gpurun_out/bench_r02l.json
bash scripts/profile_round.sh r02l 2 triangle,c4,diamond,tailed_triangle,k4
