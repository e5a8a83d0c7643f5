#!/bin/bash
# Final round-2 evidence on the committed kernel: GPU tests, C2 bench line, profile_round (launch list,
# ncu --set full of the five C2 launches, L2 stream + random-sector microbenchmark, summary), bench lines for
# configs 3-5 (per-config tau and hub budget).
export PYTHONPATH=$PWD
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_r02x.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_r02x.log
timeout 900 python bench.py > gpurun_out/bench_r02x.json 2> gpurun_out/bench_r02x.err; echo "bench rc=$?"
bash scripts/profile_round.sh r02x 2 triangle,c4,diamond,tailed_triangle,k4
cp gpurun_out/ncu_full_summary_r02x.json profiles/ncu_full_summary.json
timeout 900 python bench.py --steps 3 --warmup 3 > gpurun_out/bench_r02x2.json 2> gpurun_out/bench_r02x2.err; echo "bench2 rc=$?"
for c in 3 4 5; do
  timeout 1500 python bench.py --config $c --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/bench_r02x_config$c.json 2> gpurun_out/bench_r02x_config$c.err; echo "config $c rc=$?"
done
