#!/bin/bash
# Final round-2 evidence on the committed kernel: GPU tests, C2 bench line, profile_round (launch list,
# ncu --set full of the five C2 launches, L2 stream + random-sector microbenchmark, summary), bench lines for
# configs 3-5 (per-config tau), ncu --set full of C5 k4 (1/16 shard), C5 k4 rlr vs base at tau 100.
export PYTHONPATH=$PWD
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_r02p.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_r02p.log
timeout 900 python bench.py > gpurun_out/bench_r02p.json 2> gpurun_out/bench_r02p.err; echo "bench rc=$?"
bash scripts/profile_round.sh r02p 2 triangle,c4,diamond,tailed_triangle,k4
cp gpurun_out/ncu_full_summary_r02p.json profiles/ncu_full_summary.json
timeout 900 python bench.py --steps 3 --warmup 3 > gpurun_out/bench_r02p2.json 2> gpurun_out/bench_r02p2.err; echo "bench2 rc=$?"
for c in 3 4 5; do
  timeout 1500 python bench.py --config $c --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/bench_r02p_config$c.json 2> gpurun_out/bench_r02p_config$c.err; echo "config $c rc=$?"
done
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:tdfs_kernel -s 1 -c 1 \
  -o gpurun_out/full_r02p_c5_k4 -f python bench.py --config 5 --profile-shard-world 16 --steps 1 --warmup 0 \
  --no-cpu-baseline --no-e2e --queries k4 > gpurun_out/full_r02p_c5_k4.out 2>&1; echo "c5 capture rc=$?"
