#!/bin/bash
# C5 k4 (1/16 shard, tau 100 ms): ncu application-replay capture (kernel replay of the 2.7 s persistent launch with
# its multi-GB working set timed out in r02q) -- source counters, warp states, memory workload, speed of light.
export PYTHONPATH=$PWD
mkdir -p gpurun_out
timeout 1800 ncu --replay-mode application --section SourceCounters --section WarpStateStats --section MemoryWorkloadAnalysis \
  --section SpeedOfLight --section LaunchStats --section Occupancy --clock-control none --import-source on \
  -k regex:tdfs_kernel -s 1 -c 1 -o gpurun_out/app_r02r_c5_k4 -f \
  python bench.py --config 5 --profile-shard-world 16 --steps 1 --warmup 0 --no-cpu-baseline --no-e2e --also-degree-order 0 \
  --queries k4 > gpurun_out/app_r02r_c5_k4.out 2>&1; echo "c5 capture rc=$?"
tail -3 gpurun_out/app_r02r_c5_k4.out
