#!/bin/bash
# C5 k4 on a 1/64 shard (0.5 s launch): ncu kernel replay with the speed-of-light, memory, warp-state and source
# sections (the --set full of a 1/16 shard timed out), and C4 prism on a 1/256 shard likewise.
export PYTHONPATH=$PWD
mkdir -p gpurun_out
timeout 1200 ncu --section SpeedOfLight --section MemoryWorkloadAnalysis --section WarpStateStats --section SourceCounters \
  --section LaunchStats --section Occupancy --clock-control none --import-source on -k regex:tdfs_kernel -s 1 -c 1 \
  -o gpurun_out/sec_r02ac_c5_k4 -f python bench.py --config 5 --profile-shard-world 64 --steps 1 --warmup 0 \
  --no-cpu-baseline --no-e2e --also-degree-order 0 --queries k4 > gpurun_out/sec_r02ac_c5_k4.out 2>&1; echo "c5 rc=$?"
timeout 1200 ncu --section SpeedOfLight --section MemoryWorkloadAnalysis --section WarpStateStats --section SourceCounters \
  --section LaunchStats --section Occupancy --clock-control none --import-source on -k regex:tdfs_kernel -s 1 -c 1 \
  -o gpurun_out/sec_r02ac_c4_prism -f python bench.py --config 4 --profile-shard-world 256 --steps 1 --warmup 0 \
  --no-cpu-baseline --no-e2e --also-degree-order 0 --queries prism > gpurun_out/sec_r02ac_c4_prism.out 2>&1; echo "c4 rc=$?"
