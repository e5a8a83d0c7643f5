#!/bin/bash
# Round evidence for profiles/: (1) launch list of a 1-step bench (every kernel, device time,
# cold-cache/serialised under ncu); (2) ncu --set full of the five timed matching launches.
#   profile_round.sh TAG
set -u
export PYTHONPATH=$PWD
TAG=${1:-r01}
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/launches_${TAG}.csv python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e \
  > gpurun_out/launches_${TAG}.out 2>&1
echo "launch list rc=$?"
# launches 0-4 of tdfs_kernel are the STATS runs (W); 5-9 the timed step
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:tdfs_kernel -s 5 -c 5 \
  -o gpurun_out/full_${TAG} -f python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e \
  > gpurun_out/full_${TAG}.out 2>&1
echo "full capture rc=$?"
