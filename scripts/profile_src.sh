#!/bin/bash
# Source-level ncu capture of the matching kernel for one query on a 1/W shard of config 2.
#   profile_src.sh TAG QUERY [W] [FLAGS]
set -u
export PYTHONPATH=$PWD
TAG=$1; Q=$2; W=${3:-16}; FL=${4:-0}
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:tdfs_kernel -s 1 -c 1 \
  -o gpurun_out/src_${TAG}_${Q} -f python bench.py --steps 1 --warmup 0 --queries $Q --no-cpu-baseline --no-e2e \
  --profile-shard-world $W --flags $FL > gpurun_out/src_${TAG}_${Q}.out 2>&1
echo "rc=$?"
