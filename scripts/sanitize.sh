#!/bin/bash
# compute-sanitizer over scripts/sanitize_cases.py, one tool at a time; logs in gpurun_out/.
export PYTHONPATH=$PWD
TAG=${1:-r02}
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1500 compute-sanitizer --tool $tool --target-processes all --print-limit 50 \
    --log-file gpurun_out/sanitize_${tool}_${TAG}.log python scripts/sanitize_cases.py \
    > gpurun_out/sanitize_${tool}_${TAG}.out 2>&1
  echo "$tool rc=$? $(tail -1 gpurun_out/sanitize_${tool}_${TAG}.out) $(grep -c 'ERROR SUMMARY' gpurun_out/sanitize_${tool}_${TAG}.log) $(grep 'ERROR SUMMARY' gpurun_out/sanitize_${tool}_${TAG}.log | tail -1)"
done
