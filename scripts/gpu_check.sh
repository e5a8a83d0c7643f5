#!/bin/bash
# One GPU round-trip: the -m gpu suite (all failures listed), then a bench line.
#   gpu_check.sh TAG [pytest -k expr]
export PYTHONPATH=$PWD
TAG=${1:-x}
K=${2:-}
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q ${K:+-k "$K"} --timeout 600 --timeout-method=thread -p no:cacheprovider 2>&1 \
  > gpurun_out/gputests_${TAG}.log
grep -E "^(FAILED|ERROR)|passed|failed" gpurun_out/gputests_${TAG}.log | tail -40
timeout 900 python bench.py --steps 3 --warmup 3 --no-cpu-baseline ${BENCH_ARGS:-} > gpurun_out/bench_${TAG}.json 2> gpurun_out/bench_${TAG}.err
tail -3 gpurun_out/bench_${TAG}.err
python - <<PY
import json
d = json.load(open("gpurun_out/bench_${TAG}.json"))
print("value %.4g  ms/step %.1f  frac %.3f  e2e %.4g" % (d["value"], d["ms_per_step"], d["roofline"]["frac"], (d["e2e"] or {}).get("value", 0)))
for k, v in d["config"]["per_query"].items():
    print("  %-16s %10.2f ms  %d" % (k, v["time_to_count_ms"], v["count"]))
PY
