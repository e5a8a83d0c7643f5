#!/bin/bash
# Final sanity on the last commit: GPU test suite, smoke(), default bench line.
export PYTHONPATH=$PWD
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_r02v.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_r02v.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_r02v.log 2>&1; echo "smoke rc=$?"; tail -2 gpurun_out/smoke_r02v.log
timeout 900 python bench.py > gpurun_out/bench_r02v.json 2> gpurun_out/bench_r02v.err; echo "bench rc=$?"; tail -c 400 gpurun_out/bench_r02v.json
