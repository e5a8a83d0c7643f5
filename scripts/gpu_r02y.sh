#!/bin/bash
# The reference arm as the driver runs it (oracle on the host cores, bounded sample of config 2).
export PYTHONPATH=$PWD
mkdir -p gpurun_out
timeout 900 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/ref_r02y.json 2> gpurun_out/ref_r02y.err; echo "ref rc=$?"
cat gpurun_out/ref_r02y.json | head -c 1500
