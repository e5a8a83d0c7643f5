#!/bin/bash
export PYTHONPATH=$PWD
P=scripts/configs_probe.py
for t in 1 3; do timeout 600 python $P 4 prism,w5 1 0 0 $t 0; done
timeout 600 python $P 5 k4 1 0 0 1 0
timeout 600 python $P 3 k5 1 0 0 1 0
