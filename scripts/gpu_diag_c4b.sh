#!/bin/bash
export PYTHONPATH=$PWD
P=scripts/configs_probe.py
timeout 300 python $P 4 prism 64 0 0 10 256 stats
timeout 300 python $P 4 prism 64 0 0 100 0 stats
timeout 300 python $P 4 prism 64 0 0 1 0 stats
timeout 300 python $P 4 prism 1 0 0 10 256 stats
timeout 300 python $P 4 prism 4096 0 0 10 0 stats
