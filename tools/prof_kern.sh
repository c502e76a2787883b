#!/bin/bash
# full ncu capture (source-level) of selected kernels of one C4 bench step
# usage: tools/prof_kern.sh <tag> <regex> <count>
mkdir -p gpurun_out
BENCH="python bench.py --config 4 --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline"
timeout -s KILL 900 ncu --set full --clock-control none --import-source on -k "regex:$2" -c $3 -o gpurun_out/prof_$1 -f $BENCH > gpurun_out/prof_$1.log 2>&1
ls -la gpurun_out | tail -3
