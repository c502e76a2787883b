#!/bin/bash
# Run on the GPU box (gpurun): ncu launch list of one bench step + a full capture
# of the named kernels.  usage: tools/profile.sh <config> <tag> [kernel-regex] [count]
set -u
CFG=${1:-3}; TAG=${2:-run}; RE=${3:-"k_heavy|k_small|k_mid|k_bin|k_dense|k_seg_copy|k_tile"}; CNT=${4:-14}
mkdir -p gpurun_out
BENCH="python bench.py --config $CFG --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline"
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
    --log-file gpurun_out/launches_${TAG}.csv $BENCH > /dev/null 2> gpurun_out/launches_${TAG}.err
ncu --set full --clock-control none --import-source on -k "regex:${RE}" -c $CNT \
    -o gpurun_out/prof_${TAG} -f $BENCH > /dev/null 2> gpurun_out/prof_${TAG}.err
ls -la gpurun_out/
