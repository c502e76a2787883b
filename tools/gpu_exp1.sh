#!/bin/bash
mkdir -p gpurun_out
B="python bench.py --config 4 --steps 4 --warmup 3 --no-cpu-baseline --e2e-steps 0"
timeout -s KILL 200 env HEC_NO_RBM=1 $B > gpurun_out/bench_c4x.json 2> gpurun_out/bench_c4x.err; tail -2 gpurun_out/bench_c4x.err
python tools/show_bench.py gpurun_out/bench_c4x.json
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum
timeout -s KILL 300 env HEC_NO_RBM=1 ncu --metrics $M --clock-control none --csv --log-file gpurun_out/launches_c4x.csv python bench.py --config 4 --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
python tools/launches.py gpurun_out/launches_c4x.csv 0.3 | tail -16
