#!/bin/bash
# tests + C4 bench/launch list for the default and an experimental env setting ($EXP)
mkdir -p gpurun_out
timeout -s KILL 420 python -m pytest tests -x -q -m gpu --timeout 150 > gpurun_out/pytest.txt 2>&1; tail -2 gpurun_out/pytest.txt
B="python bench.py --config 4 --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 0"
timeout -s KILL 200 $B > gpurun_out/bench_c4.json 2> gpurun_out/bench_c4.err; tail -2 gpurun_out/bench_c4.err
timeout -s KILL 200 env $EXP $B > gpurun_out/bench_c4x.json 2> gpurun_out/bench_c4x.err; tail -2 gpurun_out/bench_c4x.err
python tools/show_bench.py gpurun_out/bench_c4.json gpurun_out/bench_c4x.json
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum
timeout -s KILL 300 ncu --metrics $M --clock-control none --csv --log-file gpurun_out/launches_c4.csv python bench.py --config 4 --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
timeout -s KILL 300 env $EXP ncu --metrics $M --clock-control none --csv --log-file gpurun_out/launches_c4x.csv python bench.py --config 4 --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
python tools/launches.py gpurun_out/launches_c4.csv 0.3 | tail -22
python tools/launches.py gpurun_out/launches_c4x.csv 0.3 | tail -22
