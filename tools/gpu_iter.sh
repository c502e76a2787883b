#!/bin/bash
# iteration cycle: GPU parity tests (bounded), C3/C4 bench lines, C4 launch list
mkdir -p gpurun_out
timeout -s KILL 480 python -m pytest tests -x -q -m gpu --timeout 200 ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/pytest.txt 2>&1; tail -3 gpurun_out/pytest.txt
for c in ${CONFIGS:-4}; do timeout -s KILL 200 env $EXP python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/bench_c$c.json 2> gpurun_out/bench_c$c.err; tail -2 gpurun_out/bench_c$c.err; python tools/show_bench.py gpurun_out/bench_c$c.json; done
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum
timeout -s KILL 300 env $EXP ncu --metrics $M --clock-control none --csv --log-file gpurun_out/launches_c4.csv python bench.py --config 4 --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
python tools/launches.py gpurun_out/launches_c4.csv 0.3 | tail -18
