#!/bin/bash
# quick cycle: GPU parity tests, C3/C4 bench lines, C4 launch list (each step bounded)
mkdir -p gpurun_out
timeout -s KILL 420 python -m pytest tests -x -q -m gpu --timeout 150 > gpurun_out/pytest.txt 2>&1; tail -2 gpurun_out/pytest.txt
for c in 3 4; do timeout -s KILL 200 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/bench_c$c.json 2> gpurun_out/bench_c$c.err; tail -3 gpurun_out/bench_c$c.err; done
python tools/show_bench.py gpurun_out/bench_c3.json gpurun_out/bench_c4.json
HEC_PIECE_STATS=1 timeout -s KILL 200 python bench.py --config 4 --steps 1 --warmup 0 --no-cpu-baseline --e2e-steps 0 2>&1 >/dev/null | grep pieces | head -3
timeout -s KILL 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum --clock-control none --csv --log-file gpurun_out/launches_c4.csv python bench.py --config 4 --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
python tools/launches.py gpurun_out/launches_c4.csv 0.3 | tail -22
