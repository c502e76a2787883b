#!/bin/bash
# round-end: full GPU suite, smoke, default bench line, C4/C5 launch lists
mkdir -p gpurun_out
timeout -s KILL 1200 python -m pytest tests -q -m gpu --timeout 400 > gpurun_out/pytest_full.txt 2>&1; tail -3 gpurun_out/pytest_full.txt
timeout -s KILL 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.txt 2>&1; tail -2 gpurun_out/smoke.txt
timeout -s KILL 400 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; python tools/show_bench.py gpurun_out/bench_default.json 2>/dev/null | head -3
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum
timeout -s KILL 300 ncu --metrics $M --clock-control none --csv --log-file gpurun_out/launches_c4.csv python bench.py --config 4 --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
timeout -s KILL 600 ncu --metrics $M --clock-control none --csv --log-file gpurun_out/launches_c5.csv python bench.py --config 5 --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
ls gpurun_out | tail -3
