#!/bin/bash
# tests + C4 bench + full ncu capture of selected kernels ($RE, $CNT) with source
mkdir -p gpurun_out
timeout -s KILL 480 python -m pytest tests -x -q -m gpu --timeout 200 ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/pytest.txt 2>&1; tail -3 gpurun_out/pytest.txt
timeout -s KILL 200 python bench.py --config 4 --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/bench_c4.json 2> gpurun_out/bench_c4.err; tail -2 gpurun_out/bench_c4.err; python tools/show_bench.py gpurun_out/bench_c4.json
BENCH="python bench.py --config 4 --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline"
timeout -s KILL 600 ncu --set full --clock-control none --import-source on -k "regex:$RE" -c ${CNT:-2} -o gpurun_out/prof_${TAG:-x} -f $BENCH > gpurun_out/prof_${TAG:-x}.log 2>&1
tail -3 gpurun_out/prof_${TAG:-x}.log
ls -la gpurun_out | tail -4
