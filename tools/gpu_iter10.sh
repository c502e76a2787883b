#!/bin/bash
# v10: direct-bin tests, C4/C5 bench lines, ncu --set full of the L1 k_drank launch of C5
mkdir -p gpurun_out
timeout -s KILL 600 python -m pytest tests -q -m gpu --timeout 300 -k "direct_bins or size_classes" > gpurun_out/pytest10.txt 2>&1; tail -2 gpurun_out/pytest10.txt
timeout -s KILL 400 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; python tools/show_bench.py gpurun_out/bench_default.json 2>/dev/null | head -3
timeout -s KILL 600 python bench.py --config 5 --steps 5 --warmup 3 --e2e-steps 2 --no-cpu-baseline > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err; python tools/show_bench.py gpurun_out/bench_c5.json 2>/dev/null| head -3
timeout -s KILL 900 ncu --set full --clock-control none --import-source on -k regex:k_drank -s 1 -c 1 -o gpurun_out/prof_drank_c5 -f python bench.py --config 5 --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline > gpurun_out/prof_drank.log 2>&1; tail -2 gpurun_out/prof_drank.log
