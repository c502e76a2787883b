#!/bin/bash
# v11: k_drank big-bins-first sweep: direct-bin/size-class tests, C5 full-size digest, C5 + C4 bench
mkdir -p gpurun_out
timeout -s KILL 600 python -m pytest tests -q -m gpu --timeout 400 -k "direct_bins or size_classes or full_size_digests" > gpurun_out/pytest11.txt 2>&1; tail -2 gpurun_out/pytest11.txt
timeout -s KILL 600 python bench.py --config 5 --steps 5 --warmup 3 --e2e-steps 1 --no-cpu-baseline > gpurun_out/bench_c5_v11.json 2> gpurun_out/bench_c5_v11.err; python tools/show_bench.py gpurun_out/bench_c5_v11.json 2>/dev/null| head -4
timeout -s KILL 400 python bench.py --e2e-steps 1 --no-cpu-baseline > gpurun_out/bench_c4_v11.json 2> gpurun_out/bench_c4_v11.err; python tools/show_bench.py gpurun_out/bench_c4_v11.json 2>/dev/null | head -3
