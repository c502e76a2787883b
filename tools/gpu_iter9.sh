#!/bin/bash
# v9: parity (construct + full-size digests incl. C5), k_drank match-aggregation A/B on C5, C4 default bench, C5 launch list
mkdir -p gpurun_out
timeout -s KILL 900 python -m pytest tests -q -m gpu --timeout 400 -k "construct or full_size or hierarchy_c" > gpurun_out/pytest9.txt 2>&1; tail -3 gpurun_out/pytest9.txt
for agg in 1 0; do HEC_DRANK_AGG=$agg timeout -s KILL 600 python bench.py --config 5 --steps 5 --warmup 3 --e2e-steps 2 --no-cpu-baseline > gpurun_out/bench_c5_agg$agg.json 2> gpurun_out/bench_c5_agg$agg.err; tail -2 gpurun_out/bench_c5_agg$agg.err; python tools/show_bench.py gpurun_out/bench_c5_agg$agg.json 2>/dev/null| head -3; done
timeout -s KILL 400 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; tail -2 gpurun_out/bench_default.err
python tools/show_bench.py gpurun_out/bench_default.json 2>/dev/null | head -14
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum
timeout -s KILL 600 ncu --metrics $M --clock-control none --csv --log-file gpurun_out/launches_c5.csv python bench.py --config 5 --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
timeout -s KILL 300 ncu --metrics $M --clock-control none --csv --log-file gpurun_out/launches_c4.csv python bench.py --config 4 --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
ls gpurun_out | tail -3
