#!/bin/bash
# test + bench C3/C4 + C4 launch list
mkdir -p gpurun_out
timeout 500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_ranges.py -x -q -m gpu > gpurun_out/pytest.txt 2>&1; tail -4 gpurun_out/pytest.txt
for c in 3 4; do timeout 200 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/bench_c$c.json 2> gpurun_out/bench_c$c.err; done
python tools/show_bench.py gpurun_out/bench_c3.json gpurun_out/bench_c4.json | grep -v "^   [a-z]\|e2e\|cpu None"
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches_c4p.csv python bench.py --config 4 --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
