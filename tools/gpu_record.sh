#!/bin/bash
# record: full bench line (defaults), C2/C3 bench lines, C3/C4 launch lists, full ncu capture of the top kernels
mkdir -p gpurun_out
timeout -s KILL 400 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; tail -2 gpurun_out/bench_default.err
python tools/show_bench.py gpurun_out/bench_default.json
for c in 2 3; do timeout -s KILL 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_c$c.json 2> gpurun_out/bench_c$c.err; python tools/show_bench.py gpurun_out/bench_c$c.json | head -3; done
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum
B="python bench.py --config 4 --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline"
timeout -s KILL 300 ncu --metrics $M --clock-control none --csv --log-file gpurun_out/launches_c4.csv $B > /dev/null 2>&1
timeout -s KILL 300 ncu --metrics $M --clock-control none --csv --log-file gpurun_out/launches_c3.csv python bench.py --config 3 --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
timeout -s KILL 900 ncu --set full --clock-control none --import-source on -k "regex:${RE:-k_hrank|k_expand2|k_part_write|k_place|k_heavy_seg|k_dense_accum2}" -c ${CNT:-10} -o gpurun_out/prof_${TAG:-rec} -f $B > gpurun_out/prof_${TAG:-rec}.log 2>&1
tail -2 gpurun_out/prof_${TAG:-rec}.log
ls -la gpurun_out | tail -5
