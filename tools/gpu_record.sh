#!/bin/bash
# record: full bench line (defaults), C4 launch list, full ncu capture of the top kernels
mkdir -p gpurun_out
timeout -s KILL 400 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; tail -2 gpurun_out/bench_default.err
python tools/show_bench.py gpurun_out/bench_default.json
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum
B="python bench.py --config 4 --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline"
timeout -s KILL 300 ncu --metrics $M --clock-control none --csv --log-file gpurun_out/launches_c4.csv $B > /dev/null 2>&1
timeout -s KILL 300 ncu --metrics $M --clock-control none --csv --log-file gpurun_out/launches_c3.csv python bench.py --config 3 --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
timeout -s KILL 900 ncu --set full --clock-control none --import-source on -k "regex:${RE:-k_hrank|k_expand2|k_part_write|k_place|k_heavy_seg|k_rbm|k_dense}" -c ${CNT:-9} -o gpurun_out/prof_${TAG:-rec} -f $B > gpurun_out/prof_${TAG:-rec}.log 2>&1
tail -2 gpurun_out/prof_${TAG:-rec}.log
ls -la gpurun_out | tail -5
