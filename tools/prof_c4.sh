#!/bin/bash
mkdir -p gpurun_out
BENCH="python bench.py --config 4 --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline"
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:k_heavy$|k_expand|k_part_count|k_part_write|k_pieces|k_rows|k_place|k_dense_accum" -c 10 -o gpurun_out/prof_c4v4 -f $BENCH > gpurun_out/prof_c4v4.log 2>&1
ls -la gpurun_out
