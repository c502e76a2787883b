#!/bin/bash
# v8 record: bench lines C2..C5 (C5 = one-GPU hierarchy of R-MAT s26 ef16), C4/C5 launch lists,
# and the raw pinned H2D bandwidth of the box (explains e2e)
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,pcie.link.gen.current,pcie.link.width.current --format=csv > gpurun_out/smi.txt
timeout -s KILL 120 python - > gpurun_out/h2d.txt 2>&1 <<'EOF'
import torch
for mb in (256, 2048):
    h = torch.empty(mb << 20, dtype=torch.uint8).pin_memory(); d = torch.empty_like(h, device="cuda")
    for _ in range(2): d.copy_(h, non_blocking=True)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize(); e0.record()
    for _ in range(5): d.copy_(h, non_blocking=True)
    e1.record(); torch.cuda.synchronize()
    print(f"h2d {mb} MB: {5 * h.numel() / (e0.elapsed_time(e1) / 1e3) / 1e9:.1f} GB/s")
EOF
cat gpurun_out/h2d.txt
for c in 2 3; do timeout -s KILL 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_c$c.json 2> gpurun_out/bench_c$c.err; python tools/show_bench.py gpurun_out/bench_c$c.json | head -3; done
timeout -s KILL 600 python bench.py --config 5 --steps 5 --warmup 3 --e2e-steps 1 --no-cpu-baseline > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err; tail -2 gpurun_out/bench_c5.err; python tools/show_bench.py gpurun_out/bench_c5.json | head -3
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum
timeout -s KILL 300 ncu --metrics $M --clock-control none --csv --log-file gpurun_out/launches_c4.csv python bench.py --config 4 --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
timeout -s KILL 600 ncu --metrics $M --clock-control none --csv --log-file gpurun_out/launches_c5.csv python bench.py --config 5 --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
ls -la gpurun_out | tail -8
