#!/bin/bash
# round-end checks: full GPU suite, smoke(), default bench line
mkdir -p gpurun_out
timeout -s KILL 900 python -m pytest tests -q -m gpu --timeout 300 > gpurun_out/pytest_full.txt 2>&1; tail -3 gpurun_out/pytest_full.txt
timeout -s KILL 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.txt 2>&1; tail -2 gpurun_out/smoke.txt
timeout -s KILL 400 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; tail -2 gpurun_out/bench_default.err
python tools/show_bench.py gpurun_out/bench_default.json
