#!/bin/bash
# A/B timing of variants on one workload: tools/ab.sh <tag> <config> "<name> <env...>" ...
# each variant: bench.py (10 steps, no e2e / cpu leg) with the given environment
TAG=$1; CFG=$2; shift 2
mkdir -p gpurun_out
for v in "$@"; do
  read -r name envs <<< "$v"
  env $envs timeout -s KILL 600 python bench.py --config $CFG --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline \
    > gpurun_out/${TAG}_$name.json 2> gpurun_out/${TAG}_$name.err
  python - gpurun_out/${TAG}_$name.json "$name" <<'PY'
import json, sys
try:
    d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    lv = " ".join("L%d %.2f(%.2f)" % (x["level"], x["ms"], x["construction_ms"]) for x in d["levels"])
    print("%-14s %8.3f ms  %s" % (sys.argv[2], d["ms_per_step"], lv))
except Exception as e:
    print(sys.argv[2], "FAILED", e)
PY
done
