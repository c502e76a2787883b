#!/bin/bash
# The one GPU-box script (run from the repo root under gpurun):
#   tools/gpu.sh <tag> <step> [<step> ...]
# steps (each bounded by its own timeout; outputs land in gpurun_out/<tag>_*):
#   build                 make -j8 all (in case the .so is stale)
#   tests[=EXPR]          pytest -m gpu [-k EXPR]
#   smoke                 __graft_entry__.smoke()
#   bench[=CFG[:STEPS]]   bench.py --config CFG (default 4) JSON line
#   launches[=CFG]        ncu launch list (time + DRAM bytes per launch) of one bench step
#   full=REGEX:COUNT[:CFG]  ncu --set full capture of COUNT launches matching REGEX
#   sanitize              compute-sanitizer memcheck / racecheck / synccheck on small hierarchies
set -u
TAG=$1; shift
mkdir -p gpurun_out
O=gpurun_out/$TAG
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum
one_step() { echo "--steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline --prof-steps 0 --config $1"; }
for step in "$@"; do
  name=${step%%=*}; arg=""; [[ "$step" == *=* ]] && arg=${step#*=}
  echo "== $step"
  case $name in
    build) make -s -j8 all > ${O}_build.txt 2>&1; tail -3 ${O}_build.txt ;;
    tests)
      if [ -n "$arg" ]; then K=(-k "$arg"); else K=(); fi
      timeout -s KILL 1500 python -m pytest tests -q -m gpu --timeout 600 "${K[@]}" > ${O}_pytest.txt 2>&1
      tail -4 ${O}_pytest.txt ;;
    smoke) timeout -s KILL 300 python -c "import __graft_entry__ as g; g.smoke()" > ${O}_smoke.txt 2>&1; tail -2 ${O}_smoke.txt ;;
    bench)
      cfg=${arg%%:*}; cfg=${cfg:-4}; st=20; [[ "$arg" == *:* ]] && st=${arg#*:}
      timeout -s KILL 900 python bench.py --config $cfg --steps $st --warmup 3 > ${O}_bench_c$cfg.json 2> ${O}_bench_c$cfg.err
      python tools/show_bench.py ${O}_bench_c$cfg.json 2>&1 | head -30; tail -3 ${O}_bench_c$cfg.err ;;
    launches)
      # launches=CFG[:warm]  (warm: --cache-control none, caches as a real run leaves them)
      cfg=${arg%%:*}; cfg=${cfg:-4}; cc=all; sfx=""
      [[ "$arg" == *:warm ]] && { cc=none; sfx=_warm; }
      timeout -s KILL 900 ncu --metrics $M --clock-control none --cache-control $cc --csv \
        --log-file ${O}_launches_c$cfg$sfx.csv python bench.py $(one_step $cfg) > ${O}_launches_c$cfg$sfx.log 2>&1
      python tools/launches.py ${O}_launches_c$cfg$sfx.csv 2>/dev/null | head -25 ;;
    full)
      IFS=: read -r rx cnt cfg <<< "$arg"; cfg=${cfg:-4}
      timeout -s KILL 1200 ncu --set full --clock-control none --import-source on -k "regex:$rx" -c $cnt \
        -o ${O}_full -f python bench.py $(one_step $cfg) > ${O}_full.log 2>&1
      tail -2 ${O}_full.log ;;
    sanitize)
      for tool in memcheck racecheck synccheck; do
        timeout -s KILL 1200 compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 20 \
          python tools/sanitize_run.py > ${O}_sanitize_$tool.txt 2>&1
        echo "$tool rc=$?"; tail -3 ${O}_sanitize_$tool.txt
      done ;;
    *) echo "unknown step $step" ;;
  esac
done
