#!/bin/bash
# One GPU session: build, GPU tests, smoke, bench, ncu launch list + one full capture.
# Usage (from the repo root, under gpurun):  bash tools/gpu_check.sh [tag] [what...]
# what: build tests smoke bench launches full  (default: all)
set -u
TAG=${1:-r1}
shift || true
WHAT=${*:-"build tests smoke bench launches full"}
OUT=gpurun_out
mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu,power.draw --format=csv > $OUT/gpu_$TAG.txt 2>&1
for w in $WHAT; do
  case $w in
    build)
      timeout 600 python -c "import __graft_entry__ as g; g.build()" > $OUT/build_$TAG.log 2>&1; echo "build rc=$?" ;;
    tests)
      timeout 1500 python -m pytest tests -m gpu -x -q > $OUT/tests_$TAG.log 2>&1; echo "tests rc=$?"; tail -3 $OUT/tests_$TAG.log ;;
    smoke)
      timeout 600 python __graft_entry__.py smoke > $OUT/smoke_$TAG.log 2>&1; echo "smoke rc=$?"; tail -2 $OUT/smoke_$TAG.log ;;
    bench)
      timeout 900 python bench.py > $OUT/bench_$TAG.log 2>&1; echo "bench rc=$?"; tail -c 3000 $OUT/bench_$TAG.log ;;
    bench2)
      timeout 900 python bench.py --config C2 --baseline --no-cpu-baseline > $OUT/bench_c2_$TAG.log 2>&1; echo "bench2 rc=$?"; tail -c 2500 $OUT/bench_c2_$TAG.log ;;
    launches)
      # the default bench command, every launch (the driver's bench line comes from the same command)
      timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
        --log-file $OUT/launches_$TAG.csv python bench.py > $OUT/launches_$TAG.log 2>&1
      echo "launches rc=$?" ;;
    full)
      timeout 1200 ncu --set full --clock-control none --import-source on -k regex:${KREGEX:-filter_kernel} -s ${KSKIP:-5} -c ${KCOUNT:-1} \
        -o $OUT/prof_$TAG -f python bench.py --steps 8 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $OUT/full_$TAG.log 2>&1
      echo "full rc=$?" ;;
  esac
done
