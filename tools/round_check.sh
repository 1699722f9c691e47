#!/bin/bash
# Round-end evidence for one commit (under gpurun): GPU tests, smoke, bench C3 + C2/C4/C5,
# launch list of a short bench, ncu --set full of one batch's 12 batched launches.
# Usage: bash tools/round_check.sh <tag>
set -u
TAG=${1:-r2u}
OUT=gpurun_out
mkdir -p $OUT
timeout 600 python -c "import __graft_entry__ as g; g.build()" > $OUT/build_$TAG.log 2>&1; echo "build rc=$?"
timeout 1200 python -m pytest tests -m gpu -x -q > $OUT/tests_$TAG.log 2>&1; echo "tests rc=$?"; tail -3 $OUT/tests_$TAG.log
timeout 300 python __graft_entry__.py smoke > $OUT/smoke_$TAG.log 2>&1; echo "smoke rc=$?"; tail -2 $OUT/smoke_$TAG.log
timeout 900 python bench.py > $OUT/bench_$TAG.log 2>&1; echo "bench rc=$?"; tail -c 600 $OUT/bench_$TAG.log
for c in C2 C4 C5; do
  timeout 600 python bench.py --config $c --no-cpu-baseline > $OUT/bench_${TAG}_$c.log 2>&1; echo "bench $c rc=$?"
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file $OUT/launches_$TAG.csv python bench.py --steps 20 --warmup 3 > $OUT/launches_$TAG.log 2>&1
echo "launches rc=$?"
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:bk_ -s ${KSKIP:-24} -c 12 \
  -o $OUT/prof_$TAG -f python bench.py --steps 4 --warmup 3 --lanes 1 --no-cpu-baseline --e2e-steps 1 --no-full-scan \
  > $OUT/full_$TAG.log 2>&1
echo "full rc=$?"
