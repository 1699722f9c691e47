#!/bin/bash
# Round-end evidence for one commit (under gpurun): GPU tests, smoke, bench lines (C3 default, C2/C4/C5,
# toolpath reuse on C5/C4, voxel split, the reference arm), the launch list of the driver's bench
# command, ncu --set full of one batch's batched launches on C3/C2/C4/C5, and of the single-pivot
# kernel on C1/C3, the single-pivot latency per pivot.
# Usage: bash tools/round_check.sh <tag> [what...]   (what: build tests smoke bench others toolpath
#        voxel reference launches full latency sp; default all)
set -u
TAG=${1:-r4}
shift || true
WHAT=${*:-"build tests smoke bench others toolpath voxel reference launches full latency sp"}
OUT=gpurun_out
mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu,power.draw --format=csv > $OUT/gpu_$TAG.txt 2>&1
for w in $WHAT; do
  case $w in
    build) timeout 600 python -c "import __graft_entry__ as g; g.build()" > $OUT/build_$TAG.log 2>&1; echo "build rc=$?" ;;
    tests) timeout 1500 python -m pytest tests -m gpu -x -q -s > $OUT/tests_$TAG.log 2>&1; echo "tests rc=$?"; tail -2 $OUT/tests_$TAG.log ;;
    smoke) timeout 300 python __graft_entry__.py smoke > $OUT/smoke_$TAG.log 2>&1; echo "smoke rc=$?"; tail -1 $OUT/smoke_$TAG.log ;;
    bench) timeout 900 python bench.py --steps 20 --warmup 3 > $OUT/bench_$TAG.log 2>&1; echo "bench rc=$?"; tail -c 400 $OUT/bench_$TAG.log; echo ;;
    others)
      for c in C2 C4 C5; do
        S=20; [ "$c" = "C5" ] && S=64  # (C5: the whole 4096-pivot toolpath batch of BASELINE configs[4])
        timeout 600 python bench.py --config $c --steps $S --pivots 4096 --warmup 3 --no-cpu-baseline > $OUT/bench_${TAG}_$c.log 2>&1; echo "bench $c rc=$?"
      done ;;
    toolpath)
      for c in C5 C4 C3; do
        timeout 600 python bench.py --config $c --toolpath --pivots 4096 --steps 60 --warmup 3 --no-cpu-baseline --no-baseline --no-full-scan > $OUT/bench_${TAG}_toolpath_$c.log 2>&1; echo "toolpath $c rc=$?"
      done ;;
    voxel) timeout 600 python bench.py --split voxel --steps 20 --warmup 3 > $OUT/bench_${TAG}_voxel.log 2>&1; echo "voxel rc=$?" ;;
    reference) timeout 900 python bench.py --impl reference --steps 3 --warmup 3 --ref-seconds 30 > $OUT/bench_${TAG}_reference.log 2>&1; echo "reference rc=$?" ;;
    launches)
      timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
        --log-file $OUT/launches_$TAG.csv python bench.py --steps 20 --warmup 3 > $OUT/launches_$TAG.log 2>&1
      echo "launches rc=$?"
      mkdir -p $OUT/prof_summ; PROF_DIR=$OUT/prof_summ python tools/summarize_ncu.py $TAG C3 64 > /dev/null 2>&1
      gzip -f $OUT/launches_$TAG.csv ;;
    full)
      for c in C3 C2 C4 C5; do
        timeout 1200 ncu --set full --clock-control none --import-source on -k regex:bk_ -s ${KSKIP:-22} -c ${KCOUNT:-11} \
          -o $OUT/prof_${TAG}_$c -f python bench.py --config $c --steps 4 --warmup 3 --lanes 1 --no-cpu-baseline \
          --no-baseline --e2e-steps 1 --no-full-scan > $OUT/full_${TAG}_$c.log 2>&1
        echo "full $c rc=$?"
        # (summarised here: the reports would exceed what gpurun brings back)
        mkdir -p $OUT/prof_summ; [ -f $OUT/prof_summ/ncu_summary.json ] || cp profiles/ncu_summary.json $OUT/prof_summ/
        PROF_DIR=$OUT/prof_summ python tools/summarize_ncu.py ${TAG}_$c $c 64 > /dev/null 2>&1
        rm -f $OUT/prof_${TAG}_$c.ncu-rep
      done ;;
    latency)
      for c in C3 C1; do
        timeout 600 ncu --set full --clock-control none --import-source on -k regex:am_latency_kernel -s 4 -c 1 \
          -o $OUT/prof_${TAG}_lat_$c -f python tools/sp_one.py $c 2 > $OUT/lat_${TAG}_$c.log 2>&1
        echo "latency $c rc=$?"
        mkdir -p $OUT/prof_summ
        PROF_DIR=$OUT/prof_summ python tools/summarize_ncu.py ${TAG}_lat_$c $c 1 > /dev/null 2>&1
        python tools/ncu_src.py $OUT/prof_${TAG}_lat_$c.ncu-rep 40 > $OUT/prof_summ/${TAG}_lat_${c}_source_top.txt 2>&1
        [ "$c" = "C3" ] || rm -f $OUT/prof_${TAG}_lat_$c.ncu-rep
      done ;;
    sp)
      for c in C1 C2 C3 C5; do SP_PER_PIVOT=1 timeout 300 python tools/sp_sweep.py $c "" "OPT_DIAG=16"; done > $OUT/sp_$TAG.txt 2>&1
      echo "sp rc=$?"; grep median $OUT/sp_$TAG.txt ;;
  esac
done
