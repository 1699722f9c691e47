#!/bin/bash
# Exploratory GPU session: coop-launch micro, a C3 bench line, ncu --set full of one C3 batch with
# per-kernel source hot spots (summarised on the box).  Usage: bash tools/explore.sh <tag> [what...]
set -u
TAG=${1:-x}
shift || true
WHAT=${*:-"build micro bench src"}
OUT=gpurun_out
mkdir -p $OUT/x_$TAG
for w in $WHAT; do
  case $w in
    build) timeout 600 python -c "import __graft_entry__ as g; g.build()" > $OUT/x_$TAG/build.log 2>&1; echo "build rc=$?" ;;
    micro)
      nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/coop tools/micro/coop_launch.cu && timeout 120 /tmp/coop > $OUT/x_$TAG/coop.txt 2>&1
      echo "micro rc=$?"; cat $OUT/x_$TAG/coop.txt ;;
    bench)
      timeout 900 python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-baseline > $OUT/x_$TAG/bench.log 2>&1; echo "bench rc=$?"
      python -c "
import json,sys
l=[x for x in open('$OUT/x_$TAG/bench.log') if x.startswith('{')][-1]; d=json.loads(l)
print('value',d['value'],'ms_per_am',d.get('ms_per_am'),'e2e',d['e2e'].get('ms_per_am'))
print('full_scan', d.get('full_scan_roofline'))
for k,v in d.get('kernels',{}).items(): print(' ',k,round(v['ms_per_am']*1e3,3),round(v['share'],3))
" ;;
    src)
      C=${SRC_CONFIG:-C3}
      timeout 1200 ncu --set full --clock-control none --import-source on -k regex:bk_ -s 26 -c 13 \
        -o $OUT/x_$TAG/prof_$C -f python bench.py --config $C --steps 4 --warmup 3 --lanes 1 --no-cpu-baseline \
        --no-baseline --e2e-steps 1 --no-full-scan > $OUT/x_$TAG/src_$C.log 2>&1
      echo "src rc=$?"
      for k in ${SRC_KERNELS:-bk_cones bk_rows bk_map bk_voxels bk_band bk_bricks}; do
        for id in 0 1 2; do
          python tools/ncu_src.py $OUT/x_$TAG/prof_$C.ncu-rep 45 -k regex:$k --launch-skip $id --launch-count 1 > $OUT/x_$TAG/src_${C}_${k}_$id.txt 2>&1
        done
      done
      ncu -i $OUT/x_$TAG/prof_$C.ncu-rep --page details --csv > $OUT/x_$TAG/details_$C.csv 2>/dev/null
      gzip -f $OUT/x_$TAG/details_$C.csv
      rm -f $OUT/x_$TAG/prof_$C.ncu-rep ;;
  esac
done
# (more legs: tests = all GPU tests; benchfs = C3 line with the full-scan leg; others = C2/C4/C5 lines)
for w in $WHAT; do
  case $w in
    tests) timeout 1500 python -m pytest tests -m gpu -x -q > $OUT/x_$TAG/tests.log 2>&1; echo "tests rc=$?"; tail -3 $OUT/x_$TAG/tests.log ;;
    benchfs)
      timeout 900 python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-baseline > $OUT/x_$TAG/benchfs.log 2>&1; echo "benchfs rc=$?"
      python -c "
import json
l=[x for x in open('$OUT/x_$TAG/benchfs.log') if x.startswith('{')][-1]; d=json.loads(l)
print('value',d['value'],'ms_per_am',d.get('ms_per_am'),'e2e',d['e2e'].get('ms_per_am'))
print('full_scan', d.get('full_scan_roofline'))
for k,v in d.get('kernels',{}).items(): print(' ',k,round(v['ms_per_am']*1e3,3),round(v['share'],3))
" ;;
    others)
      for c in C2 C4 C5; do
        timeout 600 python bench.py --config $c --steps 20 --warmup 3 --no-cpu-baseline --no-baseline --no-full-scan > $OUT/x_$TAG/bench_$c.log 2>&1
        python -c "
import json
l=[x for x in open('$OUT/x_$TAG/bench_$c.log') if x.startswith('{')][-1]; d=json.loads(l)
print('$c','ms_per_am',d.get('ms_per_am'),'e2e',d['e2e'].get('ms_per_am'))"
      done ;;
  esac
done
