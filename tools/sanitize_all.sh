#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck of tools/sanitize_run.py on C1 and T_head (under gpurun)
# (round 2, second session: compute-sanitizer is closed on the GPU pool -- "runs under it have left GPUs
#  needing a reset" -- so the new paths are checked by the plain run's map identities only; r4_sanitizer_* cover the
#  code before them)
mkdir -p gpurun_out/san
for c in C1 T_head; do
  python tools/sanitize_run.py $c 3 > gpurun_out/san/plain_$c.txt 2>&1; echo "plain $c rc=$?"; tail -1 gpurun_out/san/plain_$c.txt
  for t in memcheck racecheck synccheck; do
    timeout 1500 compute-sanitizer --tool $t --print-limit 20 python tools/sanitize_run.py $c 3 > gpurun_out/san/r5_sanitizer_${t}_$c.txt 2>&1
    echo "$t $c rc=$?"; tail -2 gpurun_out/san/r5_sanitizer_${t}_$c.txt
  done
done
