#!/bin/bash
# Option sweep of one config through bench.py (under gpurun): us per AM and per-kernel us per AM.
# Usage: bash tools/sweep.sh <config> "<args A>" "<args B>" ...
CFG=$1
shift
mkdir -p gpurun_out
i=0
for args in "$@"; do
  i=$((i+1))
  log=gpurun_out/sweep_${CFG}_$i.log
  timeout 300 python bench.py --config $CFG $args --steps 100 --warmup 5 --e2e-steps 10 --no-cpu-baseline --no-full-scan > $log 2>&1
  python - "$log" "$args" <<'PY'
import json, sys
log, args = sys.argv[1], sys.argv[2]
try:
    d = json.loads(open(log).read().strip().splitlines()[-1])
    ks = " ".join(f"{k}={1e3 * v['ms_per_am']:.2f}" for k, v in d["kernels"].items())
    print(f"[{args}]: {1e3 * d['ms_per_am']:.2f} us/AM | {ks}")
except Exception as e:
    print(f"[{args}] FAILED", e, open(log).read()[-600:])
PY
done
