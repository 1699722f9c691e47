#!/bin/bash
# Sweep one AM_OPT_* over values on several configs through bench.py (under gpurun):
#   bash tools/opt_sweep.sh <tag> <NAME> "<values>" "<configs>" [extra bench args]
TAG=$1; NAME=$2; VALS=$3; CFGS=$4; shift 4
mkdir -p gpurun_out/sw_$TAG
for c in $CFGS; do for v in $VALS; do
  timeout 300 python bench.py --config $c --steps 30 --warmup 5 --no-cpu-baseline --no-baseline --no-full-scan \
    --e2e-steps 5 --opt $NAME=$v "$@" > gpurun_out/sw_$TAG/${c}_$v.log 2>&1
  python - "$c" "$v" "gpurun_out/sw_$TAG/${c}_$v.log" <<'PY'
import json, sys
c, v, f = sys.argv[1:]
try:
    d = json.loads([l for l in open(f) if l.startswith("{")][-1])
    st = d["detail"]["stats_mean_over_pivots"]
    ks = " ".join(f"{k}={1e3 * x['ms_per_am']:.2f}" for k, x in d["kernels"].items())
    print(f"{c} {v}: {1e3 * d['ms_per_am']:.2f} us/AM live={st['voxels_live']:.0f} streamed={st['voxels_streamed']:.0f} | {ks}", flush=True)
except Exception as e:
    print(c, v, "FAILED", e, open(f).read()[-600:])
PY
done; done
