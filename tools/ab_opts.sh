#!/bin/bash
# A/B of runtime options on one library build: ms per AM and per-kernel us per AM.
# Usage (under gpurun): bash tools/ab_opts.sh "<common bench args>" "<args A>" "<args B>" ...
ARGS=$1
shift
mkdir -p gpurun_out
k=0
for extra in "$@"; do
  tag=opt$k
  k=$((k + 1))
  timeout 300 python bench.py $ARGS $extra --no-cpu-baseline --no-full-scan > gpurun_out/ab_$tag.log 2>&1
  python - "$tag" "$extra" <<'PY'
import json, sys
tag, extra = sys.argv[1], sys.argv[2]
try:
    d = json.loads(open(f"gpurun_out/ab_{tag}.log").read().strip().splitlines()[-1])
    ks = " ".join(f"{k}={1e3 * v['ms_per_am']:.2f}" for k, v in d["kernels"].items())
    print(f"[{extra}]: {1e3 * d['ms_per_am']:.2f} us/AM | {ks}")
except Exception as e:
    print(extra, "FAILED", e, open(f"gpurun_out/ab_{tag}.log").read()[-800:])
PY
done
