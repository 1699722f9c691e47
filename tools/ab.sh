#!/bin/bash
# A/B of library builds under variants/ (AM_LIBRARY override): ms per AM and per-kernel us per AM.
# Usage (under gpurun): bash tools/ab.sh "<bench args>" variants/libam_a.so variants/libam_b.so ...
ARGS=$1
shift
mkdir -p gpurun_out
for lib in "$@"; do
  tag=$(basename $lib .so)
  AM_LIBRARY=$lib timeout 300 python bench.py $ARGS --no-cpu-baseline --no-full-scan > gpurun_out/ab_$tag.log 2>&1
  python - "$tag" <<'PY'
import json, sys
tag = sys.argv[1]
try:
    d = json.loads(open(f"gpurun_out/ab_{tag}.log").read().strip().splitlines()[-1])
    ks = " ".join(f"{k}={1e3 * v['ms_per_am']:.2f}" for k, v in d["kernels"].items())
    st = d["detail"]["stats_mean_over_pivots"]
    print(f"{tag}: {1e3 * d['ms_per_am']:.2f} us/AM | {ks} | live={st['voxels_live']:.0f} streamed={st['voxels_streamed']:.0f} bricks={st['bricks_kept']:.0f}")
except Exception as e:
    print(tag, "FAILED", e, open(f"gpurun_out/ab_{tag}.log").read()[-800:])
PY
done
