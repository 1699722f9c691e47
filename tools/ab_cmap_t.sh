for t in 64 96 128 160; do
  timeout 300 python bench.py --steps 100 --no-cpu-baseline --no-full-scan --cmap-t $t > gpurun_out/abt_$t.log 2>&1
  python -c "
import json
d=json.loads(open('gpurun_out/abt_$t.log').read().strip().splitlines()[-1])
ks=' '.join(f\"{k}={1e3*v['ms_per_am']:.2f}\" for k,v in d['kernels'].items())
st=d['detail']['stats_mean_over_pivots']
print('T=$t', f\"{1e3*d['ms_per_am']:.2f}\", ks, 'live', st['voxels_live'], 'streamed', st['voxels_streamed'])"
done
