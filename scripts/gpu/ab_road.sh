for v in $VARIANTS; do
  NULPA_LIB=libs_ab/libnulpa_$v.so python bench.py --config road_50m_110m --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/abr_$v.json 2>/dev/null
  python -c "
import json
d=json.loads(open('gpurun_out/abr_$v.json').read().strip().splitlines()[-1])
r=d['roofline']
print('$v', round(d['value']/1e9,2), 'G e/s', round(d['ms_per_step'],2), 'ms', 'frac', r['frac'], [ (p['ms'], p['frac']) for p in r['per_sweep']], 'it', d['iterations'], 'Q', d['modularity_runs'])" 2>&1 | tail -1
done
for v in $PARITY; do
  NULPA_LIB=libs_ab/libnulpa_$v.so timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider > gpurun_out/ab_parity_$v.log 2>&1; echo "parity $v: $(tail -1 gpurun_out/ab_parity_$v.log)"
  NULPA_LIB=libs_ab/libnulpa_$v.so timeout 900 python -m pytest tests/test_gpu_fullsize.py -x -q -p no:cacheprovider -k "social_and_road" > gpurun_out/ab_fs_$v.log 2>&1; echo "fullsize road/rmat $v: $(tail -1 gpurun_out/ab_fs_$v.log)"
done
