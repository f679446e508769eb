# A/B of L2 cache-policy variants: bench (web, 10 steps) + ncu DRAM bytes of the warp-bin k_warp per sweep
for v in ${VARIANTS:-base s3 g1 s3g1 g2 s3g2}; do
  NULPA_LIB=libs_ab/libnulpa_$v.so python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ab_$v.json 2>/dev/null
  python -c "
import json
d=json.loads(open('gpurun_out/ab_$v.json').read().strip().splitlines()[-1])
r=d['roofline']
print('$v', round(d['value']/1e9,2), 'G e/s', round(d['ms_per_step'],2), 'ms', 'frac', r['frac'], [ (p['ms'], p['frac']) for p in r['per_sweep']], 'Q', d['modularity_runs'])"
  NULPA_LIB=libs_ab/libnulpa_$v.so timeout 600 ncu --kernel-name-base mangled -k regex:k_warpILb0ELb1ELi512 -c 2 --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,smsp__inst_executed.sum --csv python scripts/profile_run.py --runs 1 > gpurun_out/ab_ncu_$v.csv 2>/dev/null
  python - <<PY
import csv,io
rows=[r for r in csv.reader(io.StringIO(open('gpurun_out/ab_ncu_$v.csv').read())) if len(r)>10]
h=rows[0]; im=h.index('Metric Name'); iv=h.index('Metric Value'); iid=h.index('ID')
d={}
for r in rows[1:]: d.setdefault(r[iid],{})[r[im]]=r[iv]
for k,m in d.items(): print('  $v sweep',k,{kk.split('__')[1][:22]:vv for kk,vv in m.items()})
PY
done
