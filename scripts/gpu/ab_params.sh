# bench.py --param sweeps: PSETS="name:key=v,key=v name2:..."  CONFIG=web_40m_2200m
for spec in $PSETS; do
  n=${spec%%:*}; ps=${spec#*:}; args=""
  if [ -n "$ps" ]; then for kv in ${ps//,/ }; do args="$args --param $kv"; done; fi
  python bench.py --config ${CONFIG:-web_40m_2200m} --steps 10 --warmup 3 --no-e2e --no-cpu-baseline $args > gpurun_out/abp_$n.json 2>gpurun_out/abp_$n.err
  python -c "
import json
d=json.loads(open('gpurun_out/abp_$n.json').read().strip().splitlines()[-1])
r=d['roofline']
print('$n', round(d['value']/1e9,2), 'G e/s', round(d['ms_per_step'],2), 'ms', r['kernel'], 'frac', r['frac'], [ (p['ms'], p['frac']) for p in r['per_sweep']], 'it', d['iterations'], 'Q', d['modularity_runs'], {k:v['kernel_ms_per_run_serial'] for k,v in d['bins'].items()})" 2>&1 | tail -1
done
