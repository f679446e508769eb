for c in sbm_1m_20m road_50m_110m; do python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/b2_$c.json 2> gpurun_out/b2_$c.err; tail -c 300 gpurun_out/b2_$c.err; python -c "
import json
d=json.loads(open('gpurun_out/b2_$c.json').read().strip().splitlines()[-1])
r=d['roofline']
print('$c', round(d['value']/1e9,2), d['ms_per_step'], d['ms_per_step_instrumented'], d['iterations'], r['frac'], r['share_of_step'], d['gpu_launches'], d['clocks'])"; done
