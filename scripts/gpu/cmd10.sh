for v in consec:paper_conf_ipps_sahunk25_b200/libnulpa.so strided:libs_ab/libnulpa_strided.so w1:libs_ab/libnulpa_w1.so; do
  n=${v%%:*}; L=${v#*:}
  echo "== $n"; NULPA_LIB=$L python scripts/exp_thread_quality.py
  NULPA_LIB=$L python bench.py --config road_50m_110m --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r2e_road_$n.json 2>&1
  python -c "
import json
d=json.loads(open('gpurun_out/r2e_road_$n.json').read().strip().splitlines()[-1])
print('road', round(d['value']/1e9,2), d['iterations'], round(d['modularity'],4), d['roofline']['frac'])"
done
