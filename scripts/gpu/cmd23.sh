python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -x > gpurun_out/t19.log 2>&1; tail -1 gpurun_out/t19.log
for v in widewarp widetma; do for c in web_40m_2200m rmat_4m_70m; do
  NULPA_LIB=libs_ab/libnulpa_$v.so python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r2x_${c}_$v.json 2>&1
  python -c "
import json
d=json.loads(open('gpurun_out/r2x_${c}_$v.json').read().strip().splitlines()[-1])
print('$v $c', round(d['value']/1e9,2), round(d['ms_per_step'],3), round(d['modularity'],4), {k:(v['stream_span_ms_per_run'], v['kernel_ms_per_run_serial']) for k,v in d['bins'].items()})"
done; done
