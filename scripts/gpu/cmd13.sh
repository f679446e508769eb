python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider > gpurun_out/t12.log 2>&1; tail -1 gpurun_out/t12.log; grep FAILED gpurun_out/t12.log | head
for c in rmat_4m_70m web_40m_2200m; do
  python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r2g_$c.json 2> gpurun_out/r2g_$c.err; tail -c 400 gpurun_out/r2g_$c.err
  python -c "
import json
d=json.loads(open('gpurun_out/r2g_$c.json').read().strip().splitlines()[-1])
print('$c', round(d['value']/1e9,2), d['iterations'], round(d['modularity'],4), d['roofline']['kernel'], d['roofline']['frac'], {k:(v['stream_span_ms_per_run'], v['kernel_ms_per_run_serial']) for k,v in d['bins'].items()})"
done
