python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider > gpurun_out/t8.log 2>&1; tail -1 gpurun_out/t8.log
for c in sbm_1m_20m rmat_4m_70m road_50m_110m web_40m_2200m; do
  python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r2b_$c.json 2> gpurun_out/r2b_$c.err; tail -c 300 gpurun_out/r2b_$c.err
done
