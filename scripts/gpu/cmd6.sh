python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider > gpurun_out/t7.log 2>&1; tail -1 gpurun_out/t7.log
for c in web_40m_2200m sbm_1m_20m rmat_4m_70m road_50m_110m; do
  python bench.py --config $c --steps 10 --warmup 3 > gpurun_out/r2_bench_$c.json 2> gpurun_out/r2_bench_$c.err; tail -c 300 gpurun_out/r2_bench_$c.err
  ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r2_launches_$c.csv python scripts/profile_run.py --config $c --runs 1 > /dev/null 2>&1
done
ls -la gpurun_out/r2_*
