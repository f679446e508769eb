python bench.py > gpurun_out/r2_bench_default.json 2> gpurun_out/r2_bench_default.err; tail -c 200 gpurun_out/r2_bench_default.err
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r2_launches_bench.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline --quality-runs 0 > gpurun_out/r2_launches_bench.log 2>&1
for c in sbm_1m_20m rmat_4m_70m road_50m_110m; do python bench.py --config $c > gpurun_out/r2_bench_$c.json 2> gpurun_out/r2_bench_$c.err; done
