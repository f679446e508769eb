# Round-2 session-2 measurement campaign: bench lines (all BASELINE configs), ncu launch lists of the bench
# command, DRAM traffic per sweep of the dominant bins (traffic.json).
set -x
TAG=${TAG:-r2s2}
for c in web_40m_2200m sbm_1m_20m rmat_4m_70m road_50m_110m; do
  python bench.py --config $c > gpurun_out/${TAG}_bench_$c.json 2> gpurun_out/${TAG}_bench_$c.err
  tail -c 400 gpurun_out/${TAG}_bench_$c.json
done
for c in web_40m_2200m sbm_1m_20m rmat_4m_70m road_50m_110m; do
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches_$c.csv \
     python bench.py --config $c --steps 2 --warmup 1 --no-e2e --no-cpu-baseline --quality-runs 0 > gpurun_out/${TAG}_ncu_$c.log 2>&1
  timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/${TAG}_traffic_$c.csv \
     python scripts/profile_run.py --config $c --runs 1 > gpurun_out/${TAG}_trafficrun_$c.log 2>&1
done
ls -la gpurun_out/ | tail -30
