TAG=${TAG:-r2s2d}
for c in web_40m_2200m sbm_1m_20m rmat_4m_70m road_50m_110m kmer_171m_360m; do
  python bench.py --config $c > gpurun_out/${TAG}_bench_$c.json 2> gpurun_out/${TAG}_bench_$c.err
  tail -c 200 gpurun_out/${TAG}_bench_$c.err
done
for c in web_40m_2200m sbm_1m_20m rmat_4m_70m road_50m_110m kmer_171m_360m; do
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches_$c.csv \
     python bench.py --config $c --steps 2 --warmup 1 --no-e2e --no-cpu-baseline --quality-runs 0 > /dev/null 2>&1
  timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/${TAG}_traffic_$c.csv \
     python scripts/profile_run.py --config $c --runs 1 > /dev/null 2>&1
done
( time python -m pytest tests -q -m gpu -p no:cacheprovider > gpurun_out/${TAG}_gputests.log 2>&1 ) 2> gpurun_out/${TAG}_gputests.time
tail -2 gpurun_out/${TAG}_gputests.log
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
