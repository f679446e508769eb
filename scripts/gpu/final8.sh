TAG=r2s2h
for c in web_40m_2200m sbm_1m_20m rmat_4m_70m; do
  python bench.py --config $c > gpurun_out/${TAG}_bench_$c.json 2> gpurun_out/${TAG}_bench_$c.err
done
( time python -m pytest tests -q -m gpu -p no:cacheprovider > gpurun_out/${TAG}_gputests.log 2>&1 ) 2> gpurun_out/${TAG}_gputests.time
tail -1 gpurun_out/${TAG}_gputests.log
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/${TAG}_traffic_web_40m_2200m.csv python scripts/profile_run.py --config web_40m_2200m --runs 1 > /dev/null 2>&1
