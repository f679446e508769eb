set -x
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_tact -c 2 -f -o gpurun_out/r2s2_ktact_full python scripts/profile_run.py --config road_50m_110m --runs 1 > gpurun_out/r2s2_ktact_full.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_tact --launch-skip 10 -c 1 -f -o gpurun_out/r2s2_ktact_late python scripts/profile_run.py --config road_50m_110m --runs 1 > gpurun_out/r2s2_ktact_late.log 2>&1
python bench.py --config kmer_171m_360m > gpurun_out/r2s2_bench_kmer_171m_360m.json 2> gpurun_out/r2s2_bench_kmer.err
tail -c 600 gpurun_out/r2s2_bench_kmer_171m_360m.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2s2_launches_kmer_171m_360m.csv python bench.py --config kmer_171m_360m --steps 2 --warmup 1 --no-e2e --no-cpu-baseline --quality-runs 0 > /dev/null 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r2s2_traffic_kmer_171m_360m.csv python scripts/profile_run.py --config kmer_171m_360m --runs 1 > /dev/null 2>&1
ls -la gpurun_out/
