export NULPA_FULLSIZE_OUT=gpurun_out/r2_quality_fullsize.json
python -m pytest tests/test_gpu_fullsize.py -q -p no:cacheprovider -k quality_vs_full > gpurun_out/t15.log 2>&1; tail -1 gpurun_out/t15.log
for c in web_40m_2200m road_50m_110m rmat_4m_70m sbm_1m_20m; do
  ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r2_launches_$c.csv python scripts/profile_run.py --config $c --runs 1 > /dev/null 2>&1
done
ncu --set full --import-source on --clock-control none --kernel-name-base mangled -k regex:k_warpILb0ELb1ELi512 -c 2 -o gpurun_out/r2_kwarp_full -f python scripts/profile_run.py --runs 1 > gpurun_out/r2_kwarp_full.log 2>&1
du -sh gpurun_out
