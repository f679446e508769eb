export NULPA_FULLSIZE_OUT=gpurun_out/r2_quality_fullsize.json
python -m pytest tests -m gpu -q -p no:cacheprovider --durations=8 > gpurun_out/t14.log 2>&1; tail -12 gpurun_out/t14.log
# launch lists with DRAM bytes (traffic.json) for each config
for c in web_40m_2200m road_50m_110m rmat_4m_70m sbm_1m_20m; do
  ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r2_launches_$c.csv python scripts/profile_run.py --config $c --runs 1 > /dev/null 2>&1
done
# full capture of the warp-bin kernel (sweep 0 and 1) at the defaults
ncu --set full --import-source on --clock-control none --kernel-name-base mangled -k regex:k_warpILb0ELb1ELi512 -c 2 -o gpurun_out/r2_kwarp_full -f python scripts/profile_run.py --runs 1 > gpurun_out/r2_kwarp_full.log 2>&1
ncu --set full --import-source on --clock-control none -k regex:k_thread -c 2 -o gpurun_out/r2_kthread_full -f python scripts/profile_run.py --config road_50m_110m --runs 1 > gpurun_out/r2_kthread_full.log 2>&1
ncu --set full --import-source on --clock-control none -k regex:k_block -c 2 -o gpurun_out/r2_kblock_full -f python scripts/profile_run.py --config rmat_4m_70m --runs 1 > gpurun_out/r2_kblock_full.log 2>&1
ls -la gpurun_out/r2_*full*
