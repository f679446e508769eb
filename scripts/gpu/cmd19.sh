python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "modularity or shards or nccl" > gpurun_out/t16.log 2>&1; tail -1 gpurun_out/t16.log
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:k_mod --csv --log-file gpurun_out/r2_mod.csv python scripts/profile_run.py --runs 1 > /dev/null 2>&1
python scripts/launch_table.py gpurun_out/r2_mod.csv
