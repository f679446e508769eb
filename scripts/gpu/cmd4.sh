python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider > gpurun_out/t5.log 2>&1; tail -2 gpurun_out/t5.log
python scripts/profile_run.py --runs 4 > gpurun_out/prof5.txt 2>&1; cat gpurun_out/prof5.txt
ncu --clock-control none --kernel-name-base mangled -k regex:k_warpILb0ELb1ELi512 -c 2 --csv --metrics gpu__time_duration.sum,smsp__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_active python scripts/profile_run.py --runs 1 > gpurun_out/ncu5.csv 2>&1
grep -E "k_warp" gpurun_out/ncu5.csv | awk -F'","' '{print $(NF-2), $NF}'
