ncu --set full --import-source on --clock-control none --kernel-name-base mangled -k regex:k_warpILb0ELb1ELi512 -c 2 -o gpurun_out/kw_new1 -f python scripts/profile_run.py --runs 1 > gpurun_out/kw_new1.log 2>&1
tail -3 gpurun_out/kw_new1.log
