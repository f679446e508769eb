# ncu SourceCounters + WarpStateStats of the warp-bin k_warp (sweep 0 and sweep 1 of one web run)
NAME=${NAME:-kw_src}
timeout 1200 ncu --section SourceCounters --section WarpStateStats --section LaunchStats --section Occupancy --import-source on --clock-control none --kernel-name-base mangled -k regex:k_warpILb0ELb1ELi512 -c 2 -f -o gpurun_out/$NAME python scripts/profile_run.py --runs 1 > gpurun_out/$NAME.log 2>&1
ls -la gpurun_out/$NAME.ncu-rep
