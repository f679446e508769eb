# ncu --set full of the warp-bin k_warp (sweep 0 and sweep 1 of one web run), source-correlated
LIB=${NULPA_LIB:-paper_conf_ipps_sahunk25_b200/libnulpa.so}
NAME=${NAME:-kw_full}
timeout 900 ncu --set full --import-source on --clock-control none --kernel-name-base mangled -k regex:k_warpILb0ELb1ELi512 -c 2 -f -o gpurun_out/$NAME python scripts/profile_run.py --runs 1 > gpurun_out/$NAME.log 2>&1
ls -la gpurun_out/$NAME.ncu-rep
