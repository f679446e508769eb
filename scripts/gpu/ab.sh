# usage: bash scripts/gpu/ab.sh <tag> -- A/B of the in-tree library vs libs_ab/libnulpa_prev.so
T=${1:-ab}
python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider > gpurun_out/${T}_tests.log 2>&1; tail -1 gpurun_out/${T}_tests.log
for v in new prev; do
  L=paper_conf_ipps_sahunk25_b200/libnulpa.so; [ $v = prev ] && L=libs_ab/libnulpa_prev.so
  echo "== $v"; NULPA_LIB=$L python scripts/profile_run.py --runs 5 2>&1 | tail -3
  NULPA_LIB=$L ncu --clock-control none --kernel-name-base mangled -k regex:k_warpILb0ELb1ELi512 -c 2 --csv --metrics gpu__time_duration.sum,smsp__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_active python scripts/profile_run.py --runs 1 2>/dev/null | grep -E "k_warp" | awk -F'","' '{print $(NF-2), $NF}'
done
