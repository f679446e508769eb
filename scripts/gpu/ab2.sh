# usage: bash scripts/gpu/ab2.sh v1 v2 ...   (libs_ab/libnulpa_<v>.so): warp-bin ms per run + ncu per sweep
for v in "$@"; do
  L=libs_ab/libnulpa_$v.so
  echo "== $v"; NULPA_LIB=$L python scripts/profile_run.py --runs 5 2>&1 | tail -3
  NULPA_LIB=$L ncu --clock-control none --kernel-name-base mangled -k regex:k_warpILb0ELb1ELi512 -c 2 --csv --metrics gpu__time_duration.sum,smsp__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_active python scripts/profile_run.py --runs 1 2>/dev/null | grep -E "k_warp" | awk -F'","' '{print $(NF-2), $NF}'
done
