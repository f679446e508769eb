for c in web_40m_2200m rmat_4m_70m road_50m_110m; do
  timeout 900 ncu --clock-control none -k regex:'^k_(warp|block|thread|tscan|tact|giant_accumulate|giant_count|frontier)' --csv --metrics gpu__time_duration.sum,smsp__thread_inst_executed_per_inst_executed.ratio,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum python scripts/profile_run.py --runs 1 --config $c > gpurun_out/wexec_$c.csv 2>/dev/null
done
ls -la gpurun_out/wexec_*
