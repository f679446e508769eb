NULPA_FULLSIZE_SEEDS=2,3 NULPA_FULLSIZE_OUT=gpurun_out/r2_quality_fullsize_seeds23.json python -m pytest tests/test_gpu_fullsize.py -q -p no:cacheprovider -k quality_vs_full > gpurun_out/t17.log 2>&1; tail -1 gpurun_out/t17.log
for c in web_40m_2200m rmat_4m_70m; do for wd in 512 256; do
  python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --param wide_degree=$wd > gpurun_out/r2w_${c}_$wd.json 2>&1
  python -c "
import json
d=json.loads(open('gpurun_out/r2w_${c}_$wd.json').read().strip().splitlines()[-1])
print('$c wd=$wd', round(d['value']/1e9,2), round(d['ms_per_step'],3), {k:(v['stream_span_ms_per_run'], v['kernel_ms_per_run_serial']) for k,v in d['bins'].items()})"
done; done
ncu --clock-control none -k regex:"^k_(warp|block|thread|giant_accumulate|frontier)" --csv --metrics gpu__time_duration.sum,smsp__thread_inst_executed_per_inst_executed.ratio,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum python scripts/profile_run.py --runs 1 --config web_40m_2200m > gpurun_out/r2_eff_web.csv 2>&1
ncu --clock-control none -k regex:"^k_(warp|block|thread|giant_accumulate|frontier)" --csv --metrics gpu__time_duration.sum,smsp__thread_inst_executed_per_inst_executed.ratio,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum python scripts/profile_run.py --runs 1 --config rmat_4m_70m > gpurun_out/r2_eff_rmat.csv 2>&1
