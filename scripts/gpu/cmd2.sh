python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider > gpurun_out/t3.log 2>&1; tail -3 gpurun_out/t3.log
python scripts/profile_run.py --runs 4 > gpurun_out/new_prof2.txt 2>&1; cat gpurun_out/new_prof2.txt
bash scripts/ncu_quick.sh 'k_warp' ncu_new1 > gpurun_out/ncu_new1.txt 2>&1
NULPA_LIB=libs_ab/libnulpa_old.so bash scripts/ncu_quick.sh 'k_warp' ncu_old1 > gpurun_out/ncu_old1.txt 2>&1
