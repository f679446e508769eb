python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider > gpurun_out/t2.log 2>&1; tail -3 gpurun_out/t2.log
python scripts/profile_run.py --runs 4 > gpurun_out/new_prof.txt 2>&1
NULPA_LIB=libs_ab/libnulpa_old.so python scripts/profile_run.py --runs 4 > gpurun_out/old_prof.txt 2>&1
python scripts/kbench.py --async-too > gpurun_out/new_kbench.txt 2>&1
cat gpurun_out/new_prof.txt gpurun_out/old_prof.txt gpurun_out/new_kbench.txt
