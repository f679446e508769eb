NULPA_LIB=libs_ab/libnulpa_tp2.so timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider > gpurun_out/ab_parity_tp2.log 2>&1; echo "parity tp2: $(tail -1 gpurun_out/ab_parity_tp2.log)"
grep -m3 "Error\|assert" gpurun_out/ab_parity_tp2.log
for c in web_40m_2200m sbm_1m_20m rmat_4m_70m; do for v in cur tp2; do NULPA_LIB=libs_ab/libnulpa_$v.so CONFIG=$c PSETS="${c}_$v:" bash scripts/gpu/ab_params.sh; done; done
