NULPA_LIB=libs_ab/libnulpa_mj5.so timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider > gpurun_out/ab_parity_mj5.log 2>&1; echo "parity mj5: $(tail -1 gpurun_out/ab_parity_mj5.log)"
for c in rmat_4m_70m web_40m_2200m; do for v in cur mj5 cur mj5; do NULPA_LIB=libs_ab/libnulpa_$v.so CONFIG=$c PSETS="${c}_$v:" bash scripts/gpu/ab_params.sh; done; done
