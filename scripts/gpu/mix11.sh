NULPA_LIB=libs_ab/libnulpa_ths.so timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider > gpurun_out/ab_parity_ths.log 2>&1; echo "parity ths: $(tail -1 gpurun_out/ab_parity_ths.log)"
for c in rmat_4m_70m web_40m_2200m; do for v in cur ths cur ths; do NULPA_LIB=libs_ab/libnulpa_$v.so CONFIG=$c PSETS="${c}_$v:" bash scripts/gpu/ab_params.sh; done; done
