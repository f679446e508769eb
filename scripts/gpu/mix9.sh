for c in sbm_1m_20m rmat_4m_70m web_40m_2200m; do for v in cur ws0f cur ws0f; do NULPA_LIB=libs_ab/libnulpa_$v.so CONFIG=$c PSETS="${c}_$v:" bash scripts/gpu/ab_params.sh; done; done
