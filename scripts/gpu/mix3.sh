VARIANTS="tc1 v2" PARITY="v2" bash scripts/gpu/ab_road.sh
for v in v2; do
  for c in rmat_4m_70m sbm_1m_20m; do NULPA_LIB=libs_ab/libnulpa_$v.so CONFIG=$c PSETS="${c}_$v:" bash scripts/gpu/ab_params.sh; done
done
