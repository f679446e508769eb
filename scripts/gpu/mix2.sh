for c in rmat_4m_70m sbm_1m_20m; do
  CONFIG=$c PSETS="${c}_bo3: ${c}_bo1:bin_order=1 ${c}_bo2:bin_order=2" bash scripts/gpu/ab_params.sh
done
