CONFIG=web_40m_2200m PSETS="web_sb4: web_sb1:sweep_block=1 web_sb2:sweep_block=2 web_sb8:sweep_block=8 web_sb16:sweep_block=16" bash scripts/gpu/ab_params.sh
CONFIG=rmat_4m_70m PSETS="rmat_def: rmat_wd256:wide_degree=256 rmat_wd1024:wide_degree=1024 rmat_gd1024:giant_degree=1024 rmat_gd4096:giant_degree=4096 rmat_sd12:switch_degree=12 rmat_sd24:switch_degree=24" bash scripts/gpu/ab_params.sh
