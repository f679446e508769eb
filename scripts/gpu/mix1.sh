SKEL_MODES=3,7,8 timeout 900 python scripts/micro/skeleton.py 2>&1 | grep -v Warning | grep "ms$"
PSETS="def: bd128:block_degree=128 bd96:block_degree=96 bd65:block_degree=65" bash scripts/gpu/ab_params.sh
