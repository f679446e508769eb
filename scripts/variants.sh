# build variants of libnulpa with extra -D flags and time them with kbench
# usage: bash scripts/variants.sh "NAME:-DX=1 -DY=2" ...
for spec in "$@"; do
  name=${spec%%:*}; flags=${spec#*:}
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC,-O3 -shared --expt-relaxed-constexpr $flags -I include paper_conf_ipps_sahunk25_b200/csrc/nulpa.cu -o /tmp/lib_$name.so || continue
  cp /tmp/lib_$name.so paper_conf_ipps_sahunk25_b200/libnulpa.so
  echo "== $name ($flags)"; python scripts/kbench.py --async-too 2>&1 | tail -4
done
