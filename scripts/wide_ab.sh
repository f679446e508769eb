#!/bin/bash
# A/B of the wide k_warp schedule (group size / guided K) and wide_degree on the bench graph.
# bash scripts/wide_ab.sh "name:-DFOO=1 ..." "extra bench args per line;..."
for spec in $1; do
  name=${spec%%:*}; defs=${spec#*:}
  python paper_conf_ipps_sahunk25_b200/build.py --out /tmp/nulpa_$name.so ${defs//,/ } > /dev/null || { echo "build $name failed"; continue; }
  IFS=';' read -ra PS <<< "${2:- }"
  for pa in "${PS[@]}"; do
    NULPA_LIB=/tmp/nulpa_$name.so python bench.py --no-e2e --no-cpu-baseline --quality-runs 0 $pa 2>&1 | tail -n 1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$name', '$pa', round(d['value']/1e9,2), round(d['ms_per_step'],2), d['changed'], round(d['modularity'],4), {k:v['kernel_ms_per_run'] for k,v in d['bins'].items()})"
  done
done
