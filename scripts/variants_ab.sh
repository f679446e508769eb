#!/bin/bash
# A/B library variants on the GPU box: bash scripts/variants_ab.sh "NAME:-DFOO=1 NAME2:" [seeds]
# Builds each variant to /tmp/nulpa_NAME.so and runs kbench + bench (per seed) against it via NULPA_LIB.
SEEDS=${2:-"0 1"}
for spec in $1; do
  name=${spec%%:*}; defs=${spec#*:}
  python paper_conf_ipps_sahunk25_b200/build.py --out /tmp/nulpa_$name.so ${defs//,/ } > /dev/null || { echo "build $name failed"; continue; }
  echo "== $name ($defs)"
  NULPA_LIB=/tmp/nulpa_$name.so python scripts/kbench.py --async-too 2>&1 | tail -n 4
  for s in $SEEDS; do
    NULPA_LIB=/tmp/nulpa_$name.so python bench.py --no-e2e --no-cpu-baseline --seed $s 2>&1 | tail -n 1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$name seed $s', round(d['value']/1e9,2), round(d['ms_per_step'],2), d['changed'], round(d['modularity'],4), {k:v['kernel_ms_per_run'] for k,v in d['bins'].items()})"
  done
done
