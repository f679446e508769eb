#!/bin/bash
# Speed + modularity spread of library variants: bash scripts/quality_ab.sh "name:-DA=1,-DB=2 ..." "seeds" [quality runs]
for spec in $1; do
  name=${spec%%:*}; defs=${spec#*:}
  python paper_conf_ipps_sahunk25_b200/build.py --out /tmp/nulpa_$name.so ${defs//,/ } > /dev/null || { echo "build $name failed"; continue; }
  for s in ${2:-0 1 2}; do
    NULPA_LIB=/tmp/nulpa_$name.so python bench.py --no-e2e --no-cpu-baseline --seed $s --quality-runs ${3:-8} 2>&1 | tail -n 1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$name seed $s', round(d['value']/1e9,2), round(d['ms_per_step'],2), d['changed'], 'Q', min(d['modularity_runs']), max(d['modularity_runs']), d['modularity_runs'])"
  done
done
