#!/bin/bash
# like sched_ab.sh with a weights mode: bash scripts/sched_ab_w.sh none "specs" seeds
W=$1; SEEDS=${3:-"0"}
for spec in $2; do
  P=""; for kv in ${spec//,/ }; do P="$P --param $kv"; done
  for s in $SEEDS; do
    python bench.py --no-e2e --no-cpu-baseline --seed $s --weights $W $P 2>&1 | tail -n 1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$W $spec seed $s', round(d['value']/1e9,2), round(d['ms_per_step'],2), d['changed'], d['modularity_runs'], {k:v['kernel_ms_per_run'] for k,v in d['bins'].items()})"
  done
done
