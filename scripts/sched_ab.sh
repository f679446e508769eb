#!/bin/bash
# Schedule A/B: bash scripts/sched_ab.sh "first_sweep_block=1 first_sweep_block=32,sweep_block=2" [seeds]
SEEDS=${2:-"0"}
for spec in $1; do
  P=""; for kv in ${spec//,/ }; do P="$P --param $kv"; done
  for s in $SEEDS; do
    python bench.py --no-e2e --no-cpu-baseline --seed $s $P 2>&1 | tail -n 1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$spec seed $s', round(d['value']/1e9,2), round(d['ms_per_step'],2), d['changed'], d['modularity_runs'], {k:v['kernel_ms_per_run'] for k,v in d['bins'].items()})"
  done
done
