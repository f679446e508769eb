# A/B prebuilt libraries: bash scripts/abl.sh "old new" [tests] [bench]
for v in $1; do
  cp libs_ab/$v.so paper_conf_ipps_sahunk25_b200/libnulpa.so
  echo "== $v"
  if [ -n "$2" ]; then python -m pytest tests -m gpu -x -q 2>&1 | tail -1; fi
  python scripts/kbench.py --async-too 2>&1 | tail -4
  if [ -n "$3" ]; then for s in 0 1; do python bench.py --no-e2e --no-cpu-baseline --seed $s 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v', round(d['value']/1e9,2), round(d['ms_per_step'],2), d['iterations'], d['changed'], round(d['modularity'],4), {k:v['kernel_ms_per_run'] for k,v in d['bins'].items()})"; done; fi
done
