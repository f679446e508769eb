# A/B the warp-bin kernels: bash scripts/ab.sh "1 2 3" [tests]
VS=${1:-"2 3"}
if [ -n "$2" ]; then for v in $VS; do NULPA_WARP_KERNEL=$v python -m pytest tests -m gpu -x -q 2>&1 | tail -1; done; fi
for v in $VS; do echo "== v$v"; NULPA_WARP_KERNEL=$v python scripts/kbench.py --async-too 2>&1 | tail -4; done
for v in $VS; do for s in 0 1; do NULPA_WARP_KERNEL=$v python bench.py --no-e2e --no-cpu-baseline --seed $s 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('v$v', round(d['value']/1e9,2), round(d['ms_per_step'],2), d['iterations'], d['changed'], round(d['modularity'],4), {k:v['kernel_ms_per_run'] for k,v in d['bins'].items()})"; done; done
