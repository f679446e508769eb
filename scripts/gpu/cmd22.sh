for r in 1024 512; do echo "== min run $r"; NULPA_LIB=libs_ab/libnulpa_run$r.so SHARDS=4,8 python scripts/shard_quality.py 2>&1 | python -c "
import sys, json
for line in sys.stdin:
    p, d = line.split(' ', 1)
    d = json.loads(d)
    print(p, d['modularity_runs'], d['max_shard_sweep_ms_last_run'])
"; done
