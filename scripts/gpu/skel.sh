timeout 900 python scripts/micro/skeleton.py 2>&1 | grep -v Warning | tail -20
timeout 120 libs_ab/mc | tail -12
