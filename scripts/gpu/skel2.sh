SKEL_MODES=1,3,4,6 timeout 900 python scripts/micro/skeleton.py 2>&1 | grep -v Warning | tail -24
