SKEL_MODES=3,9 timeout 900 python scripts/micro/skeleton.py 2>&1 | grep "ms$"
