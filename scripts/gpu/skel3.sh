SKEL_MODES=3 SKEL_PHASES=1,2,4,8 timeout 900 python scripts/micro/skeleton.py 2>&1 | grep "ms$"
