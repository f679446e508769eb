#!/bin/bash
# bash scripts/lib_ab.sh "name:-DA=1 -DB=2;name2:-DC=3" "sched specs" "seeds"  -- build variants, run sched_ab on each
IFS=';' read -ra VS <<< "$1"
for v in "${VS[@]}"; do
  n=${v%%:*}; d=${v#*:}
  python paper_conf_ipps_sahunk25_b200/build.py --out /tmp/v_$n.so $d > /dev/null || { echo "build $n failed"; continue; }
  echo "== $n ($d)"
  NULPA_LIB=/tmp/v_$n.so bash scripts/sched_ab.sh "$2" "$3"
done
