#!/bin/bash
# bash scripts/lib_sched_ab.sh "lib1 lib2" "spec1 spec2" [seeds]  (lib "" = in-tree build; spec as in sched_ab.sh)
for L in $1; do
  echo "== $L"
  if [ "$L" = "tree" ]; then NULPA_LIB= bash scripts/sched_ab.sh "$2" "${3:-0}"; else NULPA_LIB=$L bash scripts/sched_ab.sh "$2" "${3:-0}"; fi
done
