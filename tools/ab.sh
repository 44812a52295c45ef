#!/bin/bash
# A/B timing of library variants in one GPU call, interleaved to cancel drift.
# usage: tools/ab.sh "c3:15 c2:15,2" variantA variantB ...   ("cur" = the in-tree build)
CASES=$1; shift
for rep in 1 2; do
  for v in "$@"; do
    if [ "$v" = cur ]; then unset SASSI_LIB; else export SASSI_LIB=paper_conf_isca_stephensonhlejn15_b200/lib/variants/$v/libsassi.so; fi
    for c in $CASES; do
      timeout 300 python tools/time_masks.py ${c%%:*} ${c##*:} | sed "s/^/[$v] /"
    done
  done
done
unset SASSI_LIB
