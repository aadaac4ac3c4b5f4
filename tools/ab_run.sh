#!/bin/bash
# On the GPU box: tools/ab_time.py once per build/<variant>.so for each workload.
# usage: tools/ab_run.sh "WORKLOAD..." REPS variant...
wls=$1; reps=$2; shift 2
for wl in $wls; do
  for v in "$@"; do
    GLP_LIB=build/$v.so timeout 900 python tools/ab_time.py $wl $reps 2>&1 | grep '^{' || echo "{\"lib\": \"$v\", \"failed\": true}"
  done
done
