#!/bin/bash
# Run tools/quick_perf.py once per build/<variant>.so (on the GPU box).
# usage: tools/ab.sh SCALE ITERS variant...
scale=$1; iters=$2; shift 2
for v in "$@"; do
  echo "=== $v"
  GLP_LIB=build/$v.so python tools/quick_perf.py $scale $iters 2>&1 | grep -E "^(RunInfo|iter|arcs|mfl|push|gen)" | tail -12
done
