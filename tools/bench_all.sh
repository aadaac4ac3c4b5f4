#!/bin/bash
# Every bench.py workload once on the GPU box -> gpurun_out/r2_bench_<workload>.json
# usage: tools/bench_all.sh [TAG] [workloads...]
tag=${1:-v1}; shift
wls=${@:-"rmat24 sbm1m taobao100m rmat24_llp rmat24_weighted rmat24_slp rmat24_hostarcs karate rmat28_llp"}
for wl in $wls; do
  steps=10; [ $wl = rmat28_llp ] && steps=3; [ $wl = karate ] && steps=20
  timeout 1500 python bench.py --workload $wl --steps $steps --warmup 3 > gpurun_out/r2_bench_${wl}_$tag.json 2> gpurun_out/r2_bench_${wl}_$tag.err
  echo "$wl rc=$? $(python -c "import json,sys; j=json.load(open('gpurun_out/r2_bench_${wl}_$tag.json')); print(j['value'], j['ms_per_step'], j['roofline']['frac'] if j.get('roofline') else None, j.get('e2e',{}).get('value'))" 2>&1 | tail -1)"
done
