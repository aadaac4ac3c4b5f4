#!/bin/bash
# ncu --set full (source-level) of the table kernels of a short run; launch
# times + instruction counts to gpurun_out/ncw_t.csv, SASS-level source pages
# of the launches longer than 0.3 ms gzipped to gpurun_out/ncw_src_<id>.csv.gz.
# usage (GPU box): bash tools/ncu_w.sh [lib] [workload] [iters] [kernel regex]
LIB=${1:-}; WL=${2:-rmat24}; IT=${3:-3}; KR=${4:-'mfl_(warp|block|low)'}
[ -n "$LIB" ] && export GLP_LIB=$LIB
ncu --profile-from-start off --set full --import-source on --clock-control none -k regex:"$KR" -o /tmp/ncw -f python tools/prof_it.py $WL $IT > gpurun_out/ncw.log 2>&1
echo rc=$?
ncu -i /tmp/ncw.ncu-rep --page raw --csv --metrics gpu__time_duration.sum,smsp__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__warps_active.avg.pct_of_peak_sustained_active > gpurun_out/ncw_t.csv
python tools/ncu_summary.py /tmp/ncw.ncu-rep > gpurun_out/ncw_summary.txt
n=$(($(wc -l < gpurun_out/ncw_t.csv) - 2))
for k in $(seq 0 $((n-1))); do
  t=$(python -c "import csv;r=list(csv.reader(open('gpurun_out/ncw_t.csv')));h=r[0];print(r[2+$k][h.index('gpu__time_duration.sum')])")
  if python -c "import sys; sys.exit(0 if float('$t') > 0.3 else 1)"; then
    ncu -i /tmp/ncw.ncu-rep --page source --csv --print-source cuda,sass --launch-skip $k --launch-count 1 2>/dev/null | gzip -c > gpurun_out/ncw_src_$k.csv.gz
  fi
done
