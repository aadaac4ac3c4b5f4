#!/bin/bash
# Full ncu capture (source-level) of every MFL launch of an ITERS-iteration run
# of WORKLOAD (class kernels serialised); summary + source pages of the 4
# longest launches into gpurun_out/.
# Usage (on the GPU box): bash tools/ncu_it2.sh TAG [workload] [iters]
TAG=${1:-it2}; WL=${2:-rmat24}; IT=${3:-2}
mkdir -p gpurun_out
REP=/tmp/ncu_${TAG}
ncu --profile-from-start off --set full --import-source on --clock-control none \
    -k regex:'mfl_' -o $REP -f python tools/prof_it.py $WL $IT > gpurun_out/ncu_${TAG}.log 2>&1
echo "ncu rc=$?"
python tools/ncu_summary.py $REP.ncu-rep > gpurun_out/ncu_${TAG}_summary.txt
ncu -i $REP.ncu-rep --page raw --csv --metrics gpu__time_duration.sum > /tmp/ncu_${TAG}_t.csv 2>/dev/null
for k in $(python - <<PY
import csv
r=list(csv.reader(open('/tmp/ncu_${TAG}_t.csv')))
h=r[0]; t=h.index('gpu__time_duration.sum')
rows=sorted(((float(x[t]),j) for j,x in enumerate(r[2:]) if x[t]), reverse=True)
print(' '.join(str(j) for _,j in rows[:4]))
PY
); do
  ncu -i $REP.ncu-rep --page source --csv --print-source cuda,sass --launch-skip $k --launch-count 1 > /tmp/src_$k.csv 2>/dev/null
  python tools/src_hot.py /tmp/src_$k.csv 40 > gpurun_out/ncu_${TAG}_src_$k.txt
done
ls -la gpurun_out
