#!/bin/bash
# ncu evidence for profiles/: (1) the launch list of the bench command,
# (2) one --set full capture of every MFL launch of a whole R24 run,
# summarised on the box (the report itself exceeds gpurun's copy-back limit).
ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"mfl_|k_|glp" -c 3000 --csv --log-file gpurun_out/r2_ncu_launches_rmat24.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu > gpurun_out/r2_ncu_launches_bench.log 2>&1
echo "launches rc=$?"
ncu --set full --import-source on --clock-control none --profile-from-start off -k regex:mfl_ -o /tmp/r2_rmat24_full python tools/prof_it.py rmat24 20 > gpurun_out/r2_ncu_full.log 2>&1
echo "full rc=$?"
python tools/ncu_summary.py /tmp/r2_rmat24_full.ncu-rep > gpurun_out/r2_ncu_rmat24_all_launches.txt
python tools/ncu_traffic.py /tmp/r2_rmat24_full.ncu-rep rmat24 9 > gpurun_out/r2_traffic_rmat24.json
ncu -i /tmp/r2_rmat24_full.ncu-rep --page raw --csv > gpurun_out/r2_ncu_rmat24_raw.csv 2>/dev/null
cp profiles/traffic.json gpurun_out/traffic.json
ls -la gpurun_out
