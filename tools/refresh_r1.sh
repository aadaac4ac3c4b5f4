# One GPU call: ncu full capture of every MFL launch of one RMAT-24 run (DRAM
# traffic per launch -> profiles/traffic.json, summary kept, report deleted:
# gpurun copies back <= 64 MiB), the bench launch list, then the bench lines.
cd ${GRAFT_REPO_ROOT:-.}
o=gpurun_out
ncu --set full --clock-control none -k regex:mfl_ -o /tmp/r24_full -f python tools/prof_r24.py 24 20 > $o/ncu_r24_full.log 2>&1
python tools/ncu_traffic.py /tmp/r24_full.ncu-rep rmat24 ${ITERS:-9} > $o/traffic_r24.log 2>&1; cp profiles/traffic.json $o/traffic.json
python tools/ncu_summary.py /tmp/r24_full.ncu-rep > $o/ncu_r24_full_summary.txt 2>&1
rm -f /tmp/r24_full.ncu-rep
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $o/launches_r24.csv python bench.py --steps 2 --warmup 3 --no-cpu --no-e2e > $o/bench_under_ncu.log 2>&1
python bench.py > $o/bench_rmat24.json 2> $o/bench_rmat24.err
python bench.py --impl reference --steps 3 --warmup 3 > $o/bench_reference.json 2> $o/bench_reference.err
for w in sbm1m taobao100m rmat24_llp; do python bench.py --workload $w > $o/bench_$w.json 2> $o/bench_$w.err; done
python bench.py --workload rmat28_llp --steps 3 --warmup 3 --no-e2e > $o/bench_rmat28_llp.json 2> $o/bench_rmat28_llp.err
