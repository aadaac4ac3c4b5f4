# One GPU call: the bench line of every workload (no ncu), into gpurun_out/.
cd ${GRAFT_REPO_ROOT:-.}
o=gpurun_out
python bench.py > $o/bench_rmat24.json 2> $o/bench_rmat24.err
python bench.py --impl reference --steps 3 --warmup 3 > $o/bench_reference.json 2> $o/bench_reference.err
for w in sbm1m taobao100m rmat24_llp; do python bench.py --workload $w > $o/bench_$w.json 2> $o/bench_$w.err; done
python bench.py --workload rmat28_llp --steps 3 --warmup 3 --no-e2e > $o/bench_rmat28_llp.json 2> $o/bench_rmat28_llp.err
python -c "import __graft_entry__ as g; g.smoke()" > $o/smoke.log 2>&1
