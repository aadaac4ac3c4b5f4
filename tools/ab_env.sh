cd $GRAFT_REPO_ROOT
run() { echo "=== $*"; env "$@" python tools/quick_perf.py 24 0 2>&1 | grep -E "^(RunInfo|mfl)" | sed 's/RunInfo.*elapsed_ms=\([0-9.]*\).*/ \1/' | head -3 | tr '\n' ' '; echo; }
run GLP_LIB=build/base.so
run GLP_LIB=build/hot.so GLP_HOT=8192
run GLP_LIB=build/hot.so GLP_HOT=24576
run GLP_LIB=build/hot.so GLP_HOT=65536
run GLP_LIB=build/hot.so GLP_HOT=0
run GLP_LIB=build/base.so GLP_CARVEOUT=50
run GLP_LIB=build/hot.so GLP_HOT=24576 GLP_CARVEOUT=50
run GLP_LIB=build/hot.so GLP_HOT=40000 GLP_CARVEOUT=40
