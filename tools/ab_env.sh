# usage (on the GPU box): bash tools/ab_env.sh SCALE "ENV1=a ENV2=b" "ENV..." ...   (GLP_LIB=build/x.so selects a variant)
cd ${GRAFT_REPO_ROOT:-.}
scale=$1; shift
for spec in "$@"; do
  echo "=== $spec"
  env $spec python tools/quick_perf.py $scale 0 2>&1 | grep -E "^(RunInfo|mfl)" | sed 's/RunInfo.*elapsed_ms=\([0-9.]*\).*/ \1/' | head -3 | tr '\n' ' '; echo
done
