cd ${GRAFT_REPO_ROOT:-.}
for v in "$@"; do echo "== $v"; GLP_LIB=$v python tools/e2e_probe.py 24; done
