#!/bin/bash
# Build libglp.so in-tree, then run "$1" on the B200 through gpurun (log -> $2).
cd /root/repo || exit 1
python -c "from paper_conf_sigmod_yelhls21_b200 import _build; _build.build()" || exit 1
timeout ${GPU_TIMEOUT_OUTER:-3300} /usr/local/graft/bin/gpurun --timeout ${GPU_TIMEOUT:-1500} -- "$1" > "$2" 2>&1
echo "gpurun exit $?"
