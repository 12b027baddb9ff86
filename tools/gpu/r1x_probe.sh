#!/bin/bash
# launch list of one bench step with the final round-1 build (ncu, cold-cache serialised: shares only)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/x_launch.csv python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1
python tools/launch_summary.py $O/x_launch.csv > $O/x_launch.txt
ls -la $O
