#!/bin/bash
# binned PageRank probe: parity subset, launch times per geometry, ncu captures
set -x
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "binned or in_star or ordered" 2>&1 | tail -5 > $O/t_binned.log
for fs in 15 12 10; do
  GTS_PB_FINE_SHIFT=$fs timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/pr_launch_fs$fs.csv python tools/profile_run.py --algos pr --order --pr-iters 2 > /dev/null 2>&1
  python tools/launch_summary.py $O/pr_launch_fs$fs.csv > $O/pr_launch_fs$fs.txt
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:pr_bin -c 2 -o $O/pb_bin -f python tools/profile_run.py --algos pr --order --pr-iters 1 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:pr_apply -c 1 -o $O/pb_apply -f python tools/profile_run.py --algos pr --order --pr-iters 1 > /dev/null 2>&1
ls -la $O
