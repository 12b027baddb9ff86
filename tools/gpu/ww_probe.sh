#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "binned or in_star or ordered" 2>&1 | tail -5 > $O/t_ww.log
for ww in 1 0; do
  GTS_PR_WW=$ww timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/pr_launch_ww$ww.csv python tools/profile_run.py --algos pr --order --pr-iters 3 > /dev/null 2>&1
  python tools/launch_summary.py $O/pr_launch_ww$ww.csv > $O/pr_launch_ww$ww.txt
done
timeout 300 python bench.py --algos pr --no-cpu-baseline --no-e2e --steps 3 --warmup 3 > $O/pr_ww.json 2>/dev/null
timeout 600 ncu --set full --clock-control none --import-source on -k regex:pr_scatter_ww -s 1 -c 1 -o $O/pr_ww -f python tools/profile_run.py --algos pr --order --pr-iters 2 > /dev/null 2>&1
python tools/ncu_summary.py $O/pr_ww.ncu-rep > $O/pr_ww_ncu.txt 2>&1
