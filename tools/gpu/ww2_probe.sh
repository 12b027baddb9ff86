#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out
GTS_WW=1 timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q 2>&1 | tail -4 > $O/t_ww2.log
for ww in 0 1; do
  GTS_WW=$ww timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/bsw_ww$ww.csv python tools/profile_run.py --algos bfs,sssp,wcc --order > /dev/null 2>&1
  python tools/launch_summary.py $O/bsw_ww$ww.csv > $O/bsw_ww$ww.txt
done
