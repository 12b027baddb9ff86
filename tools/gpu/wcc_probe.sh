#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "wcc" 2>&1 | tail -4 > $O/t_wcc.log
for k in 0 1 2; do
  GTS_WCC_SAMPLE=$k timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/wcc_launch_k$k.csv python tools/profile_run.py --algos wcc --order > /dev/null 2>&1
  python tools/launch_summary.py $O/wcc_launch_k$k.csv > $O/wcc_launch_k$k.txt
done
timeout 900 python -m pytest tests/test_gpu_fullsize.py -m gpu -x -q -k "wcc" 2>&1 | tail -4 >> $O/t_wcc.log
