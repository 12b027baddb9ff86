#!/bin/bash
# full GPU suite + ncu capture of the largest SSSP round
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -4 > $O/t_full.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sssp_expand -s 3 -c 1 -o $O/sssp_full -f python tools/profile_run.py --algos sssp --order > /dev/null 2>&1
ls -la $O
