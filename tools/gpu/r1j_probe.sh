#!/bin/bash
# tail deferral of the PageRank scatter: parity + A/B over the threshold
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "ordered_variants or in_star or pagerank_tolerance" 2>&1 | tail -4 > $O/t_r1j.log
timeout 900 python tools/pr_variants.py --scale 27 --variants "base:;t8:GTS_PR_TAIL=8388608;t16:GTS_PR_TAIL=16777216;t25:GTS_PR_TAIL=25165824;t40:GTS_PR_TAIL=41943040;t25np:GTS_PR_TAIL=25165824,GTS_L2_PERSIST=0" --out $O/pr_tail.json > $O/pr_tail.log 2>&1
timeout 300 python tools/nvml_probe.py > $O/nvml_probe.txt 2>&1
ls -la $O
