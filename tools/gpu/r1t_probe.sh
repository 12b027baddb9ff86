#!/bin/bash
# per-call breakdown of the bench step (wall / lib wall / kernels / finish) to locate the BFS call overhead
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out
timeout 900 python tools/step_breakdown.py 27 > $O/t_break_default.txt 2>&1
GTS_BFS_BATCH=16 GTS_L2_PERSIST_BFS=0 timeout 900 python tools/step_breakdown.py 27 > $O/t_break_b16_nopersist.txt 2>&1
ls -la $O
