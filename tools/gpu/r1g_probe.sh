#!/bin/bash
# per-call wall vs kernel breakdown of the bench step: current defaults vs session-start settings
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out
timeout 600 python tools/step_breakdown.py 27 > $O/sb_default.txt 2>&1
GTS_BFS_SLOTS=0 GTS_BFS_OCC=2 GTS_WCC_OCC=2 timeout 600 python tools/step_breakdown.py 27 > $O/sb_old.txt 2>&1
ls -la $O
