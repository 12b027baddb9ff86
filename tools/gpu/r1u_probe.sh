#!/bin/bash
# device timelines (CUPTI via torch.profiler) of one BFS / WCC / SSSP call on degree-ordered RMAT-27
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out
for a in bfs wcc sssp; do
  timeout 600 python tools/bfs_timeline.py 27 $a > $O/u_tl_$a.txt 2>&1
done
ls -la $O
