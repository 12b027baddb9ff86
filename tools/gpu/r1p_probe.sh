#!/bin/bash
# warp-window item gather: parity (whole parity file) + BFS/SSSP/WCC A/B
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py -m gpu -x -q 2>&1 | tail -4 > $O/t_r1p.log
for gw in 0 1; do
  GTS_GWW=$gw GTS_BENCH_CLOCKS=off timeout 600 python bench.py --algos bfs,sssp,wcc --no-cpu-baseline --no-e2e --steps 5 > $O/bench_gww$gw.json 2> $O/bench_gww$gw.err
done
ls -la $O
