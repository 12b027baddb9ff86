#!/bin/bash
# batched BFS levels: parity (whole parity file) + BFS A/B batch 1 vs 4
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py -m gpu -x -q 2>&1 | tail -4 > $O/t_r1q.log
for b in 1 4 8; do
  GTS_BFS_BATCH=$b GTS_BENCH_CLOCKS=off timeout 600 python bench.py --algos bfs --no-cpu-baseline --no-e2e --steps 5 > $O/bench_b$b.json 2> $O/bench_b$b.err
done
ls -la $O
