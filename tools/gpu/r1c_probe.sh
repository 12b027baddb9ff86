#!/bin/bash
# level-fill rewrite + unweighted dense-tile shortcut: parity, BFS bench A/B (occupancy), launch list
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "level_slots or bit_exact or degree_ordered or wcc or tile_walk or streamed or micro or pid16 or fullsize" 2>&1 | tail -4 > $O/t_r1c.log
for occ in 2 3; do
  GTS_BFS_OCC=$occ timeout 600 python bench.py --algos bfs,wcc --no-cpu-baseline --no-e2e > $O/bench_bfs_occ$occ.json 2> $O/bench_bfs_occ$occ.err
done
GTS_BFS_OCC=3 timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/bfs_launch.csv python bench.py --algos bfs --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1
python tools/launch_summary.py $O/bfs_launch.csv > $O/bfs_launch.txt
ls -la $O
