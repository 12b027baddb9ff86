#!/bin/bash
# full GPU suite + BFS A/B (occupancy 2 vs 3 default) + launch list of a BFS step
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -4 > $O/t_r1d.log
for occ in 2 3; do
  GTS_BFS_OCC=$occ timeout 600 python bench.py --algos bfs,wcc --no-cpu-baseline --no-e2e > $O/bench_bfs_occ$occ.json 2> $O/bench_bfs_occ$occ.err
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/bfs_launch.csv python bench.py --algos bfs --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1
python tools/launch_summary.py $O/bfs_launch.csv > $O/bfs_launch.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bfs_expand -s 2 -c 1 -o $O/bfs_full2 -f python tools/profile_run.py --algos bfs --order > /dev/null 2>&1
ls -la $O
