#!/bin/bash
# round-1 (session 3) probe: parity of the level slots and fixed-point hot set,
# PageRank scatter A/B, BFS-only bench, and an ncu source capture of the biggest BFS level
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "level_slots or ordered_variants or in_star or bit_exact or degree_ordered" 2>&1 | tail -4 > $O/t_r1b.log
timeout 600 python tools/pr_variants.py --scale 27 --out $O/pr_variants.json > $O/pr_variants.log 2>&1
timeout 600 python bench.py --algos bfs --no-cpu-baseline --no-e2e > $O/bench_bfs.json 2> $O/bench_bfs.err
GTS_BFS_SLOTS=0 timeout 600 python bench.py --algos bfs --no-cpu-baseline --no-e2e > $O/bench_bfs_noslots.json 2> $O/bench_bfs_noslots.err
GTS_BFS_OCC=3 timeout 600 python bench.py --algos bfs --no-cpu-baseline --no-e2e > $O/bench_bfs_occ3.json 2> $O/bench_bfs_occ3.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/bfs_launch.csv python bench.py --algos bfs --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1
python tools/launch_summary.py $O/bfs_launch.csv > $O/bfs_launch.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bfs_expand -s 2 -c 1 -o $O/bfs_full -f python tools/profile_run.py --algos bfs --order > /dev/null 2>&1
ls -la $O
