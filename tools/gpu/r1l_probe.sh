#!/bin/bash
# LP slicing: parity (incl. full suite subset) + BFS/SSSP A/B + launch list
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "lp_slicing or bit_exact or level_slots or streamed or degree_ordered or sssp or micro or cache" 2>&1 | tail -4 > $O/t_r1l.log
for sp in 0 1; do
  GTS_SPLIT=$sp GTS_BENCH_CLOCKS=off timeout 600 python bench.py --algos bfs,sssp --no-cpu-baseline --no-e2e --steps 5 > $O/bench_split$sp.json 2> $O/bench_split$sp.err
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/bfs_launch.csv python bench.py --algos bfs,sssp --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1
python tools/launch_summary.py $O/bfs_launch.csv > $O/bfs_launch.txt
ls -la $O
