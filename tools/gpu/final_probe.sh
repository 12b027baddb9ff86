#!/bin/bash
# end-of-round evidence: smoke, full GPU suite, the bench lines (RMAT-27, Twitter-shaped),
# the launch list of one bench step and an ncu capture of the largest BFS level
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" > $O/f_smoke.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -4 > $O/f_tests.log
timeout 1200 python bench.py > $O/f_bench.json 2> $O/f_bench.err
timeout 900 python bench.py --workload twitter --no-cpu-baseline > $O/f_twitter.json 2> $O/f_twitter.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/f_launch.csv python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1
python tools/launch_summary.py $O/f_launch.csv > $O/f_launch.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bfs_expand -s 2 -c 1 -o $O/f_bfs_full -f python tools/profile_run.py --algos bfs --order > /dev/null 2>&1
ls -la $O
