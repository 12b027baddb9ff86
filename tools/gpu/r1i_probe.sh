#!/bin/bash
# round bench line (default settings) + twitter line + launch list of one bench step
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out
timeout 1200 python bench.py > $O/bench_line.json 2> $O/bench_line.err
timeout 900 python bench.py --workload twitter --no-cpu-baseline > $O/bench_twitter.json 2> $O/bench_twitter.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/step_launch.csv python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1
python tools/launch_summary.py $O/step_launch.csv > $O/step_launch.txt
ls -la $O
