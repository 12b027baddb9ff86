#!/bin/bash
# full GPU suite, the bench line, and the launch list of one bench step
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -4 > $O/t_all.log
timeout 900 python bench.py > $O/bench_final.json 2> $O/bench_final.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/bench_launch.csv python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1
python tools/launch_summary.py $O/bench_launch.csv > $O/bench_launch.txt
