#!/bin/bash
# bench line + SSSP/WCC occupancy A/B + launch list of one full bench step
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out
timeout 900 python bench.py > $O/bench_full.json 2> $O/bench_full.err
timeout 600 python bench.py --algos sssp,wcc --no-cpu-baseline --no-e2e > $O/bench_sw_occ2.json 2> $O/bench_sw_occ2.err
GTS_SSSP_OCC=3 GTS_WCC_OCC=3 timeout 600 python bench.py --algos sssp,wcc --no-cpu-baseline --no-e2e > $O/bench_sw_occ3.json 2> $O/bench_sw_occ3.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/step_launch.csv python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1
python tools/launch_summary.py $O/step_launch.csv > $O/step_launch.txt
ls -la $O
