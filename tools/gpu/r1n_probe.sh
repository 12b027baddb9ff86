#!/bin/bash
# weighted dense-tile threshold: parity + SSSP A/B + launch list
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "sssp or weighted or micro or occupancy or lp_slicing or streamed" 2>&1 | tail -4 > $O/t_r1n.log
for wd in 0 1; do
  GTS_WDENSE=$wd GTS_BENCH_CLOCKS=off timeout 600 python bench.py --algos sssp --no-cpu-baseline --no-e2e --steps 5 > $O/bench_wd$wd.json 2> $O/bench_wd$wd.err
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/sssp_launch.csv python bench.py --algos sssp --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1
python tools/launch_summary.py $O/sssp_launch.csv > $O/sssp_launch.txt
ls -la $O
