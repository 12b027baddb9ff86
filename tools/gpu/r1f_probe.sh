#!/bin/bash
# lean PageRank scatter: parity + A/B against the tile walk and the ww walk; bench with NVML clock sampling
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "ordered_variants or in_star or occupancy or degree_ordered" 2>&1 | tail -4 > $O/t_r1f.log
timeout 600 python tools/pr_variants.py --scale 27 --variants "base:;lean:GTS_PR_LEAN=1;ww:GTS_PR_WW=1" --out $O/pr_lean.json > $O/pr_lean.log 2>&1
GTS_BENCH_CLOCKS=nvml timeout 900 python bench.py --no-cpu-baseline --no-e2e > $O/bench_nvml.json 2> $O/bench_nvml.err
GTS_BENCH_CLOCKS=off timeout 900 python bench.py --no-cpu-baseline --no-e2e > $O/bench_off.json 2> $O/bench_off.err
timeout 900 python bench.py --no-cpu-baseline --no-e2e > $O/bench_smi.json 2> $O/bench_smi.err
GTS_PR_LEAN=1 timeout 900 ncu --set full --clock-control none --import-source on -k regex:pr_scatter -s 3 -c 1 -o $O/pr_lean_full -f python tools/profile_run.py --algos pr --order > /dev/null 2>&1
ls -la $O
