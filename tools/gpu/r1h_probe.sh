#!/bin/bash
# bench with per-step call times (diagnose call-time variance), twice; step breakdown in between
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out
timeout 900 python bench.py --no-cpu-baseline --no-e2e --steps 5 > $O/bench_a.json 2> $O/bench_a.err
GTS_BENCH_CLOCKS=off timeout 900 python bench.py --no-cpu-baseline --no-e2e --steps 5 > $O/bench_b.json 2> $O/bench_b.err
ls -la $O
