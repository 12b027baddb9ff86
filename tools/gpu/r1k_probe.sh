#!/bin/bash
# clock sampling interference: NVML latency probe with control; bench (kicked NVML sampling) x2
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out
timeout 300 python tools/nvml_probe.py > $O/nvml_probe.txt 2>&1
timeout 900 python bench.py --no-cpu-baseline --no-e2e --steps 5 > $O/bench_k1.json 2> $O/bench_k1.err
timeout 900 python bench.py --no-cpu-baseline --no-e2e --steps 5 > $O/bench_k2.json 2> $O/bench_k2.err
ls -la $O
