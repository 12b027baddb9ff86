#!/bin/bash
# weighted dense-tile variants: parity + SSSP A/B (0 default vs 2 never-dense)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "weighted or sssp or tile_walk" 2>&1 | tail -4 > $O/t_r1o.log
for wd in 0 2; do
  GTS_WDENSE=$wd GTS_BENCH_CLOCKS=off timeout 600 python bench.py --algos sssp --no-cpu-baseline --no-e2e --steps 5 > $O/bench_wd$wd.json 2> $O/bench_wd$wd.err
done
ls -la $O
