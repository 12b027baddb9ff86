#!/bin/bash
# WCC deliver fusion parity + WCC bench; PageRank persisting-window size sweep; device L2 properties
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out
python -c "import torch; p=torch.cuda.get_device_properties(0); print(p); print('L2', p.L2_cache_size)" > $O/r_props.txt 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "wcc or degree_ordered or device_output" 2>&1 | tail -3 > $O/t_r1r.log
GTS_BENCH_CLOCKS=off timeout 600 python bench.py --algos wcc --no-cpu-baseline --no-e2e --steps 5 > $O/bench_wcc.json 2> $O/bench_wcc.err
timeout 900 python tools/pr_variants.py --scale 27 --variants "p96:;p32:GTS_L2_PERSIST=32;p64:GTS_L2_PERSIST=64;p80:GTS_L2_PERSIST=80;p112:GTS_L2_PERSIST=112;p0:GTS_L2_PERSIST=0" --out $O/pr_persist.json > $O/pr_persist.log 2>&1
ls -la $O
