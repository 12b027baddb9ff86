#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q 2>&1 | tail -3 > $O/t_persist.log
summ() { python -c "import json,sys;d=json.load(open(sys.argv[1]));print(sys.argv[1], 'GTEPS %.1f'%d['value'], 'ms/step %.1f'%d['ms_per_step'], {k:round(v*1e3,2) for k,v in d['kernel_s_per_step'].items()}, 'pr s/it %.2f ms'%(d['pagerank_s_per_iter']*1e3), 'sssp %.1f'%(d['sssp_s']*1e3), 'wcc %.1f'%(d['wcc_s']*1e3))" $1; }
timeout 400 python bench.py --no-cpu-baseline --no-e2e --steps 3 --warmup 3 > $O/bench_pA.json 2>/dev/null; summ $O/bench_pA.json
GTS_L2_PERSIST_BFS=0 GTS_L2_PERSIST_SSSP=0 GTS_L2_PERSIST_WCC=0 timeout 400 python bench.py --no-cpu-baseline --no-e2e --steps 3 --warmup 3 > $O/bench_pB.json 2>/dev/null; summ $O/bench_pB.json
GTS_WW=0 timeout 400 python bench.py --no-cpu-baseline --no-e2e --steps 3 --warmup 3 > $O/bench_pC.json 2>/dev/null; summ $O/bench_pC.json
