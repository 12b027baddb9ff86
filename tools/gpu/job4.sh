cd ${GRAFT_REPO_ROOT:-/root/repo}
O=gpurun_out; mkdir -p $O
AB_TESTS="bfs" AB_ALGOS=bfs AB_VARIANTS="vh8k:;vh0:GTS_DEV_VHEAD=0;vh4k:GTS_DEV_VHEAD=4096;vh12k:GTS_DEV_VHEAD=12288" bash tools/gpu/job_ab.sh
timeout 900 python bench.py --steps 12 --warmup 3 --no-streamed --no-e2e --no-cpu-baseline > $O/bench_gc.json 2> $O/bench_gc.log
python -c "import json;d=json.load(open('$O/bench_gc.json'));print(d['value'], d['ms_per_step'],d['call_ms_each_step'],d['kernel_s_per_step'])"
