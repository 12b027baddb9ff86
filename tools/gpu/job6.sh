cd ${GRAFT_REPO_ROOT:-/root/repo}
O=gpurun_out; mkdir -p $O
AB_TESTS="bfs" AB_ALGOS=bfs AB_VARIANTS="plain:;noplain:GTS_DEV_NO_PLAIN=1" bash tools/gpu/job_ab.sh
timeout 900 python bench.py --steps 12 --warmup 3 --no-streamed --no-e2e --no-cpu-baseline > $O/bench6.json 2> $O/bench6.log
python -c "import json;d=json.load(open('$O/bench6.json'));print(d['value'], d['ms_per_step'],d['call_ms_each_step'],d['kernel_s_per_step'])"
