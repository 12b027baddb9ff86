cd ${GRAFT_REPO_ROOT:-/root/repo}
O=gpurun_out; mkdir -p $O
AB_TESTS=sssp AB_ALGOS=sssp AB_VARIANTS="dexp:;nodexp:GTS_DEV_NO_DEXP=1" bash tools/gpu/job_ab.sh
for mode in kick off; do
  GTS_BENCH_CLOCKS=$mode timeout 900 python bench.py --steps 12 --warmup 3 --no-streamed --no-e2e --no-cpu-baseline > $O/bench_$mode.json 2> $O/bench_$mode.log
  python -c "import json;d=json.load(open('$O/bench_$mode.json'));print('$mode',d['ms_per_step'],d['call_ms_each_step']['sssp'],d['call_ms_each_step']['wcc'],d['clocks'])"
done
