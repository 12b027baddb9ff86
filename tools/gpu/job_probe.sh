cd ${GRAFT_REPO_ROOT:-/root/repo}
O=gpurun_out; mkdir -p $O
{ echo "== cgroup"; cat /sys/fs/cgroup/cpu.max; cat /sys/fs/cgroup/cpu.stat; nproc; cat /proc/loadavg; ps -eo pid,pcpu,comm --sort=-pcpu | head -15; } > $O/host_probe.txt 2>&1
bash tools/gpu/run.sh ncu 'bfs_expand' 3 --algos bfs
ncu -i $O/ncu_full.ncu-rep --page source --csv --print-source cuda > $O/bfs_src_cuda.csv 2>/dev/null
ncu -i $O/ncu_full.ncu-rep --page details --csv > $O/bfs_details.csv 2>/dev/null
bash tools/gpu/run.sh launches --algos sssp,wcc
{ echo "== cpu.stat before"; cat /sys/fs/cgroup/cpu.stat; } >> $O/host_probe.txt 2>&1
timeout 900 python bench.py --steps 12 --warmup 3 --no-streamed --no-e2e --no-cpu-baseline > $O/bench_var.json 2> $O/bench_var.log
{ echo "== cpu.stat after"; cat /sys/fs/cgroup/cpu.stat; } >> $O/host_probe.txt 2>&1
