cd ${GRAFT_REPO_ROOT:-/root/repo}
O=gpurun_out; mkdir -p $O
timeout 900 python tools/kernel_ab.py --scale 27 --algos bfs,sssp,wcc --reps 5 > $O/ab5.jsonl 2> $O/ab5.log; cut -c1-250 $O/ab5.jsonl
timeout 1200 python tools/call_jitter.py --scale 27 --steps 20 > $O/jitter.txt 2> $O/jitter.log; echo "jitter rc=$?"; cat $O/jitter.txt; tail -3 $O/jitter.log
