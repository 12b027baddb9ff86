# A/B job: GPU SSSP parity (+ full-size), then kernel_ab over the given variants
cd ${GRAFT_REPO_ROOT:-/root/repo}
O=gpurun_out; mkdir -p $O
timeout 1200 python -m pytest -m gpu -x -q -k "${AB_TESTS:-sssp}" tests > $O/ab_tests.log 2>&1; echo "tests rc=$?"; tail -3 $O/ab_tests.log
timeout 1500 python tools/kernel_ab.py --scale ${AB_SCALE:-27} --algos ${AB_ALGOS:-sssp} --reps ${AB_REPS:-5} --variants "$AB_VARIANTS" > $O/ab.jsonl 2> $O/ab.log; echo "ab rc=$?"; cat $O/ab.jsonl | cut -c1-400
