cd ${GRAFT_REPO_ROOT:-/root/repo}
O=gpurun_out; mkdir -p $O
AB_TESTS="bfs or abi" AB_ALGOS=bfs AB_VARIANTS="" bash tools/gpu/job_ab.sh
