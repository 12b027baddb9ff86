cd ${GRAFT_REPO_ROOT:-/root/repo}
O=gpurun_out; mkdir -p $O
AB_TESTS="bfs" AB_ALGOS=bfs AB_VARIANTS="p6:;p4:GTS_DEV_PLAIN8=4;p3:GTS_DEV_PLAIN8=3;p2:GTS_DEV_PLAIN8=2;p1:GTS_DEV_PLAIN8=1" bash tools/gpu/job_ab.sh
