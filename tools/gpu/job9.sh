cd ${GRAFT_REPO_ROOT:-/root/repo}
O=gpurun_out; mkdir -p $O
AB_TESTS="wcc or plain or ordered" AB_ALGOS=wcc AB_VARIANTS="plain:;noplain:GTS_DEV_NO_WCC_PLAIN=1" bash tools/gpu/job_ab.sh
