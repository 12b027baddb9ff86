#!/bin/bash
# re-entry check after container re-creation: smoke, full GPU suite, default bench line
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" > $O/s_smoke.log 2>&1
timeout 1800 python -m pytest tests -m gpu -x -q 2>&1 | tail -6 > $O/s_tests.log
timeout 1200 python bench.py > $O/s_bench.json 2> $O/s_bench.err
ls -la $O
