#!/bin/bash
# 4-wide caller-order gathers + interleaved WCC finalize: timelines, full GPU suite, bench line
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out
for a in bfs wcc sssp; do
  timeout 600 python tools/bfs_timeline.py 27 $a > $O/v_tl_$a.txt 2>&1
done
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -6 > $O/v_tests.log
timeout 1200 python bench.py > $O/v_bench.json 2> $O/v_bench.err
python -c "import __graft_entry__ as g; g.smoke()" > $O/v_smoke.log 2>&1
ls -la $O
