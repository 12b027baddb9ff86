#!/bin/bash
# 16-byte label_min, 2x grids for level_fill4 / pr_finish: timelines, full GPU suite, bench line, smoke
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out
for a in bfs wcc pr; do
  timeout 600 python tools/bfs_timeline.py 27 $a > $O/w_tl_$a.txt 2>&1
done
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -6 > $O/w_tests.log
timeout 1200 python bench.py > $O/w_bench.json 2> $O/w_bench.err
python -c "import __graft_entry__ as g; g.smoke()" > $O/w_smoke.log 2>&1
ls -la $O
