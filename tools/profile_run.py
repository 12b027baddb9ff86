"""Run selected GTS algorithms once on RMAT-S (for ncu captures; not a benchmark)."""
import argparse
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import inputs  # noqa: E402
import paper_conf_sigmod_0002apsk16_b200 as G  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--scale", type=int, default=27)
ap.add_argument("--algos", default="bfs,pr")
ap.add_argument("--pr-iters", type=int, default=2)
ap.add_argument("--page-bytes", type=int, default=1 << 20)
ap.add_argument("--reps", type=int, default=1)
a = ap.parse_args()
t = time.time()
g = inputs.rmat(a.scale)
w = inputs.edge_weights(g) if "sssp" in a.algos else None
gr = G.gts_build_pages(g.row_ptr, g.col, page_bytes=a.page_bytes)
grw = G.gts_build_pages(g.row_ptr, g.col, w, page_bytes=a.page_bytes) if w is not None else None
print("built", time.time() - t, flush=True)
ctx = G.gts_context_create(0)
for _ in range(a.reps):
    for algo in a.algos.split(","):
        if algo == "bfs":
            _, st = G.gts_bfs(ctx, gr, 0, timing=True)
        elif algo == "pr":
            _, st = G.gts_pagerank(ctx, gr, a.pr_iters, timing=True)
        elif algo == "sssp":
            _, st = G.gts_sssp(ctx, grw, 0, timing=True)
        elif algo == "wcc":
            _, st = G.gts_wcc(ctx, gr, timing=True)
        print(algo, st, flush=True)
